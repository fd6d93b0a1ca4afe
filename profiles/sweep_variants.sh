#!/bin/bash
# A/B compile-time variants of libnfc.so on the same bench command (GPU box).
CFG=${1:-C1}
shift
for lib in variants/libnfc_*.so; do
  v=$(NFC_LIB=$PWD/$lib timeout 300 python bench.py --config $CFG --no-cpu --no-e2e "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "$lib $CFG $v"
done
