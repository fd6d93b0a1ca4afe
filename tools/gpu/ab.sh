#!/bin/bash
# GPU box A/B: the default lib and every variants/libnfc_*.so on each bench-args string
# (one per line in $CASES), REPS rounds interleaved.  Prints value and frac per run.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
one() {  # lib args
  NFC_LIB=$1 timeout 300 python bench.py --no-cpu --no-e2e --no-unfused --steps ${STEPS:-10} --warmup 3 $2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'], d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
for r in $(seq ${REPS:-2}); do
  while IFS= read -r c; do
    [ -z "$c" ] && continue
    for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $(ls variants/libnfc_*.so 2>/dev/null); do
      echo "r$r $(basename $lib) [$c] $(one $lib "$c")"
    done
  done <<< "$CASES"
done
