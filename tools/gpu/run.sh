#!/bin/bash
# GPU-box helper: build, run the given pytest selection, then optional bench lines.
# Usage: bash tools/gpu/run.sh "<pytest args>" "<bench args 1>" "<bench args 2>" ...
TESTS=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then
  eval "timeout 1500 python -m pytest $TESTS -v -x --timeout=300" > gpurun_out/pytest.log 2>&1
  echo "pytest rc=$?"; grep -E "PASSED|FAILED|ERROR|Timeout" gpurun_out/pytest.log | tail -3; tail -4 gpurun_out/pytest.log
fi
i=0
for B in "$@"; do
  i=$((i+1))
  timeout 600 python bench.py $B > gpurun_out/bench_$i.json 2> gpurun_out/bench_$i.err
  python - "$i" "$B" <<'PY'
import json, sys
i, args = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/bench_{i}.json"))
    r = d["roofline"]
    print(f"[{args}] {d['value']} {d['unit']} frac={r['frac']} {r['bound']} clk={d['clocks'].get('sm_mhz')} launches={d.get('gpu_launches')}")
except Exception as e:
    print(f"[{args}] ERR {e}: " + open(f"gpurun_out/bench_{i}.err").read()[-1500:])
PY
done
