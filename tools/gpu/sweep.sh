#!/bin/bash
# GPU box: the SURVEY 8(d) sweep -- C5 k=1..6 x {64, 512, 1500, IMIX} plus C2/C3/C4 -- one bench
# line each (no CPU leg, no baselines: the C1 line carries those), into gpurun_out/sweep_<tag>/.
TAG=${1:-r02}
OUT=gpurun_out/sweep_$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || exit 1
run() {  # name, bench args
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-unfused --no-e2e $2 > $OUT/$1.json 2> $OUT/$1.err
  python - $OUT/$1.json $1 <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1])); r = d["roofline"]
    x = f" dpi_frac={r['dpi_lookups']['frac']}" if "dpi_lookups" in r else ""
    print(f"{sys.argv[2]:14s} {d['value']:10.1f} Mpps {d['gbps']:9.1f} Gbps frac={r['frac']} ({r['bound']}){x}")
except Exception as e:
    print(sys.argv[2], "ERR", e)
PY
}
for c in C2 C3 C4; do run $c "--config $c"; done
for k in 1 2 3 4 5 6; do
  for pl in 64 512 1500 0; do run C5_k${k}_$pl "--config C5 --k $k --pkt-len $pl"; done
done
