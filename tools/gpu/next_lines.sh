#!/bin/bash
# GPU box: NEXT-2 / NEXT-3 bench lines (N3 at 200 / 1K / 10K rules x 64 / 1500 B, NX2 FW / IDS)
TAG=${1:-r02d}
OUT=gpurun_out/next_$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || exit 1
for r in 200 1000 10000; do for pl in 64 1500; do
  timeout 300 python bench.py --config N3 --acl-rules $r --pkt-len $pl --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/N3_${r}_${pl}.json 2> $OUT/N3_${r}_${pl}.err
  python -c "import json; d=json.load(open('$OUT/N3_${r}_${pl}.json')); print('N3', $r, $pl, d['value'], d['roofline']['frac'], (d.get('unfused_baseline') or {}).get('fused_speedup'))"
done; done
for c in NX2_FW NX2_IDS; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/$c.json 2> $OUT/$c.err
  python -c "import json; d=json.load(open('$OUT/$c.json')); print('$c', d['value'], (d.get('next2_configs') or {}).keys())"
done
