#!/bin/bash
# GPU box: the round's evidence -- gpu tests, smoke(), the default bench line (the driver's
# command), its ncu launch list, one ncu --set full capture of the C1 kernel, S1 / S1R lines.
TAG=${1:-r02}
OUT=gpurun_out/final_$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail -20 $OUT/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x --timeout=300 -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > $OUT/clocks.csv &
SMI=$!
timeout 600 python bench.py --gpus 1 --steps 20 --warmup 5 > $OUT/bench_C1.json 2> $OUT/bench_C1.err
kill $SMI
python -c "import json; d=json.load(open('$OUT/bench_C1.json')); print('C1', d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C1.csv \
    python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sfc_kernel -s 1 -c 1 \
    -o $OUT/prof_C1 -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-unfused > $OUT/ncu_C1.log 2>&1
for c in S1 S1R; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > $OUT/bench_$c.json 2> $OUT/bench_$c.err
  python -c "import json; d=json.load(open('$OUT/bench_$c.json')); print('$c', d['value'], d['roofline']['frac'], (d.get('e2e') or {}).get('value'))"
done
ls $OUT
