python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in 0 50000 1000000; do
  timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu --no-unfused --match-ppm $m > gpurun_out/exp1_$m.json 2>gpurun_out/exp1_$m.err
  python -c "import json; d=json.load(open('gpurun_out/exp1_$m.json')); print('match_ppm $m', d['value'], d['roofline']['frac'])" 2>&1 | tail -1
done
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q --durations=20 -p no:cacheprovider > gpurun_out/pt_full.log 2>&1
echo "fullsize rc=$?"; tail -30 gpurun_out/pt_full.log
