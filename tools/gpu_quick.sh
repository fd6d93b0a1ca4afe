# GPU box: parity tests + a C1 bench line (+ optional extra bench configs)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu.log
for c in ${CFGS:-C1}; do
  timeout 300 python bench.py --config $c --no-cpu --no-e2e $BENCH_ARGS > gpurun_out/q_$c.json 2> gpurun_out/q_$c.err; echo "$c rc=$?"
  python -c "import json;d=json.load(open('gpurun_out/q_$c.json'));print('$c', d['value'], d['unit'], d['ms_per_step'], d['roofline']['frac'])" 2>&1 | tail -1
  tail -2 gpurun_out/q_$c.err
done
