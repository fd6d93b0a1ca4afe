# GPU box: gpu tests, then the default lib and every variants/libnfc_*.so on the bench configs (CFGS)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
if [ -z "$NOTEST" ]; then timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log; fi
for c in ${CFGS:-C1}; do
  v=$(timeout 300 python bench.py --config $c --no-cpu --no-e2e $BENCH_ARGS 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "default $c $v"
  bash profiles/sweep_variants.sh $c $BENCH_ARGS
done
