# GPU box: gpu tests (unless NOTEST), then the default lib and every variants/libnfc_*.so on the
# bench configs (CFGS), REPS rounds interleaved (box-to-box and run-to-run variance)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
if [ -z "$NOTEST" ]; then timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log; fi
one() {  # lib cfg
  NFC_LIB=$1 timeout 300 python bench.py --config $2 --no-cpu --no-e2e --no-unfused $BENCH_ARGS 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])"
}
for r in $(seq ${REPS:-2}); do
for c in ${CFGS:-C1}; do
  for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $(ls variants/libnfc_*.so 2>/dev/null); do
    echo "r$r $(basename $lib) $c $(one $lib $c)"
  done
done
done
