# GPU box: ncu full capture of the fused kernel for one config (source counters on)
CFG=${1:-C1}; TAG=${2:-x}; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sfc_kernel -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${CFG} -f python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > gpurun_out/ncu_${TAG}_${CFG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_${TAG}_${CFG}.log
