# GPU box: build, parity tests, smoke, bench lines for C1-C4 (+C5 sweep with SWEEP=1, N3 lines with N3=1), launch list + ncu full capture of PROF configs
TAG=${TAG:-r01f}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
nproc; lscpu | grep "Model name"
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
for c in C1 C2 C3 C4; do timeout 400 python bench.py --config $c --cpu-seconds 5 > gpurun_out/bench_${TAG}_$c.json 2> gpurun_out/bench_${TAG}_$c.err; echo "$c rc=$?"; cat gpurun_out/bench_${TAG}_$c.json; tail -2 gpurun_out/bench_${TAG}_$c.err; done
if [ -n "$SWEEP" ]; then for k in 1 2 3 4 5 6; do timeout 300 python bench.py --config C5 --k $k --no-cpu --no-e2e > gpurun_out/bench_${TAG}_C5_k$k.json 2>gpurun_out/bench_${TAG}_C5_k$k.err; cat gpurun_out/bench_${TAG}_C5_k$k.json; done; fi
if [ -n "$N3" ]; then for a in 200 1000 10000; do for pl in 64 128 1500; do timeout 300 python bench.py --config N3 --acl-rules $a --pkt-len $pl --no-cpu --no-e2e > gpurun_out/bench_${TAG}_N3_${a}_${pl}.json 2>gpurun_out/bench_${TAG}_N3_${a}_${pl}.err; cat gpurun_out/bench_${TAG}_N3_${a}_${pl}.json; done; done; fi
for c in ${PROF:-C1 C3}; do
  a=""; [ "$c" = "N3" ] && a="--acl-rules 1000"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_$c.csv \
    python bench.py --config $c $a --steps 3 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo "launches $c rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sfc_kernel -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_$c -f python bench.py --config $c $a --steps 1 --warmup 1 --no-e2e --no-cpu --no-unfused > gpurun_out/ncu_${TAG}_$c.log 2>&1; echo "ncu $c rc=$?"
done
