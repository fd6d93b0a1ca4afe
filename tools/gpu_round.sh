set -x
mkdir -p gpurun_out
nproc; lscpu | grep "Model name"
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_gpu.log
for c in C1 C2 C3 C4; do timeout 400 python bench.py --config $c --cpu-seconds 5 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo "$c rc=$?"; cat gpurun_out/bench_$c.json; tail -3 gpurun_out/bench_$c.err; done
for k in 1 2 3 4 5 6; do timeout 300 python bench.py --config C5 --k $k --no-cpu --no-e2e > gpurun_out/bench_C5_k$k.json 2>gpurun_out/bench_C5_k$k.err; cat gpurun_out/bench_C5_k$k.json; done
