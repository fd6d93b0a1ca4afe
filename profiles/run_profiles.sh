#!/bin/bash
# GPU-box script: bench lines + ncu evidence for the fused SFC kernel.
# Usage (under gpurun): bash profiles/run_profiles.sh <tag> [config]
set -x
TAG=${1:-r01}
CFG=${2:-C1}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python bench.py --config $CFG $BENCH_ARGS > $OUT/bench_${TAG}_${CFG}.json 2> $OUT/bench_${TAG}_${CFG}.err
# launch list of the same command (cold-cache, serialised; compare shares not absolutes)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${TAG}_${CFG}.csv \
    python bench.py --config $CFG --steps 3 --warmup 1 --no-e2e --no-cpu $BENCH_ARGS > /dev/null 2>&1
# one full capture of the top kernel
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sfc_kernel -s 1 -c 1 \
    -o $OUT/prof_${TAG}_${CFG} -f python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu $BENCH_ARGS > $OUT/ncu_${TAG}_${CFG}.log 2>&1
ls -la $OUT
