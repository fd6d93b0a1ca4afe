#!/bin/bash
# GPU-box script: one ncu --set full capture of the fused kernel for a bench config.
# Usage (under gpurun): bash profiles/prof_one.sh <tag> <bench args...>
TAG=$1; shift
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sfc_kernel -s 1 -c 1 \
    -o $OUT/prof_${TAG} -f python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-unfused "$@" > $OUT/ncu_${TAG}.log 2>&1
echo "ncu rc=$?"
