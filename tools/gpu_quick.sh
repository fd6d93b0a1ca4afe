# GPU box: parity tests + bench lines (CFGS, each "C:args" e.g. "C5:--k 3 --pkt-len 0")
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_gpu.log
for spec in ${CFGS:-C1}; do
  c=${spec%%:*}; a=""; [ "$c" != "$spec" ] && a=${spec#*:}; a=${a//_/ }; tag=$(echo "$spec" | tr -c 'A-Za-z0-9' '_')
  timeout 300 python bench.py --config $c $a --no-cpu --no-e2e $BENCH_ARGS > gpurun_out/q_$tag.json 2> gpurun_out/q_$tag.err; echo "$spec rc=$?"
  python -c "import json;d=json.load(open('gpurun_out/q_$tag.json'));u=d.get('unfused_baseline') or {};print('$spec', d['value'], d['unit'], d['ms_per_step'], d['roofline']['bound'], d['roofline']['frac'], 'unfused', u.get('value'))" 2>&1 | tail -1
  tail -2 gpurun_out/q_$tag.err
done
