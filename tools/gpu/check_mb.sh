python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build4.log 2>&1
timeout 900 python -m pytest tests/test_gpu_gen.py tests/test_gpu_multi.py tests/test_gpu_parity.py -x -q > gpurun_out/pt4.log 2>&1
tail -3 gpurun_out/pt4.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu --no-unfused > gpurun_out/b4_mb.json 2> gpurun_out/b4_mb.err
timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu --no-unfused --batch-pkts 0 > gpurun_out/b4_sb.json 2> gpurun_out/b4_sb.err
python - <<'PY'
import json
for f in ("b4_mb","b4_sb"):
    try:
        d=json.load(open(f"gpurun_out/{f}.json")); print(f, d["value"], d["roofline"]["frac"], d["config"]["batches_per_step_per_gpu"], d["clocks"])
    except Exception as e: print(f, "ERR", e, open(f"gpurun_out/{f}.err").read()[-2000:])
PY
