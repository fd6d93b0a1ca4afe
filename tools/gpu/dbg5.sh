python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build5.log 2>&1
python tools/gpu/gen_debug.py > gpurun_out/gen_debug.txt 2>&1
bash profiles/prof_one.sh c1mb --config C1
cat gpurun_out/gen_debug.txt | head -30
