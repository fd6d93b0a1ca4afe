mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for lib in paper_conf_hpca_hul18_b200/libnfc.so $(ls variants/libnfc_*.so); do NFC_LIB=$PWD/$lib timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "c2 or c4 or c5 or C1 or n3" 2>&1 | tail -1; done
for r in 1 2; do for c in C2 C4; do for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $(ls variants/libnfc_*.so); do
 v=$(NFC_LIB=$lib timeout 300 python bench.py --config $c --no-cpu --no-e2e --no-unfused 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'], d['config']['launch']['grid'])")
 echo "r$r $(basename $lib) $c $v"; done; done; done
