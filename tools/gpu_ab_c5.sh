# GPU box: parity of variants/libnfc_spec6.so on the C1/C5 tests, then C5 k2-k4 + C1 A/B
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
NFC_LIB=$PWD/variants/libnfc_spec6.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "c1 or c5 or unfused or parallel" 2>&1 | tail -1
for r in 1 2; do for a in "C5 --k 2" "C5 --k 3" "C5 --k 4" "C1"; do for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $PWD/variants/libnfc_spec6.so; do
 v=$(NFC_LIB=$lib timeout 300 python bench.py --config $a --no-cpu --no-e2e --no-unfused 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'])")
 echo "r$r $(basename $lib) $a $v"; done; done; done
