# GPU box: N3 parity with the default lib, then N3 (200/1K/10K, 64 B) + C1 A/B against variants/
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "n3 or c3 or c1_full" 2>&1 | tail -1
for r in 1 2; do for a in "N3 --acl-rules 1000" "N3 --acl-rules 10000" "N3 --acl-rules 200" "C3"; do for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $(ls $PWD/variants/libnfc_*.so); do
 v=$(NFC_LIB=$lib timeout 300 python bench.py --config $a --no-cpu --no-e2e --no-unfused 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'])")
 echo "r$r $(basename $lib) $a $v"; done; done; done
