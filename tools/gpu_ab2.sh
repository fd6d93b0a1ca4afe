# GPU box: A/B of the default lib and every variants/libnfc_*.so on bench argument sets
# (ARGS: ';'-separated bench argument strings), REPS rounds interleaved
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
IFS=';' read -ra SETS <<< "${ARGS:---config C1}"
for r in $(seq ${REPS:-1}); do
for a in "${SETS[@]}"; do
  for lib in $PWD/paper_conf_hpca_hul18_b200/libnfc.so $(ls variants/libnfc_*.so 2>/dev/null); do
    v=$(NFC_LIB=$lib timeout 300 python bench.py $a --no-cpu --no-e2e --no-unfused 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
    echo "r$r [$a] $(basename $lib) $v"
  done
done
done
