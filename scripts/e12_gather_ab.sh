# E1+E2 gather: two rows per thread together (OTIF_E12_GATHER2) vs the rolled loop
for v in "" "-DOTIF_E12_GATHER2=0" "" "-DOTIF_E12_GATHER2=0"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_parity.py -q -x -k "proxy or full_size or end_to_end" 2>&1 | tail -1)
  echo "[$v] $t | $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1)" >> gpurun_out/e12_gather_ab.log
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
