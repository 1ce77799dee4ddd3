# A/B of tc_gemm build variants (OTIF_TC_K / OTIF_TC_MINB) on the NEXT-3 training step
for v in "-DOTIF_TC_K=16 -DOTIF_TC_MINB=2" "-DOTIF_TC_K=16 -DOTIF_TC_MINB=3" "-DOTIF_TC_K=32 -DOTIF_TC_MINB=1" "-DOTIF_TC_K=32 -DOTIF_TC_MINB=2"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "$v: $(python scripts/train_time.py 2>&1 | tail -1)"
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_train.py -x -q 2>&1 | tail -1
