# A/B of the tc_gemm register prefetch (OTIF_TC_PREFETCH: 0 none, 1 two sets, 2 three sets) and stage depth on the NEXT-3 training step
for v in "-DOTIF_TC_PREFETCH=1" "-DOTIF_TC_PREFETCH=2" "-DOTIF_TC_PREFETCH=1 -DOTIF_TC_K=32 -DOTIF_TC_MINB=1" "-DOTIF_TC_PREFETCH=2 -DOTIF_TC_MINB=1" "-DOTIF_TC_PREFETCH=1"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "$v: $(timeout 120 python scripts/train_time.py 2>&1 | tail -1)"
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 400 python -m pytest tests/test_gpu_train.py -x -q 2>&1 | tail -2
