# A/B of the weight-gradient split-K target (OTIF_WGRAD_WAVES CTAs per SM) on the NEXT-3 training step
for v in "-DOTIF_WGRAD_WAVES=2" "-DOTIF_WGRAD_WAVES=3" "-DOTIF_WGRAD_WAVES=4" "-DOTIF_WGRAD_WAVES=6" "-DOTIF_WGRAD_WAVES=2"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "$v: $(timeout 120 python scripts/train_time.py 2>&1 | tail -1)"
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 400 python -m pytest tests/test_gpu_train.py -x -q 2>&1 | tail -2
