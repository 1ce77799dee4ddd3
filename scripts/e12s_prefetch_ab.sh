# e12s: L2 bulk prefetch of the source rows 1 / 2 tiles ahead of the converters (warp 0) vs
# none; per-stage times on C2 and C3 (scripts/e12_stage_time.py), parity first
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-e12s_prefetch}_ab.log
for v in "" "-DOTIF_E12S_PREFETCH=1" "-DOTIF_E12S_PREFETCH=2" ""; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_parity.py -q -x -k "fused_scores" 2>&1 | tail -1)
  echo "[$v] $t | C2 $(timeout 120 python scripts/e12_stage_time.py C2 2>&1 | tail -1) | C3 $(timeout 200 python scripts/e12_stage_time.py C3 2>&1 | tail -1)" >> $LOG
done
