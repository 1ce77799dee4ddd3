# e12s_umma_kernel buffer counts (slabs x plane buffers) vs the L1 left to the converters'
# source loads: parity first, then per-stage times on C2 and C3 (scripts/e12_stage_time.py)
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-e12s_smem}_ab.log
while read -r v; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "proxy or full_size or pack_overlap or stages or fused_scores" 2>&1 | tail -1)
  echo "[$v] $t | C2 $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1) | C2 $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1) | C3 $(timeout 200 python scripts/e12_stage_time.py C3 2>&1 | tail -1)" >> $LOG
done <<VARS
${VARIANTS:-
-DOTIF_E12S_NP=1
-DOTIF_E12S_NSLAB=1
-DOTIF_E12S_NSLAB=1 -DOTIF_E12S_NP=1}
VARS
