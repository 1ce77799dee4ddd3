# e12s with the 1-tile L2 prefetch: converter load flavour (OTIF_E12S_LD) and plane buffers
# (OTIF_E12S_NP) A/B; per-stage times on C2 and C3 (scripts/e12_stage_time.py), parity first
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-e12s_ld}_ab.log
while read -r v; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_parity.py -q -x -k "fused_scores" 2>&1 | tail -1)
  echo "[$v] $t | C2 $(timeout 120 python scripts/e12_stage_time.py C2 2>&1 | tail -1) | C2 $(timeout 120 python scripts/e12_stage_time.py C2 2>&1 | tail -1) | C3 $(timeout 200 python scripts/e12_stage_time.py C3 2>&1 | tail -1)" >> $LOG
done <<VARS
${VARIANTS:-
-DOTIF_E12S_LD=3
-DOTIF_E12S_LD=1
-DOTIF_E12S_NP=1
-DOTIF_E12S_LD=3 -DOTIF_E12S_NP=1}
VARS
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
