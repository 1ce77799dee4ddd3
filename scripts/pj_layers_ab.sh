# fused-pack layer sets (OTIF_PJ_LAYERS: bit li, 0 = E2 .. 4 = D1) on C3 and C2 with the
# frozen q = 0.7 threshold (the bench's), pack_overlap 2: per-stage and step times
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-pj_layers}_ab.log
for v in ${VARIANTS:-0x18 0x1C 0x1A 0x1E}; do
  OTIF_NVCC_EXTRA="-DOTIF_PJ_LAYERS=$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_pipeline.py -q -x 2>&1 | tail -1)
  echo "[$v] $t | C3 $(timeout 200 python scripts/e12_stage_time.py C3 2 0.7 2>&1 | tail -1) | C2 $(timeout 200 python scripts/e12_stage_time.py C2 2 0.7 2>&1 | tail -1) | C4b $(timeout 200 python scripts/e12_stage_time.py C4b 2 0.7 2>&1 | tail -1)" >> $LOG
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
