# grouping-kernel A/B: windowing parity tests, then per-stage times with the bench threshold
# (q = 0.7) on C3, C4b and C2 (scripts/e12_stage_time.py); VARIANTS = nvcc flag sets ("-" = none)
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-sel}_ab.log
for v in ${VARIANTS:--}; do
  [ "$v" = "-" ] && v=""
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 900 python -m pytest tests/test_gpu_windowing.py tests/test_gpu_parity.py -q -x -k "select or windowing or group or mask or stress or full_size or stages or end_to_end" 2>&1 | tail -1)
  echo "[$v] $t | C3 $(timeout 200 python scripts/e12_stage_time.py C3 0 0.7 2>&1 | tail -1) | C4b $(timeout 200 python scripts/e12_stage_time.py C4b 0 0.7 2>&1 | tail -1) | C2 $(timeout 200 python scripts/e12_stage_time.py C2 0 0.7 2>&1 | tail -1)" >> $LOG
done
