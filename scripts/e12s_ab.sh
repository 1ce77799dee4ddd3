# space-to-depth (e12s) vs tile (e12) variant of the fused E1+E2 kernel: parity then stage times
mkdir -p gpurun_out
for v in "" "-DOTIF_E12S=0" ""; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "proxy or full_size or end_to_end or pack_overlap" 2>&1 | tail -3 | tr '\n' ' ')
  echo "[$v] $t | $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1) | $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1)" >> gpurun_out/e12s_ab.log
done
