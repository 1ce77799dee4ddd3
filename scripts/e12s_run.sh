# fused-resize s2d E1+E2 kernel: parity then stage times (default build)
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
t=$(timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "proxy or full_size or end_to_end or pack_overlap or host_vs_stages" 2>&1 | tail -3 | tr '\n' ' ')
echo "[$OTIF_NVCC_EXTRA] $t | $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1) | $(timeout 120 python scripts/e12_stage_time.py 2>&1 | tail -1)" >> gpurun_out/e12s_run.log
