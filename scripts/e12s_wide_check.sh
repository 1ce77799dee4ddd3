mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "proxy or full_size or pack_overlap or stages or fused_scores or end_to_end" > gpurun_out/c4d_tests.log 2>&1; tail -3 gpurun_out/c4d_tests.log
for w in C4d C4a C2 C3; do echo "$w $(timeout 200 python scripts/e12_stage_time.py $w 0 0.7 2>&1 | tail -1)"; done
