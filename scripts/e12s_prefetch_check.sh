mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py tests/test_gpu_c5.py -q -x > gpurun_out/pf_tests.log 2>&1; tail -2 gpurun_out/pf_tests.log
for w in C2 C3 C4b C4d C1; do echo "$w $(timeout 200 python scripts/e12_stage_time.py $w 0 0.7 2>&1 | tail -1)"; done
timeout 600 python bench.py --headline-only --no-e2e --no-cpu-baseline --no-c5 --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, d['clocks'])"
