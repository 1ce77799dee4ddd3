timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "proxy or end_to_end or full_size or pipeline_host" > gpurun_out/t.log 2>&1; echo pytest=$? >> gpurun_out/t.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-perfect --no-next3 --no-next4"
echo "TS on" > gpurun_out/s.log; timeout 200 $B 2>&1 | grep '^{' >> gpurun_out/s.log
echo "TS off" >> gpurun_out/s.log; OTIF_E12_TS=0 timeout 200 $B 2>&1 | grep '^{' >> gpurun_out/s.log
