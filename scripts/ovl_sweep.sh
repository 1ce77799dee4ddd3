# overlap-mode sweep (A/B knobs via env); writes gpurun_out/s.log
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "overlap or pipeline" > gpurun_out/t.log 2>&1; echo pytest=$? >> gpurun_out/t.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-perfect --no-next3 --no-next4"
run() { echo "$1 | $2 | ov=$3" >> gpurun_out/s.log; env $2 timeout 200 $B --overlap $3 2>&1 | grep '^{' >> gpurun_out/s.log; }
run serial "X=1" 0
run mode1 "X=1" 2
run mode1 "X=1" 4
run mode1 "X=1" 8
run mode1 "OTIF_OVL_PACK_STAGE=16384" 4
run mode1 "OTIF_OVL_PACK_STAGES=6 OTIF_OVL_PACK_STAGE=8192" 4
run mode1 "OTIF_OVL_PROXY_SMEM=204800 OTIF_OVL_PACK_STAGE=8192" 4
