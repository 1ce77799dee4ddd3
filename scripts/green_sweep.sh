# SM-partitioned overlap (green contexts): OTIF_OVL_GREEN = SMs of the memory partition
OTIF_OVL_GREEN=32 timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "overlap" > gpurun_out/t.log 2>&1; echo pytest=$? >> gpurun_out/t.log
B="python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --no-perfect --no-next3 --no-next4"
run() { echo "$1 | ov=$2" >> gpurun_out/s.log; env $1 timeout 200 $B --overlap $2 2>&1 | grep '^{' >> gpurun_out/s.log; }
run "X=1" 0
run "OTIF_OVL_GREEN=24" 4
run "OTIF_OVL_GREEN=32" 4
run "OTIF_OVL_GREEN=40" 4
run "OTIF_OVL_GREEN=32" 8
run "OTIF_OVL_GREEN=48" 8
