timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "overlap or pipeline" > gpurun_out/t.log 2>&1; echo pytest=$? >> gpurun_out/t.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-perfect --no-next3 --no-next4"
for ov in 0 4 8; do echo "ov=$ov" >> gpurun_out/s.log; timeout 200 $B --overlap $ov 2>&1 | grep '^{' >> gpurun_out/s.log; done
for st in 8192 16384; do echo "ov=4 stage=$st" >> gpurun_out/s.log; OTIF_OVL_PACK_STAGE=$st timeout 200 $B --overlap 4 2>&1 | grep '^{' >> gpurun_out/s.log; done
echo "ov=4 ctas=296 stage 8192" >> gpurun_out/s.log; OTIF_OVL_PACK_CTAS=296 OTIF_OVL_PACK_STAGE=8192 timeout 200 $B --overlap 4 2>&1 | grep '^{' >> gpurun_out/s.log
echo "ov=4 proxysmem=200k stage 8192" >> gpurun_out/s.log; OTIF_OVL_PROXY_SMEM=204800 OTIF_OVL_PACK_STAGE=8192 timeout 200 $B --overlap 4 2>&1 | grep '^{' >> gpurun_out/s.log
