# A/B of two builds of libotif.so on the same box: $1 = extra nvcc flags for build B
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-next3 --no-next4"
echo "A: default" > gpurun_out/s.log; timeout 200 $B 2>&1 | grep '^{' >> gpurun_out/s.log
OTIF_NVCC_EXTRA="$1" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)"
echo "B: $1" >> gpurun_out/s.log; timeout 200 $B 2>&1 | grep '^{' >> gpurun_out/s.log
echo "A again" >> gpurun_out/s.log; python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)"
timeout 200 $B 2>&1 | grep '^{' >> gpurun_out/s.log
