# A/B of e12 build variants (nvcc -D flags) on the proxy pass time (scripts/e12_time.py),
# each variant checked against the oracle first (proxy parity tests)
for v in "" "-DOTIF_E12_ACC=1 -DOTIF_E12_E1SLOTS=3" ""; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "proxy_parity or full_size" 2>&1 | tail -1)
  echo "[$v] $t | $(python scripts/e12_time.py 2>&1 | tail -1) | $(python scripts/e12_time.py 2>&1 | tail -1)" >> gpurun_out/e12_ab.log
done
