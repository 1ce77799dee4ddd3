# fused pack copy warps: claim one unit ahead and prefetch it to L2 (OTIF_PJ_PREFETCH) vs not;
# pipeline tests, then the headline bench (pack_overlap 2) and C3 stage times
mkdir -p gpurun_out
LOG=gpurun_out/${TAG:-pj_prefetch}_ab.log
for v in "" "-DOTIF_PJ_PREFETCH=0" "" "-DOTIF_PJ_PREFETCH=0"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 400 python -m pytest tests/test_gpu_pipeline.py tests/test_gpu_windowing.py -q -x -k "pack" 2>&1 | tail -1)
  b=$(timeout 600 python bench.py --headline-only --no-e2e --no-cpu-baseline --no-c5 --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, round(d['stages']['pack']['slot_and_drain_ms_per_step'],3), d['clocks']['sm_mhz'])")
  echo "[$v] $t | $b | C3 $(timeout 200 python scripts/e12_stage_time.py C3 2 0.7 2>&1 | tail -1)" >> $LOG
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
