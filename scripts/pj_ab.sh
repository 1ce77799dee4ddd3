# A/B of the fused-pack copy role (build flags) on the C2 headline, pack_overlap 2 vs 0
B="python bench.py --headline-only --no-e2e --no-cpu-baseline --no-c5 --steps 30"
for v in "-DOTIF_PJ_WARPS=8" "-DOTIF_PJ_WARPS=4" "-DOTIF_PJ_WARPS=4 -DOTIF_PJ_UNROLL=4" "-DOTIF_PJ_WARPS=8 -DOTIF_PJ_LAYERS=0x18" "-DOTIF_PJ_WARPS=2 -DOTIF_PJ_UNROLL=8" "-DOTIF_PJ_WARPS=8 -DOTIF_PJ_LAYERS=0x1E"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $($B --pack-overlap 2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, round(d['stages']['pack']['ms_per_step'],3), d['clocks']['sm_mhz'])")" >> gpurun_out/pj_ab.log
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
echo "[ov0] $($B --pack-overlap 0 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, round(d['stages']['pack']['ms_per_step'],3), d['clocks']['sm_mhz'])")" >> gpurun_out/pj_ab.log
