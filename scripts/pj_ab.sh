# A/B of the fused-pack copy role (build flags) on the C2 headline (pack_overlap 2 unless noted)
B="python bench.py --headline-only --no-e2e --no-cpu-baseline --no-c5 --steps 30"
run() {  # $1 = nvcc flags, $2 = pack_overlap
  OTIF_NVCC_EXTRA="$1" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$1 ov$2] $($B --pack-overlap $2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, round(d['stages']['pack']['ms_per_step'],3), d['clocks']['sm_mhz'])")" >> gpurun_out/pj_ab2.log
}
run "-DOTIF_PJ_E12=4 -DOTIF_PJ_LAYERS=0x18" 2
run "-DOTIF_PJ_E12=4 -DOTIF_PJ_LAYERS=0x10" 2
run "-DOTIF_PJ_E12=4 -DOTIF_PJ_LAYERS=0x0" 2
run "-DOTIF_PJ_E12=0 -DOTIF_PJ_LAYERS=0x18" 2
run "-DOTIF_PJ_E12=4 -DOTIF_PJ_LAYERS=0x18" 0
run "-DOTIF_PJ_E12=0 -DOTIF_PJ_LAYERS=0x18" 0
run "-DOTIF_PJ_E12=4 -DOTIF_PJ_LAYERS=0x18" 2
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
