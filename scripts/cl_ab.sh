# A/B of weight-sharing CTA pairs (OTIF_CONV_CL_LAYERS) x pack overlap on the C2 headline;
# each build's proxy parity checked first
B="python bench.py --headline-only --no-e2e --no-cpu-baseline --no-c5 --steps 30"
run() {  # $1 = nvcc flags, $2 = pack_overlap
  OTIF_NVCC_EXTRA="$1" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  t=$(timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipeline.py -q -x -k "proxy_parity or full_size or pack_overlap" 2>&1 | tail -1)
  echo "[$1 ov$2] $t :: $($B --pack-overlap $2 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['roofline']['layers'].items()}, round(d['stages']['pack']['ms_per_step'],3), d['clocks']['sm_mhz'])")" >> gpurun_out/cl_ab.log
}
run "-DOTIF_CONV_CL_LAYERS=0x1C" 0
run "-DOTIF_CONV_CL_LAYERS=0x0" 0
run "-DOTIF_CONV_CL_LAYERS=0x1C" 2
run "-DOTIF_CONV_CL_LAYERS=0x0" 2
run "-DOTIF_CONV_CL_LAYERS=0x1E" 0
run "-DOTIF_CONV_CL_LAYERS=0x1C -DOTIF_PJ_LAYERS=0x1C" 2
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
