# per-role hand-off timeline of the band kernel (CTA 0, bands 20..35), trace build
OTIF_NVCC_EXTRA="-DOTIF_E12_TRACE_BUILD" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
python - <<'PY' > gpurun_out/e12b_trace.log 2>&1
import torch, paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
wl = configs.C2
img = torch.randint(0, 256, (4500, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
s = px.score(img); torch.cuda.synchronize()
PY
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
for v in "" "-DOTIF_E12B=0"; do
  OTIF_NVCC_EXTRA="$v" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  echo "[$v] $(python scripts/e12_stage_time.py)" >> gpurun_out/e12b_stage.log
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
