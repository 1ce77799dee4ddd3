set -e
OTIF_NVCC_EXTRA="-DOTIF_E12_TRACE_BUILD ${TRACE_J0:+-DOTIF_E12_TRACE_J0=$TRACE_J0}" python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)"
for t in 1; do
  echo "== OTIF_E12_TRACE=$t"
  OTIF_E12_TRACE=$t python - <<'PY'
import torch, paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
wl = configs.C2
img = torch.randint(0, 256, (4500, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
s = px.score(img); torch.cuda.synchronize()
PY
done
