#!/bin/bash
# E1+E2 fused-kernel hand-off timeline (CTA 0, first 16 plane jobs) and the tcgen05 MMA
# issue-rate microbenchmark.  Debug only: rebuilds libotif.so with -DOTIF_E12_TRACE_BUILD.
set -e
cd "$(dirname "$0")/.."
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mma_rate scripts/micro/mma_rate.cu && /tmp/mma_rate
OTIF_NVCC_EXTRA=-DOTIF_E12_TRACE_BUILD python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)"
for t in 1 3; do
  echo "== OTIF_E12_TRACE=$t"
  OTIF_E12_TRACE=$t python - <<'PY'
import torch, paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
wl = configs.C2
img = torch.randint(0, 256, (1024, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
s = px.score(img); torch.cuda.synchronize()
PY
done
python -c "from paper_conf_sigmod_bastanim22_b200 import build as b; b.build(force=True)"
