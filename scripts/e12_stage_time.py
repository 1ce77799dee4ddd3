"""Per-stage times (pipeline stage events) on a workload, 5 steps.
usage: e12_stage_time.py [workload (default C2, the headline)] [pack_overlap (default 0)] [quantile q] [proxy_batch]
With q the threshold is the frozen B_q of the workload (tests/golden/thresholds.json),
else 0.5; "total" = the mean step time (CUDA events around each run_device)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
wl = getattr(configs, name, None) or {w.name: w for w in configs.C4_SWEEP}[name]
ov = int(sys.argv[2]) if len(sys.argv) > 2 else 0
thr = 0.5
if len(sys.argv) > 3:
    from tests.helpers import threshold
    thr = threshold(wl.name, float(sys.argv[3])) if float(sys.argv[3]) > 0 else 0.5
src = torch.empty((wl.n_frames, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
video.make_scene(wl).render(range(wl.n_frames), out=src)
pb = int(sys.argv[4]) if len(sys.argv) > 4 else 0
pipe = otif.Pipeline(wl, weights.proxy_weights(), thr, max_batch=wl.n_frames, pack_overlap=ov, proxy_batch=pb)
pipe.run_device(src)
torch.cuda.synchronize()
pipe.set_timing(True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    pipe.run_device(src)
if ov:
    pipe.flush()
e1.record()
torch.cuda.synchronize()
ms, _ = pipe.stage_ms()
out = {k: round(v / 5, 4) for k, v in ms.items()}
out["total"] = round(e0.elapsed_time(e1) / 5, 4)
print(json.dumps(out))
