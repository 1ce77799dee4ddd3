"""Per-stage times (pipeline stage events) on a workload (default C2, the headline; argv[1] names another), 5 steps."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights
wl = getattr(configs, sys.argv[1]) if len(sys.argv) > 1 else configs.C2
src = torch.empty((wl.n_frames, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
video.make_scene(wl).render(range(wl.n_frames), out=src)
pipe = otif.Pipeline(wl, weights.proxy_weights(), 0.5, max_batch=wl.n_frames)
pipe.run_device(src)
torch.cuda.synchronize()
pipe.set_timing(True)
for _ in range(5):
    pipe.run_device(src)
ms, _ = pipe.stage_ms()
print(json.dumps({k: round(v / 5, 4) for k, v in ms.items()}))
