"""Probe: can the copy engines move the full-frame detector batch (a device-to-device copy)
while the SMs run the tensor-bound proxy?  Times (CUDA events) a 7 GB D2D cudaMemcpyAsync
alone, the C2 proxy pass alone (stage path, 4500 frames), and both on two streams."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import cuda.bindings.runtime as rt
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights

wl = configs.C2
n = wl.n_frames
src = torch.empty((n, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
video.make_scene(wl).render(range(n), out=src)
dst = torch.empty_like(src)
img = otif.otif_resize(src, wl.proxy_h, wl.proxy_w)
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
ws = px.workspace(n)
out = torch.empty((n, 17, 30), dtype=torch.float32, device="cuda")
s_copy = torch.cuda.Stream()
nbytes = src.numel()


def copy(stream, parts=1):
    step = nbytes // parts
    for i in range(parts):
        err, = rt.cudaMemcpyAsync(dst.data_ptr() + i * step, src.data_ptr() + i * step, step,
                                  rt.cudaMemcpyKind.cudaMemcpyDeviceToDevice, stream.cuda_stream)
        assert err == rt.cudaError_t.cudaSuccess, err


def timed(fn, reps=3):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for _ in range(2):
    px.score(img, out=out, workspace=ws)
    copy(s_copy)
torch.cuda.synchronize()
res = {}
res["copy_alone_ms"] = timed(lambda: copy(torch.cuda.current_stream()))
res["copy_alone_GBps"] = 2 * nbytes / res["copy_alone_ms"] / 1e6
res["proxy_alone_ms"] = timed(lambda: px.score(img, out=out, workspace=ws))


def both():
    cur = torch.cuda.current_stream()
    s_copy.wait_stream(cur)
    copy(s_copy)
    px.score(img, out=out, workspace=ws)
    cur.wait_stream(s_copy)


res["both_ms"] = timed(both)
assert torch.equal(dst, src)
print(json.dumps({k: round(v, 3) for k, v in res.items()}))
