"""The native runtime's stage-5 scheduling (otif_pipeline_desc.pack_overlap): the pack of
device batch b copied by spare warps of batch b+1's tensor-bound proxy kernels (E4..D1)
plus a drain kernel.  The detector batches are byte-identical to the oracle's identity
crop of the same windows, and windows / counts / counters are identical
to the serial schedule, for full-frame and sub-frame (windowing-active) windows."""
import numpy as np
import pytest
import torch

import oracle
from synth import configs, video, weights
from tests.helpers import threshold

pytestmark = pytest.mark.gpu

otif = pytest.importorskip("paper_conf_sigmod_bastanim22_b200")


def _oracle_batches(frames, windows, sizes, caps, sh, sw):
    win = np.zeros(len(windows), oracle.WINDOW_DTYPE)
    for i, f in enumerate(oracle.WINDOW_DTYPE.names):
        win[f] = windows[:, i]
    return oracle.pack_windows(frames, sh, sw, win, sizes, caps)[0]


@pytest.mark.parametrize("case", ["random_full_frame", "trained_subframe"])
def test_pack_overlap_matches_serial_and_oracle(case):
    n = 96
    if case == "random_full_frame":
        wl = configs.C2
        blob = weights.proxy_weights()
        thr, sizes = threshold("C2", 0.7), list(wl.sizes)
    else:
        # off-peak traffic and a proxy trained by NEXT-3 on later frames of the same camera:
        # object-aligned sub-frame windows of several sizes (the windowing-active path)
        from scripts import train_proxy
        wl = configs.C2S
        blob, _ = train_proxy.train_weights(wl, steps=200, batch=32, clip=0, start=4 * n)
        thr, sizes = 0.5, [(960, 540), (224, 160), (320, 512), (128, 128), (256, 224)]
    src_a = video.frames(wl, n).cuda()
    src_b = video.frames(wl, n, start=n).cuda()
    caps = [n * 6 if (s[0], s[1]) != (wl.src_w, wl.src_h) else n for s in sizes]
    ref = otif.Pipeline(wl, blob, thr, max_batch=n, sizes=sizes, batch_cap=caps, pack_overlap=0)
    ovl = otif.Pipeline(wl, blob, thr, max_batch=n, sizes=sizes, batch_cap=caps, pack_overlap=2)
    # call 1 (batch A): pack pending; call 2 (batch B): A's pack rides in B's proxy
    ovl.run_device(src_a)
    ovl.run_device(src_b, frame_base=n)
    torch.cuda.synchronize()
    got_a = [ovl.detector_batch(s).cpu().numpy() for s in range(len(sizes))]
    ovl.flush()
    got_b = [ovl.detector_batch(s).cpu().numpy() for s in range(len(sizes))]
    # serial reference and the oracle crop of the same windows
    for src, got, base in ((src_a, got_a, 0), (src_b, got_b, n)):
        win, counts, sc, tot = ref.run_host(src.cpu().contiguous())
        exp = _oracle_batches(src.cpu().numpy(), win, sizes, caps, wl.src_h, wl.src_w)
        for s in range(len(sizes)):
            k = min(int(sc[s]), caps[s])
            assert np.array_equal(got[s][:k], exp[s][:k]), (case, base, s)
    # counters (windows, hash, per-size, dropped, packed pixels) equal the serial schedule's
    ref.reset_counters()
    ref.run_device(src_a)
    ref.run_device(src_b, frame_base=n)
    ovl.reset_counters()
    ovl.run_device(src_a)
    ovl.run_device(src_b, frame_base=n)
    ovl.flush()
    torch.cuda.synchronize()
    assert torch.equal(ref.counters().cpu(), ovl.counters().cpu())
    if case == "trained_subframe":
        c = ref.counters().cpu().tolist()
        assert sum(c[6:10]) > n          # sub-frame windows were packed


def test_pack_overlap_multi_batch_call():
    """pack_overlap = 1 with several device batches per call (the pack of batch b inside
    batch b+1's proxy, the last drained before returning): counters equal the serial run."""
    wl = configs.C1
    blob = weights.proxy_weights()
    src = video.frames(wl, 70).cuda()
    a = otif.Pipeline(wl, blob, threshold("C1", 0.7), max_batch=16, pack_overlap=0)
    b = otif.Pipeline(wl, blob, threshold("C1", 0.7), max_batch=16, pack_overlap=1)
    a.run_device(src)
    b.run_device(src)
    torch.cuda.synchronize()
    assert torch.equal(a.counters().cpu(), b.counters().cpu())
    for s in range(len(wl.sizes)):
        assert torch.equal(a.detector_batch(s), b.detector_batch(s))
