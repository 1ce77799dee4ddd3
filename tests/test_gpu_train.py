"""GPU parity of NEXT-3, proxy training, against the fp64 oracle: labels
bit-exact; loss and gradients of the fp32 trainer within fp32 accumulation error of the
oracle's; Adam within fp32 rounding; a full-size (C2 proxy shape, batch 32) property
check; and the loss falls when training on synthetic ground truth."""
import numpy as np
import pytest
import torch

import oracle
from synth import configs, video, weights

pytestmark = pytest.mark.gpu

otif = pytest.importorskip("paper_conf_sigmod_bastanim22_b200")
from paper_conf_sigmod_bastanim22_b200 import train  # noqa: E402

TINY_ENC, TINY_DEC = (2, 3, 4, 4, 4), 3


def gt(wl, frames_idx, clip=0):
    sc = video.make_scene(wl, clip=clip)
    boxes = []
    for i, t in enumerate(frames_idx):
        boxes += [(i, *b) for b in sc.gt_boxes(t) if b[0] < b[2] and b[1] < b[3]]
    return np.array(boxes, np.int32).reshape(-1, 5)


def layer_slices(enc, dec):
    out, off, cin = [], 0, 3
    for L, cout in enumerate(list(enc) + [dec, 1]):
        k = 1 if L == 6 else 3
        n = cout * k * k * cin + cout
        out.append(slice(off, off + n))
        off += n
        cin = cout
    return out


def rel_err(a, b):
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def test_labels_bit_exact():
    wl = configs.C2
    idx = list(range(0, 40, 2))
    boxes = gt(wl, idx)
    extra = np.array([[0, -50, -50, 10, 10], [1, 950, 530, 2000, 2000], [2, 5, 5, 5, 40], [99, 0, 0, 50, 50]],
                     np.int32)
    boxes = np.concatenate([boxes, extra])
    gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
    want = oracle.cell_labels(np.clip(boxes, [0, 0, 0, 0, 0], [99, wl.src_w, wl.src_h, wl.src_w, wl.src_h]),
                              len(idx), gh, gw, wl.cell, wl.src_w, wl.src_h)
    got = train.otif_cell_labels(torch.from_numpy(boxes).cuda(), len(idx), (gh, gw), wl.src_w, wl.src_h, wl.cell)
    assert np.array_equal(got.cpu().numpy(), want)


@pytest.mark.parametrize("case", ["tiny", "full_width"])
def test_gradients_match_oracle(case):
    if case == "tiny":
        rng = np.random.default_rng(5)
        img = rng.integers(0, 256, size=(3, 24, 40, 3), dtype=np.uint8)
        enc, dec, ns = TINY_ENC, TINY_DEC, 2
        blob = rng.normal(0, 0.5, size=oracle.proxy_n_weights(enc, dec)).astype(np.float32)
        gh, gw = oracle.proxy_grid(24, 40, ns)
        labels = (rng.uniform(size=(3, gh, gw)) < 0.4).astype(np.uint8)
    else:
        wl = configs.C1
        frames = video.frames(wl, 2).numpy()
        img = oracle.resize(frames, wl.proxy_h, wl.proxy_w)
        enc, dec, ns = configs.ENC_WIDTHS, configs.DEC_WIDTH, wl.n_strided
        blob = weights.proxy_weights()
        gh, gw = oracle.proxy_grid(wl.proxy_h, wl.proxy_w, ns)
        labels = oracle.cell_labels(gt(wl, [0, 1]), 2, gh, gw, wl.cell, wl.src_w, wl.src_h)
    loss, grad = oracle.proxy_grad(img, ns, enc, dec, blob.astype(np.float64), labels)
    tr = train.Trainer(img.shape[1], img.shape[2], ns, blob, max_batch=4, enc=enc, dec=dec)
    g_loss = tr.backward(torch.from_numpy(img).cuda(), torch.from_numpy(labels).cuda())
    g_grad = tr.grads_tensor().cpu().numpy().astype(np.float64)
    assert abs(float(g_loss.item()) - loss) <= 1e-5 * abs(loss)
    for L, sl in enumerate(layer_slices(enc, dec)):
        assert rel_err(g_grad[sl], grad[sl]) < 2e-4, (case, L, rel_err(g_grad[sl], grad[sl]))


def test_adam_matches_oracle():
    rng = np.random.default_rng(9)
    n = 10000
    w0 = rng.normal(size=n).astype(np.float32)
    ow, om, ov = w0.astype(np.float64), np.zeros(n), np.zeros(n)
    gw_, gm, gv = [torch.from_numpy(a).cuda() for a in (w0.copy(), np.zeros(n, np.float32), np.zeros(n, np.float32))]
    for t in range(1, 4):
        g = (rng.normal(size=n) * 10.0 ** rng.uniform(-6, 0, size=n)).astype(np.float32)
        oracle.adam(ow, om, ov, g.astype(np.float64), t, 1e-3)
        train.otif_adam_step(gw_, gm, gv, torch.from_numpy(g).cuda(), t, 1e-3)
    assert np.max(np.abs(gw_.cpu().numpy() - ow)) < 1e-6


def test_full_size_batch_is_mean_of_frames():
    """C2 proxy shape (135 x 240), batch 32 (the launch configuration the training
    script times): the batch gradient equals the mean of the per-frame gradients (the loss
    is a mean over cells), and frame 0's gradient matches the oracle."""
    wl = configs.C2
    n = 32
    idx = list(range(0, 4 * n, 4))
    frames = video.frames(wl, 4 * n, device="cuda")[idx]
    img = otif.otif_resize(frames, wl.proxy_h, wl.proxy_w)
    gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
    labels = train.otif_cell_labels(torch.from_numpy(gt(wl, idx)).cuda(), n, (gh, gw), wl.src_w, wl.src_h, wl.cell)
    blob = weights.proxy_weights()
    tr = train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, blob, max_batch=n)
    tr.backward(img, labels)
    g_batch = tr.grads_tensor().cpu().numpy().astype(np.float64)
    acc = np.zeros_like(g_batch)
    for i in range(n):
        tr.backward(img[i:i + 1], labels[i:i + 1])
        gi = tr.grads_tensor().cpu().numpy().astype(np.float64)
        acc += gi / n
        if i == 0:
            g0 = gi
    for sl in layer_slices(configs.ENC_WIDTHS, configs.DEC_WIDTH):
        assert rel_err(g_batch[sl], acc[sl]) < 2e-4
    loss, grad = oracle.proxy_grad(img[:1].cpu().numpy(), wl.n_strided, configs.ENC_WIDTHS, configs.DEC_WIDTH,
                                   blob.astype(np.float64), labels[:1].cpu().numpy())
    for sl in layer_slices(configs.ENC_WIDTHS, configs.DEC_WIDTH):
        assert rel_err(g0[sl], grad[sl]) < 2e-4


def test_training_lowers_the_loss():
    wl = configs.C1
    frames = video.frames(wl, 32, device="cuda")
    img = otif.otif_resize(frames, wl.proxy_h, wl.proxy_w)
    gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
    labels = train.otif_cell_labels(torch.from_numpy(gt(wl, range(32))).cuda(), 32, (gh, gw), wl.src_w, wl.src_h,
                                    wl.cell)
    tr = train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights(), max_batch=32)
    first = float(tr.step(img, labels, 1e-3).item())
    for _ in range(60):
        last = float(tr.step(img, labels, 1e-3).item())
    assert last < 0.7 * first


def test_simt_and_tensor_core_gemms_agree(tmp_path):
    """The tcgen05 3xTF32 training GEMMs (default) and the fp32 SIMT GEMMs
    (OTIF_TRAIN_SIMT=1, read once per process, hence a subprocess) give the same gradients
    within fp32 accumulation-order error, on the full-width C1 case."""
    import json
    import os
    import subprocess
    import sys
    code = r'''
import json, sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle
from synth import configs, video, weights
from paper_conf_sigmod_bastanim22_b200 import train
wl = configs.C1
img = oracle.resize(video.frames(wl, 2).numpy(), wl.proxy_h, wl.proxy_w)
gh, gw = oracle.proxy_grid(wl.proxy_h, wl.proxy_w, wl.n_strided)
lab = (np.arange(2 * gh * gw).reshape(2, gh, gw) % 3 == 0).astype(np.uint8)
tr = train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights(), max_batch=2)
loss = float(tr.backward(torch.from_numpy(img).cuda(), torch.from_numpy(lab).cuda()).item())
np.save(sys.argv[2], tr.grads_tensor().cpu().numpy())
print(json.dumps({"loss": loss}))
'''
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = {}
    for mode in ("tc", "simt"):
        env = dict(os.environ)
        env.pop("OTIF_TRAIN_SIMT", None)
        if mode == "simt":
            env["OTIF_TRAIN_SIMT"] = "1"
        path = str(tmp_path / f"{mode}.npy")
        r = subprocess.run([sys.executable, "-c", code, root, path], env=env, capture_output=True, text=True,
                           timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        out[mode] = (json.loads(r.stdout.strip().splitlines()[-1])["loss"], np.load(path).astype(np.float64))
    (l_tc, g_tc), (l_simt, g_simt) = out["tc"], out["simt"]
    assert abs(l_tc - l_simt) <= 1e-5 * abs(l_simt)
    for L, sl in enumerate(layer_slices(configs.ENC_WIDTHS, configs.DEC_WIDTH)):
        assert rel_err(g_tc[sl], g_simt[sl]) < 2e-4, (L, rel_err(g_tc[sl], g_simt[sl]))
