"""Pins for the NEXT-3 oracle, proxy training: label closed forms and an
independent rasteriser, convolution backward and the whole-proxy gradient against torch
autograd (fp64) and central finite differences, Adam against torch.optim.Adam."""
import numpy as np
import pytest
import torch

import oracle
from synth import configs, video, weights

TINY_ENC, TINY_DEC = (2, 3, 4, 4, 4), 3


# ----------------------------------------------------------------------------- labels
def test_labels_closed_forms():
    # 416x256 frame, cell 32 -> 13 x 8 grid
    b = np.array([[0, 40, 40, 50, 50],        # inside cell (1, 1)
                  [0, 0, 0, 32, 32],          # exactly cell (0, 0): half-open, touches nothing else
                  [1, 100, 200, 170, 256],    # spans cells x 3..5, y 6..7
                  [1, 400, 10, 416, 20],      # clipped edge cell x = 12 (covers 384..416)
                  [0, 300, 100, 300, 200]],   # empty (x0 == x1): intersects nothing
                 np.int32)
    lab = oracle.cell_labels(b, 2, 8, 13, 32, 416, 256)
    assert lab.shape == (2, 8, 13)
    want0 = np.zeros((8, 13), np.uint8)
    want0[1, 1] = want0[0, 0] = 1
    want1 = np.zeros((8, 13), np.uint8)
    want1[6:8, 3:6] = 1
    want1[0, 12] = 1
    assert np.array_equal(lab[0], want0) and np.array_equal(lab[1], want1)


def test_labels_match_independent_rasteriser():
    wl = configs.C2
    sc = video.make_scene(wl)
    gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
    boxes, masks = [], []
    for t in range(20):
        bx = sc.gt_boxes(t)
        masks.append(video.gt_mask(bx, wl.src_w, wl.src_h, wl.cell))
        boxes += [(t, *b) for b in bx if b[0] < b[2] and b[1] < b[3]]
    lab = oracle.cell_labels(np.array(boxes), 20, gh, gw, wl.cell, wl.src_w, wl.src_h)
    assert np.array_equal(lab, np.stack(masks))


# ----------------------------------------------------------------------------- conv backward
@pytest.mark.parametrize("h,w,cin,cout,k,s", [(7, 9, 3, 4, 3, 1), (8, 11, 5, 2, 3, 2), (5, 6, 4, 1, 1, 1),
                                             (9, 7, 2, 3, 3, 2)])
def test_conv_backward_matches_autograd(h, w, cin, cout, k, s):
    rng = np.random.default_rng(h * 100 + w)
    x = rng.normal(size=(2, h, w, cin))
    wt = rng.normal(size=(cout, k, k, cin))
    ho, wo = -(-h // s), -(-w // s)
    dy = rng.normal(size=(2, ho, wo, cout))
    dx, dW, db = oracle.conv_backward(x, wt, dy, s)
    tx = torch.tensor(x).permute(0, 3, 1, 2).requires_grad_()
    tw = torch.tensor(wt).permute(0, 3, 1, 2).requires_grad_()
    tb = torch.zeros(cout, dtype=torch.float64, requires_grad=True)
    y = torch.nn.functional.conv2d(tx, tw, tb, stride=s, padding=(k - 1) // 2)
    y.backward(torch.tensor(dy).permute(0, 3, 1, 2))
    assert np.allclose(dx, tx.grad.permute(0, 2, 3, 1).numpy(), atol=1e-12)
    assert np.allclose(dW, tw.grad.permute(0, 2, 3, 1).numpy(), atol=1e-12)
    assert np.allclose(db, tb.grad.numpy(), atol=1e-12)


# ----------------------------------------------------------------------------- whole proxy
def torch_proxy_loss(img, n_strided, enc, dec, blob, labels):
    """Independent torch fp64 model of the proxy (NCHW conv2d chain) + mean BCE-with-logits."""
    x = (torch.tensor(img, dtype=torch.float64).permute(0, 3, 1, 2) - 128.0) / 128.0
    widths = list(enc) + [dec, 1]
    cin, off, params = 3, 0, []
    for L, cout in enumerate(widths):
        k = 1 if L == 6 else 3
        nw = cout * k * k * cin
        W = torch.tensor(blob[off:off + nw].reshape(cout, k, k, cin)).permute(0, 3, 1, 2).contiguous().requires_grad_()
        off += nw
        b = torch.tensor(blob[off:off + cout]).requires_grad_()
        off += cout
        params += [W, b]
        s = 2 if (L < 5 and L < n_strided) else 1
        x = torch.nn.functional.conv2d(x, W, b, stride=s, padding=(k - 1) // 2)
        if L < 6:
            x = torch.relu(x)
        cin = cout
    z = x[:, 0]
    loss = torch.nn.functional.binary_cross_entropy_with_logits(z, torch.tensor(labels, dtype=torch.float64))
    loss.backward()
    grad = np.concatenate([np.concatenate([W.grad.permute(0, 2, 3, 1).reshape(-1).numpy(), b.grad.numpy()])
                           for W, b in zip(params[0::2], params[1::2])])
    return float(loss.detach()), grad


def test_proxy_grad_matches_autograd_full_width():
    wl = configs.C1
    img = oracle.resize(video.frames(wl, 2).numpy(), wl.proxy_h, wl.proxy_w)[:, :40, :48].copy()
    blob = weights.proxy_weights().astype(np.float64)
    gh, gw = oracle.proxy_grid(40, 48, wl.n_strided)
    labels = (np.random.default_rng(1).uniform(size=(2, gh, gw)) < 0.3).astype(np.uint8)
    loss, grad = oracle.proxy_grad(img, wl.n_strided, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, labels)
    tl, tg = torch_proxy_loss(img, wl.n_strided, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, labels)
    assert loss == pytest.approx(tl, rel=1e-12)
    assert np.max(np.abs(grad - tg)) <= 1e-10 * max(1.0, np.max(np.abs(tg)))


def test_proxy_grad_finite_differences():
    rng = np.random.default_rng(7)
    img = rng.integers(0, 256, size=(2, 12, 20, 3), dtype=np.uint8)
    nw = oracle.proxy_n_weights(TINY_ENC, TINY_DEC)
    blob = rng.normal(0, 0.5, size=nw)
    gh, gw = oracle.proxy_grid(12, 20, 2)
    labels = (rng.uniform(size=(2, gh, gw)) < 0.5).astype(np.uint8)
    loss, grad = oracle.proxy_grad(img, 2, TINY_ENC, TINY_DEC, blob, labels)
    h = 1e-6
    for i in rng.choice(nw, 40, replace=False):
        bp, bm = blob.copy(), blob.copy()
        bp[i] += h
        bm[i] -= h
        fd = (oracle.proxy_grad(img, 2, TINY_ENC, TINY_DEC, bp, labels)[0] -
              oracle.proxy_grad(img, 2, TINY_ENC, TINY_DEC, bm, labels)[0]) / (2 * h)
        assert abs(fd - grad[i]) <= 1e-6 * max(1.0, abs(fd))


def test_bce_closed_form():
    # all-zero weights: z = 0 everywhere -> loss = ln 2, dL/dz = (1/2 - y)/M
    rng = np.random.default_rng(3)
    img = rng.integers(0, 256, size=(1, 8, 8, 3), dtype=np.uint8)
    blob = np.zeros(oracle.proxy_n_weights(TINY_ENC, TINY_DEC))
    gh, gw = oracle.proxy_grid(8, 8, 1)
    labels = (rng.uniform(size=(1, gh, gw)) < 0.5).astype(np.uint8)
    loss, grad = oracle.proxy_grad(img, 1, TINY_ENC, TINY_DEC, blob, labels)
    assert loss == pytest.approx(np.log(2.0), rel=1e-15)
    M = gh * gw
    assert grad[-1] == pytest.approx(np.sum(0.5 - labels) / M, abs=1e-15)     # D2 bias gradient


# ----------------------------------------------------------------------------- Adam
def test_adam_matches_torch():
    rng = np.random.default_rng(11)
    w0 = rng.normal(size=50)
    w, m, v = w0.copy(), np.zeros(50), np.zeros(50)
    tw = torch.tensor(w0, requires_grad=True)
    opt = torch.optim.Adam([tw], lr=1e-2, betas=(0.9, 0.999), eps=1e-8)
    for t in range(1, 4):
        g = rng.normal(size=50)
        oracle.adam(w, m, v, g, t, 1e-2)
        opt.zero_grad()
        tw.grad = torch.tensor(g)
        opt.step()
        assert np.allclose(w, tw.detach().numpy(), rtol=0, atol=1e-14)
