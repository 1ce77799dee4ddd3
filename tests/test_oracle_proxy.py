"""Pins for the oracle's proxy CNN (readings R1–R4).

* conv layers: torch.nn.functional.conv2d in fp64 (an independent library routine)
  on the same tensors;
* bf16 rounding: torch's fp32 -> bf16 conversion (RNE) and hand-computed ties;
* grid shapes: the values PAPER.md prints (tests/golden/paper_pins.json);
* threshold: strictness and the two degenerate thresholds.
"""
import json
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
from synth import configs, video, weights

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")


def test_round_bf16_hand_ties():
    # spacing of bf16 at 1.0 is 2^-7; halfway cases round to the even significand
    assert oracle.round_bf16(1.0 + 2 ** -8) == 1.0
    assert oracle.round_bf16(1.0 + 3 * 2 ** -8) == 1.0 + 2 ** -6
    assert oracle.round_bf16(-(1.0 + 3 * 2 ** -8)) == -(1.0 + 2 ** -6)
    assert oracle.round_bf16(1.0 + 2 ** -8 + 2 ** -30) == 1.0 + 2 ** -7
    assert oracle.round_bf16(0.0) == 0.0
    assert oracle.round_bf16(3.0) == 3.0


def test_round_bf16_matches_torch_on_fp32_values():
    rng = np.random.default_rng(1)
    x = np.concatenate([rng.standard_normal(20000) * 10 ** rng.uniform(-6, 6, 20000),
                        (rng.integers(0, 2 ** 16, 2000).astype(np.float64) + 0.5) * 2.0 ** -15]).astype(np.float32)
    ref = torch.from_numpy(x).to(torch.bfloat16).to(torch.float64).numpy()
    got = np.array([oracle.round_bf16(float(v)) for v in x])
    assert np.array_equal(got, ref)


def _torch_conv(x, w, b, stride, relu):
    xt = torch.from_numpy(x).permute(0, 3, 1, 2)
    wt = torch.from_numpy(w).permute(0, 3, 1, 2)
    k = w.shape[1]
    y = F.conv2d(xt, wt, torch.from_numpy(b), stride=stride, padding=(k - 1) // 2)
    if relu:
        y = torch.relu(y)
    return y.permute(0, 2, 3, 1).numpy()


@pytest.mark.parametrize("h,w,cin,cout,k,stride", [
    (9, 13, 3, 8, 3, 2), (10, 12, 5, 4, 3, 2), (7, 11, 16, 8, 3, 1), (17, 30, 8, 6, 3, 1),
    (6, 5, 12, 1, 1, 1), (1, 1, 4, 3, 3, 1), (2, 3, 4, 3, 3, 2)])
def test_conv_matches_torch_conv2d_fp64(h, w, cin, cout, k, stride):
    rng = np.random.default_rng(h * 100 + w)
    x = rng.standard_normal((2, h, w, cin))
    wt = rng.standard_normal((cout, k, k, cin))
    b = rng.standard_normal(cout)
    for relu in (False, True):
        got = oracle.conv(x, wt, b, stride, relu=relu)
        ref = _torch_conv(x, wt, b, stride, relu)
        assert got.shape == ref.shape == (2, -(-h // stride), -(-w // stride), cout)
        assert np.allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_conv_bf16_output_rounding():
    rng = np.random.default_rng(3)
    x = rng.standard_normal((1, 8, 8, 4))
    wt = rng.standard_normal((5, 3, 3, 4))
    b = rng.standard_normal(5)
    got = oracle.conv(x, wt, b, 1, relu=True, round_bf16_out=True)
    ref = _torch_conv(x, wt, b, 1, True)
    # every output is a bf16 value within half a bf16 ulp of the exact result
    as_bf16 = torch.from_numpy(got).to(torch.float32).to(torch.bfloat16).to(torch.float64).numpy()
    assert np.array_equal(as_bf16, got)
    ulp = np.where(ref != 0, 2.0 ** (np.floor(np.log2(np.abs(ref) + 1e-300)) - 7), 0)
    assert (np.abs(got - ref) <= ulp / 2 + 1e-15).all()


def _torch_proxy(img, n_strided, blob, quant):
    """Independent fp64 proxy: torch conv2d chain (reading R2/R4)."""
    layers = weights.split(blob)
    x = (torch.from_numpy(img).double() - 128.0) / 128.0
    x = x.permute(0, 3, 1, 2)

    def q(t):
        return t.float().to(torch.bfloat16).double() if quant else t

    for i, (w, b) in enumerate(layers):
        wt = torch.from_numpy(w).double().permute(0, 3, 1, 2)
        if quant:
            wt = q(wt)
        stride = 2 if (i < 5 and i < n_strided) else 1
        x = F.conv2d(x, wt, torch.from_numpy(b).double(), stride=stride, padding=(w.shape[1] - 1) // 2)
        if i < 6:
            x = torch.relu(x)
            if quant:
                x = q(x)
    return torch.sigmoid(x[:, 0]).numpy()


@pytest.mark.parametrize("quant", [oracle.QUANT_NONE, oracle.QUANT_BF16])
def test_proxy_matches_torch_chain(quant):
    img = oracle.resize(video.frames(configs.C1, 2).numpy(), 64, 104)
    blob = weights.proxy_weights()
    got = oracle.proxy_score(img, 3, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, quant)
    ref = _torch_proxy(img, 3, blob, quant)
    assert got.shape == (2, 8, 13)
    if quant == oracle.QUANT_NONE:
        assert np.allclose(got, ref, rtol=0, atol=1e-12)
    else:
        # torch rounds fp64 -> fp32 -> bf16 (double rounding) where the oracle rounds once;
        # rare near-tie flips of one bf16 activation propagate a little downstream
        d = np.abs(got - ref)
        assert d.max() < 5e-3 and d.mean() < 5e-4
    assert ((got > 0) & (got < 1)).all()


def test_quant_none_vs_bf16_close():
    img = oracle.resize(video.frames(configs.C1, 1).numpy(), 64, 104)
    blob = weights.proxy_weights()
    a = oracle.proxy_score(img, 3, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, oracle.QUANT_NONE)
    b = oracle.proxy_score(img, 3, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, oracle.QUANT_BF16)
    assert np.abs(a - b).max() < 2e-2 and np.abs(a - b).max() > 0


def test_grid_shapes_from_paper():
    pins = json.load(open(GOLDEN))["proxy_grid"]
    for p in pins:
        assert oracle.proxy_grid(p["input_h"], p["input_w"], p["n_strided"]) == (p["grid_h"], p["grid_w"]), p["cite"]
    # and through a full (tiny-width) proxy at the paper's S = 32
    enc, dec = (4, 4, 4, 4, 4), 4
    rng = np.random.default_rng(0)
    blob = rng.uniform(-0.3, 0.3, oracle.proxy_n_weights(enc, dec)).astype(np.float32)
    for p in pins:
        img = rng.integers(0, 256, (1, p["input_h"], p["input_w"], 3), dtype=np.uint8)
        s = oracle.proxy_score(img, 5, enc, dec, blob)
        assert s.shape == (1, p["grid_h"], p["grid_w"])


def test_workload_grids():
    # reading R1/R14: grid = ceil(detector / cell) = ceil(proxy / S)
    for wl in list(configs.ALL.values()):
        gh, gw = oracle.proxy_grid(wl.proxy_h, wl.proxy_w, wl.n_strided)
        assert (gh, gw) == (-(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)), wl.name


def test_threshold_strict_and_degenerate():
    s = np.array([[0.1, 0.5, 0.7], [0.5, 0.9, 0.2]], np.float32).astype(np.float64)  # fp32-exact
    m = oracle.threshold(s, 0.5)
    assert m.tolist() == [[0, 0, 1], [0, 1, 0]]
    assert oracle.threshold(s, float(s.max())).sum() == 0
    assert oracle.threshold(s, float(np.nextafter(np.float32(s.min()), np.float32(-1)))).all()
    # B is an fp32 constant compared in fp64: 0.1 (fp64) > float32(0.1)?
    assert oracle.threshold(np.array([0.1]), 0.1)[0] == int(0.1 > float(np.float32(0.1)))
