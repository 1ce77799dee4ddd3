"""Random-init proxy weights (north_star: "random-init weights of the paper's proxy shape").

Reading R3: numpy PCG64(seed=20220612); per layer in the order
E1..E5, D1, D2: W[Cout][kh][kw][Cin] ~ He-uniform U(±sqrt(6/fan_in)), then
b[Cout] ~ U(±0.05).  D2 (the 1x1 head) is He-uniform x2 with its mean subtracted
(zero-sum) and bias 0, which spreads the scores so that few cells sit near a
quantile threshold.  One fp32 blob, passed unchanged to
both the oracle and the CUDA library.
"""
from __future__ import annotations

import numpy as np

from .configs import DEC_WIDTH, ENC_WIDTHS, WEIGHT_SEED


def layer_shapes(enc=ENC_WIDTHS, dec=DEC_WIDTH):
    """[(cout, k, cin)] for E1..E5, D1, D2."""
    shapes, c = [], 3
    for e in enc:
        shapes.append((e, 3, c))
        c = e
    shapes.append((dec, 3, c))
    shapes.append((1, 1, dec))
    return shapes


def proxy_weights(seed: int = WEIGHT_SEED, enc=ENC_WIDTHS, dec=DEC_WIDTH, head_gain: float = 2.0) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    parts = []
    shapes = layer_shapes(enc, dec)
    for i, (cout, k, cin) in enumerate(shapes):
        fan_in = k * k * cin
        bound = np.sqrt(6.0 / fan_in)
        w = rng.uniform(-bound, bound, size=(cout, k, k, cin))
        if i == len(shapes) - 1:
            w = w * head_gain
            w = w - w.mean()
            b = np.zeros(cout)
        else:
            b = rng.uniform(-0.05, 0.05, size=cout)
        parts.append(w.reshape(-1))
        parts.append(b.reshape(-1))
    return np.concatenate(parts).astype(np.float32)


def split(blob: np.ndarray, enc=ENC_WIDTHS, dec=DEC_WIDTH):
    """blob -> [(W[cout,k,k,cin], b[cout])] (fp32 views)."""
    out, off = [], 0
    for (cout, k, cin) in layer_shapes(enc, dec):
        nw = cout * k * k * cin
        w = blob[off:off + nw].reshape(cout, k, k, cin)
        off += nw
        b = blob[off:off + cout]
        off += cout
        out.append((w, b))
    assert off == blob.size
    return out
