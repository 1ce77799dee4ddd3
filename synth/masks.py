"""Seeded synthetic cell masks for the grouping (stage 4) and pack (stage 5) parity tests.

Input generation only: no arithmetic of the method lives here (components, grouping,
placement and costs are computed by the oracle and by the CUDA library independently).
Every recipe takes an explicit numpy Generator, so a failing case is reproduced from
its seed alone (the tests log the seed).

Recipes ("mask recipes"):
  sparse   independent cells at a per-frame density U[lo, hi] (a noisy proxy at a high
           threshold: scattered small components);
  blobs    1..max_objects axis-aligned rectangles of 1..max_side cells (object-shaped
           positives, the perfect-proxy structure of P:L153 at random positions);
  lattice  cells on a step x step lattice with random dropout and jitter: many small
           components (> 128 per frame on 23x40 grids) that are close enough to merge.
"""
from __future__ import annotations

import numpy as np


def sparse(rng: np.random.Generator, n: int, gh: int, gw: int, lo: float = 0.01, hi: float = 0.1) -> np.ndarray:
    dens = rng.uniform(lo, hi, size=(n, 1, 1))
    return (rng.random((n, gh, gw)) < dens).astype(np.uint8)


def blobs(rng: np.random.Generator, n: int, gh: int, gw: int, max_objects: int = 12, max_side: int = 4) -> np.ndarray:
    out = np.zeros((n, gh, gw), np.uint8)
    for f in range(n):
        for _ in range(int(rng.integers(1, max_objects + 1))):
            h = int(rng.integers(1, max_side + 1))
            w = int(rng.integers(1, max_side + 1))
            y = int(rng.integers(0, max(gh - h, 0) + 1))
            x = int(rng.integers(0, max(gw - w, 0) + 1))
            out[f, y:y + h, x:x + w] = 1
    return out


def lattice(rng: np.random.Generator, n: int, gh: int, gw: int, step: int = 2, keep: float = 0.8,
            jitter: float = 0.1) -> np.ndarray:
    out = np.zeros((n, gh, gw), np.uint8)
    base = np.zeros((gh, gw), bool)
    base[::step, ::step] = True
    for f in range(n):
        m = base & (rng.random((gh, gw)) < keep)
        m |= rng.random((gh, gw)) < jitter * 0.1
        out[f] = m
    return out
