"""Shared test helpers: frozen thresholds, oracle fan-out over host threads, window
record conversion.  Test infrastructure (may call oracle/)."""
from __future__ import annotations

import json
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

import oracle
from synth import configs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
BAND = 1e-3  # "except for cells whose oracle score lies within 1e-3 of the threshold" (north_star)


THRESHOLD_NAMES = tuple(json.load(open(os.path.join(GOLDEN, "thresholds.json")))["workloads"].keys())


def threshold(name: str, q: float = 0.7) -> float:
    d = json.load(open(os.path.join(GOLDEN, "thresholds.json")))
    return d["workloads"][name][str(q)]["B"]


def oracle_scores(img: np.ndarray, wl, blob, quant=oracle.QUANT_BF16, workers: int | None = None) -> np.ndarray:
    n = img.shape[0]
    workers = workers or os.cpu_count()
    with ThreadPoolExecutor(workers) as ex:
        parts = list(ex.map(lambda i: oracle.proxy_score(img[i:i + 1], wl.n_strided, configs.ENC_WIDTHS,
                                                         configs.DEC_WIDTH, blob, quant), range(n)))
    return np.concatenate(parts)


def windows_np(win_t, total: int) -> np.ndarray:
    """GPU int32 [cap, 6] -> structured array like oracle.WINDOW_DTYPE."""
    a = win_t[:total].cpu().numpy().astype(np.int32)
    out = np.zeros(total, oracle.WINDOW_DTYPE)
    for i, f in enumerate(oracle.WINDOW_DTYPE.names):
        out[f] = a[:, i]
    return out


def as_tuples(w) -> list:
    return [tuple(int(r[f]) for f in oracle.WINDOW_DTYPE.names) for r in w]
