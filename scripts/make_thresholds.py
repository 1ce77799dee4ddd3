#!/usr/bin/env python
"""Freeze the proxy thresholds B_q per workload (reading R5).

B_q = the q-quantile of the quant=bf16 ORACLE scores over the first 32 frames of the
workload, rounded to fp32.  Calls only oracle/ (plus the shared input generator), so
no threshold ever comes from the CUDA path.  Output: tests/golden/thresholds.json.
"""
import json
import os
import sys
import time
from concurrent.futures import ThreadPoolExecutor

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from synth import configs, video, weights  # noqa: E402

QUANTILES = (0.5, 0.7, 0.8, 0.9)
N_FRAMES = 32


def oracle_scores(wl, blob, n=N_FRAMES):
    src = video.frames(wl, n).numpy()
    img = oracle.resize(src, wl.proxy_h, wl.proxy_w)
    with ThreadPoolExecutor(os.cpu_count()) as ex:
        parts = list(ex.map(lambda i: oracle.proxy_score(img[i:i + 1], wl.n_strided, configs.ENC_WIDTHS,
                                                         configs.DEC_WIDTH, blob, oracle.QUANT_BF16), range(n)))
    return np.concatenate(parts)


def main():
    blob = weights.proxy_weights()
    out = {"_about": __doc__.strip(), "n_frames": N_FRAMES, "workloads": {}}
    for name in ["C1", "C2", "C3"] + [w.name for w in configs.C4_SWEEP]:
        wl = configs.ALL[name]
        t = time.time()
        s = oracle_scores(wl, blob)
        entry = {}
        for q in QUANTILES:
            b = float(np.float32(np.quantile(s, q)))
            band = float((np.abs(s - b) <= 1e-3).mean())
            entry[str(q)] = {"B": b, "band_share": band}
        out["workloads"][name] = entry
        print(name, {k: round(v["B"], 6) for k, v in entry.items()}, f"{time.time() - t:.1f}s", flush=True)
    path = os.path.join(ROOT, "tests", "golden", "thresholds.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
