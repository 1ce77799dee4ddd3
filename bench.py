#!/usr/bin/env python
"""bench.py — OTIF proxy + windowing hot path on B200: frames/s, rooflines, CPU oracle baseline.

A "step" is one pass of the whole hot path (resize -> proxy CNN -> threshold ->
connected components + window selection -> crop/pack) over the BASELINE.json configs[1]
workload: a 960x540 traffic clip, 10 min at 30 fps sampled every 4th frame = 4500 frames
(C2, synthetic, rendered on the device before timing), resident in HBM (7.0 GB of u8,
larger than the 126 MB L2, so no L2 flush is needed between steps).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl otif|reference]

N > 1: one process per GPU over NCCL.  Without torchrun in the environment the script
re-launches itself under `torch.distributed.run` (127.0.0.1).  Every rank processes its
own 4500-frame clip set (weak scaling, no data-path collective); per-rank counters are
combined with one all_gather at the end.  The "c5" object runs the fixed 8-hour corpus
(480 one-minute clips) sharded by contiguous clip ranges.

Beside the headline line (random-init proxy, north_star) the JSON carries: the other
BASELINE configs (C1, C3, C4b, C4d) with their own rooflines and oracle samples, the
windowing-active path (trained proxy + the NEXT-1 window set W*, and the perfect proxy
under W*), the NEXT-3 / NEXT-4 rows, e2e through the C ABI with host buffers, and the
oracle timed on the host cores.  --impl reference times the CPU oracle (oracle/, plain
fp64 C) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import tempfile
import time
from concurrent.futures import ThreadPoolExecutor

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "proxy+windowing frames/sec at 1/2/4/8 B200; % HBM / tensor-pipe peak"
FALLBACK_PEAKS = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}


# --------------------------------------------------------------------------- helpers
def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return d, "measured (MEASURED_PEAKS.json)"
    return dict(FALLBACK_PEAKS), "fallback (B200_PROFILING.md)"


def threshold_for(name: str, q: float = 0.7) -> float:
    d = json.load(open(os.path.join(ROOT, "tests", "golden", "thresholds.json")))
    return d["workloads"][name][str(q)]["B"]


def conv_macs_per_frame(wl, enc, dec):
    """Algorithmic MACs of E1..E5, D1 per frame: Ho*Wo*Cout*Cin*k^2 with Ho = ceil(Hi/2) for
    strided layers (P:L135 shape, readings R1/R2); and the D2 head's MACs."""
    h, w, c = wl.proxy_h, wl.proxy_w, 3
    layers = []
    for i in range(6):
        cout = enc[i] if i < 5 else dec
        s = 2 if (i < 5 and i < wl.n_strided) else 1
        h, w = -(-h // s), -(-w // s)
        layers.append(h * w * cout * c * 9)
        c = cout
    head = h * w * dec
    return layers, head   # layers[0] = E1, [1..5] = E2..E5, D1


def conv_act_bytes_per_frame(wl, enc, dec):
    """Algorithmic activation bytes of E2..E5, D1 per frame (bf16 input + output; D1 writes the
    fp32 scores): the HBM bytes a layer-by-layer schedule must move (weights are L2-resident)."""
    h, w, c = wl.proxy_h, wl.proxy_w, 3
    dims = []
    for i in range(6):
        cout = enc[i] if i < 5 else dec
        s = 2 if (i < 5 and i < wl.n_strided) else 1
        h2, w2 = -(-h // s), -(-w // s)
        dims.append((h * w * c, h2 * w2 * cout))
        h, w, c = h2, w2, cout
    out = [2 * (dims[i][0] + dims[i][1]) for i in range(1, 5)]
    out.append(2 * dims[5][0] + 4 * h * w)
    return out   # [E2, E3, E4, E5, D1]


def resize_bytes_per_frame(wl):
    """Algorithmic bytes of stage 1: the distinct source rows bilinear touches + the output."""
    rows = set()
    for y in range(wl.proxy_h):
        sy = max(((2 * y + 1) * wl.src_h - wl.proxy_h) / (2 * wl.proxy_h), 0.0)
        y0 = min(int(np.floor(sy)), wl.src_h - 1)
        rows.add(y0)
        rows.add(min(y0 + 1, wl.src_h - 1))
    return len(rows) * wl.src_w * 3 + wl.proxy_h * wl.proxy_w * 3


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, gpu_index: int):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(gpu_index), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "50"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        # nvidia-smi needs a few hundred ms to start sampling: wait for its first line so the
        # samples cover the timed region, and keep only the lines written after this point
        self.skip = 0
        t0 = time.time()
        while self.p is not None and time.time() - t0 < 5.0:
            self.f.flush()
            with open(self.f.name) as fh:
                n = len(fh.read().splitlines())
            if n > 0:
                self.skip = n
                break
            time.sleep(0.02)

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            self.p.wait(5)
        except Exception:
            self.p.kill()
        self.f.flush()
        self.f.seek(0)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        lines = self.f.read().splitlines()
        if len(lines) > self.skip:
            lines = lines[self.skip:]      # samples taken during the timed region
        for line in lines:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                smax.append(float(parts[2]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        os.unlink(self.f.name)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# --------------------------------------------------------------------------- CPU oracle leg
def oracle_frames_per_s(wl, frames_u8: np.ndarray, threshold: float, cores: int, blob=None, sizes=None):
    """Time the oracle (as it stands) on a bounded sample: resize, proxy (quant=bf16),
    threshold, grouping and pack per frame, one frame per task over `cores` threads."""
    import oracle
    from synth import configs, weights
    blob = weights.proxy_weights() if blob is None else blob
    sizes = [tuple(s) for s in (wl.sizes if sizes is None else sizes)]

    def one(i):
        f = frames_u8[i:i + 1]
        img = oracle.resize(f, wl.proxy_h, wl.proxy_w)
        s = oracle.proxy_score(img, wl.n_strided, configs.ENC_WIDTHS, configs.DEC_WIDTH, blob, oracle.QUANT_BF16)
        m = oracle.threshold(s, threshold)
        win, cnt, off, tot = oracle.select_windows(m, wl.cell, wl.src_w, wl.src_h, sizes)
        oracle.pack_windows(f, wl.src_h, wl.src_w, win, sizes)
        return tot

    n = frames_u8.shape[0]
    t0 = time.perf_counter()
    with ThreadPoolExecutor(cores) as ex:
        list(ex.map(one, range(n)))
    dt = time.perf_counter() - t0
    return n / dt, dt


def cpu_baseline_for(wl, thr, n, cores):
    from synth import video
    frames = video.frames(wl, n).numpy()
    fps, dt = oracle_frames_per_s(wl, frames, thr, cores)
    return {"value": fps, "unit": "frames/s", "cores": cores, "kind": "oracle",
            "sample": f"first {n} {wl.name} frames, full path per frame (resize, fp64 proxy quant=bf16, threshold, "
                      f"grouping, pack), one frame per task on {cores} threads, {dt:.1f} s wall"}


def run_reference(args):
    """--impl reference: the CPU oracle is this tier's reference arm."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    from synth import configs, video
    wl = configs.C2
    b = threshold_for(wl.name)
    cores = len(os.sched_getaffinity(0))
    per_step = args.oracle_frames
    frames = video.frames(wl, per_step * (args.steps + args.warmup)).numpy()
    for i in range(args.warmup):
        oracle_frames_per_s(wl, frames[i * per_step:(i + 1) * per_step], b, cores)
    times = []
    for i in range(args.steps):
        s = (args.warmup + i) * per_step
        _, dt = oracle_frames_per_s(wl, frames[s:s + per_step], b, cores)
        times.append(dt)
    ms = 1000.0 * float(np.mean(times))
    value = per_step / (ms / 1000.0)
    sample = f"{per_step} C2 frames per step (of 4500), full path per frame, {cores} threads"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "C2: 960x540 traffic clip, 10 min @30 fps, every 4th frame (4500 frames); "
                                   "oracle sample per step", "frames_per_step": per_step, "proxy": "240x135, S=8",
                       "cell": 32, "W": [list(s) for s in wl.sizes], "threshold_q": 0.7},
            "cpu_baseline": {"value": value, "unit": "frames/s", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# --------------------------------------------------------------------------- GPU measurement helpers
def measure_pipeline(otif, wl, blob, thr, src, steps, warmup, sizes=None, caps=None, batch=None, overlap=2):
    """Whole path (otif_pipeline_run_device) over the device-resident frames `src`: warm-up,
    then `steps` timed passes bracketed by CUDA events on the launching stream; per-stage
    event times, kernel launches and device counters.  overlap = the pipeline's pack_overlap:
    2 = the pack of step s is copied under step s+1's proxy; the last one is flushed INSIDE
    the timed region, so every step's work is timed."""
    import torch
    n = src.shape[0]
    pipe = otif.Pipeline(wl, blob, thr, max_batch=batch or n, sizes=sizes, batch_cap=caps, pack_overlap=overlap)
    stream = torch.cuda.current_stream()
    for _ in range(warmup):
        pipe.run_device(src)
    pipe.flush()
    torch.cuda.synchronize()
    pipe.reset_counters()
    pipe.set_timing(True)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        pipe.run_device(src)
    pipe.flush()
    e1.record(stream)
    torch.cuda.synchronize()
    ms_total = e0.elapsed_time(e1)
    stage_ms, launches = pipe.stage_ms()
    pack_units = pipe.pack_units() if overlap else None   # which layer carried how much of the copy
    ctr = pipe.counters()
    out = {"pipe": pipe, "ms_total": ms_total, "stage_ms": stage_ms, "launches": launches, "ctr": ctr,
           "frames": n * steps, "steps": steps, "overlap": overlap, "resize_fused": pipe.resize_fused(),
           "pack_units": pack_units}
    return out


CONV_STAGES = ["proxy_prep_e1", "conv_e2", "conv_e3", "conv_e4", "conv_e5", "conv_d1_head"]


def rooflines(wl, m, peaks, peak_src, traffic=None, fused_pack=False):
    """Per-kernel rooflines of one measured pipeline: the proxy convolutions (tensor) against
    the measured bf16 burst peak (the timed regions are well under a second, at the
    maximum SM clock) with the sustained peak beside it; resize and pack (HBM) against
    the measured copy bandwidth; the grouping as ns/frame and share of the step."""
    from synth import configs
    sm = m["stage_ms"]
    frames = int(m["ctr"][0].item())
    steps = m["steps"]
    macs, head = conv_macs_per_frame(wl, configs.ENC_WIDTHS, configs.DEC_WIDTH)
    conv_ms = sum(sm[s] for s in CONV_STAGES)
    conv_flops = 2.0 * sum(macs) * frames
    tflops = conv_flops / (conv_ms / 1e3) / 1e12 if conv_ms > 0 else 0.0
    burst = float(peaks.get("bf16_tflops"))
    sustained = float(peaks.get("bf16_tflops_sustained", burst))
    per_layer = {}
    for i, s in enumerate(CONV_STAGES[1:]):
        fl = 2.0 * (macs[i + 1] + (macs[0] if i == 0 else 0)) * frames
        ms = sm[s] + (sm["proxy_prep_e1"] if i == 0 else 0.0)
        name = "conv_e1_e2" if i == 0 else s
        per_layer[name] = {"ms_per_step": ms / steps, "tflops": fl / (ms / 1e3) / 1e12 if ms > 0 else None,
                           "frac_burst": fl / (ms / 1e3) / 1e12 / burst if ms > 0 else None}
        if i == 0 and m.get("resize_fused") and ms > 0:
            # the launch also streams the frames (stage 1 fused in): its own roofline is the
            # larger of the HBM time of those bytes and the tensor time of E1 + E2
            src_b = (resize_bytes_per_frame(wl) - wl.proxy_h * wl.proxy_w * 3) * frames
            t_hbm = src_b / (float(peaks.get("hbm_gbs")) * 1e9) * 1e3
            t_tc = fl / (burst * 1e12) * 1e3
            per_layer[name].update({"reads_frames_bytes_per_step": src_b / steps,
                                    "roofline_ms_per_step": max(t_hbm, t_tc) / steps,
                                    "roofline_bound": "hbm" if t_hbm >= t_tc else "tensor",
                                    "frac_of_roofline": max(t_hbm, t_tc) / ms})
    hbm = float(peaks.get("hbm_gbs"))
    rs_bytes = resize_bytes_per_frame(wl) * frames
    pk_bytes = 2.0 * 3 * int(m["ctr"][14].item())
    pu = m.get("pack_units")
    drain_share = None
    if pu and pu["total"] > 0:
        # fused pack: a layer that also copied detector-batch units has the combined roofline
        # max(tensor time of its FLOPs, HBM time of its activation bytes + the pack bytes it
        # copied); pack bytes per layer from the unit claim counter (average unit size)
        act = conv_act_bytes_per_frame(wl, configs.ENC_WIDTHS, configs.DEC_WIDTH)
        for i, (name, key) in enumerate(zip(["conv_e3", "conv_e4", "conv_e5", "conv_d1_head"],
                                            ["E3", "E4", "E5", "D1"])):
            if pu[key] == 0 or per_layer[name]["ms_per_step"] <= 0:
                continue
            share = pu[key] / pu["total"]
            pb = share * pk_bytes / steps
            ab = act[i + 1] * frames / steps
            fl = 2.0 * macs[i + 2] * frames / steps
            t_tc, t_hbm = fl / (burst * 1e12) * 1e3, (ab + pb) / (hbm * 1e9) * 1e3
            per_layer[name].update({"pack_share": share, "pack_bytes_per_step": pb, "act_bytes_per_step": ab,
                                    "combined_roofline_ms_per_step": max(t_tc, t_hbm),
                                    "combined_bound": "hbm" if t_hbm >= t_tc else "tensor",
                                    "frac_of_combined_roofline": max(t_tc, t_hbm) / per_layer[name]["ms_per_step"]})
        drain_share = pu["drain"] / pu["total"]
    step_sum = sum(sm.values())
    conv = {"bound": "tensor", "achieved": tflops, "peak": burst, "unit": "TFLOP/s", "frac": tflops / burst,
            "frac_vs_sustained": tflops / sustained, "traffic": traffic,
            "peak_source": peak_src + ": bf16 burst (cuBLAS 8192^3 best of 10 at the max SM clock); "
                                      "sustained (4 s loop under the power cap) beside it",
            "algorithmic": f"2 x {sum(macs) / 1e6:.1f} MMAC/frame (E1..D1) x {frames // steps} frames per launch set",
            "layers": per_layer, "ms_per_step": conv_ms / steps, "share_of_step": conv_ms / step_sum}
    if drain_share is not None:
        conv["pack_units_left_to_drain"] = drain_share
    out = {"conv": conv}
    for k, byts in (("resize", rs_bytes), ("pack", pk_bytes)):
        ms = sm[k]
        if k == "resize" and m.get("resize_fused"):
            # stage 1 runs inside the E1+E2 kernel (its converter warps read the frames; the
            # proxy image is never written): the source-row bytes against that kernel's time
            src_b = byts - wl.proxy_h * wl.proxy_w * 3 * frames
            e12_ms = sm["proxy_prep_e1"] + sm["conv_e2"]
            gbs = src_b / (e12_ms / 1e3) / 1e9 if e12_ms > 0 else None
            out[k] = {"bound": "hbm", "fused_into": "conv_e1_e2 (e12s_umma_kernel: converter warps read the frames)",
                      "bytes_per_step": src_b / steps, "e1_e2_ms_per_step": e12_ms / steps,
                      "achieved_in_e1_e2": gbs, "peak": hbm, "unit": "GB/s", "frac": gbs / hbm if gbs else None}
            continue
        if k == "pack" and fused_pack:
            # the copy runs inside the E5 / D1 kernels of the next step; "pack" holds only the
            # slot kernel and the drain of what the fused warps left
            out[k] = {"bound": "hbm", "fused_into": "conv_e5, conv_d1_head (next step)", "bytes_per_step": byts / steps,
                      "slot_and_drain_ms_per_step": ms / steps,
                      "hbm_frac_of_step": byts / steps / (float(m["ms_total"]) / steps / 1e3) / 1e9 / hbm}
            continue
        gbs = byts / (ms / 1e3) / 1e9 if ms > 0 else None
        out[k] = {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s", "frac": gbs / hbm if gbs else None,
                  "frac_spec_8tbs": gbs / 8000.0 if gbs else None, "bytes_per_step": byts / steps,
                  "ms_per_step": ms / steps}
    out["select"] = {"ms_per_step": sm["select"] / steps, "ns_per_frame": sm["select"] * 1e6 / max(frames, 1),
                     "share_of_step": sm["select"] / step_sum if step_sum else None}
    return out


def window_stats(m, wl, sizes):
    c = m["ctr"].cpu().tolist()
    frames = c[0]
    full_idx = [i for i, s in enumerate(sizes) if (int(s[0]), int(s[1])) == (wl.src_w, wl.src_h)]
    full = sum(c[5 + i] for i in full_idx)
    return {"windows_per_frame": c[2] / max(frames, 1), "fallback_share": full / max(frames, 1),
            "window_area_fraction": c[3] / max(frames * wl.src_w * wl.src_h, 1),
            "per_size": c[5:5 + len(sizes)], "dropped_windows": c[13], "positive_cell_fraction":
            c[1] / max(frames * (-(-wl.src_h // wl.cell)) * (-(-wl.src_w // wl.cell)), 1)}


def caps_for(wl, sizes, n, per_frame=8):
    """Detector batch capacities: one full-frame slot per frame; per_frame slots of each
    smaller size (bounded by how many such windows fit in a frame)."""
    out = []
    for s in sizes:
        if (int(s[0]), int(s[1])) == (wl.src_w, wl.src_h):
            out.append(n)
        else:
            fit = max(1, (wl.src_w // int(s[0])) * (wl.src_h // int(s[1])))
            out.append(n * min(per_frame, fit))
    return out


def choose_wstar(otif_tuning, wl, clip, start, n, k, dev):
    """NEXT-1 on the GPU: W* from the perfect-proxy masks of frames
    [start, start + n) of `clip` (the same camera, earlier/later than the measured frames)."""
    import torch
    from synth import video
    sc = video.make_scene(wl, clip=clip)
    masks = torch.from_numpy(np.stack([video.gt_mask(sc.gt_boxes(t), wl.src_w, wl.src_h, wl.cell)
                                       for t in range(start, start + n)])).to(dev)
    cands = otif_tuning.candidate_sizes(wl.src_w, wl.src_h, wl.cell)
    chosen, sums, idx = otif_tuning.choose_window_sizes(masks, wl.src_w, wl.src_h, wl.cell, cands, k=k)
    return [tuple(int(v) for v in c[:2]) for c in chosen], sums


def windowing_scenario(otif, otif_tuning, wl, src, rank, dev, peaks, peak_src, args):
    """The path with the windowing active: the proxy trained by NEXT-3 and the
    window set W* chosen by NEXT-1, both from frames [n, n + 1024) of the
    same camera (the training split, later in time than the measured frames [0, n)),
    through the whole pipeline; and stages 3–5 on the perfect proxy."""
    import torch
    from scripts import train_proxy
    from synth import video
    n = src.shape[0]
    t0 = time.time()
    tw, tinfo = train_proxy.train_weights(wl, steps=args.train_steps, batch=32, clip=rank, start=n)
    wstar = {k: choose_wstar(otif_tuning, wl, rank, n, 600, k, dev) for k in (3, 5)}
    out = {"what": f"{wl.name}: {n} frames of one camera through the whole path with the trained proxy (B = 0.5) "
                   f"and W*; training and W* from frames [{n}, {n + 1024}) of the same camera",
           "objects_mean": wl.objects,
           "train": {k: tinfo[k] for k in ("steps", "batch", "ms_per_step", "loss", "train_frames")},
           "prep_s": None}
    for k, (W, sums) in wstar.items():
        out[f"W*_k{k}"] = [list(x) for x in W]
    out["prep_s"] = time.time() - t0
    for k, (W, _) in wstar.items():
        caps = caps_for(wl, W, n)
        mw = measure_pipeline(otif, wl, tw, 0.5, src, args.steps, args.warmup, sizes=W, caps=caps,
                              overlap=args.pack_overlap)
        out[f"trained_k{k}"] = {"frames_per_s": mw["frames"] / (mw["ms_total"] / 1e3),
                                "ms_per_step": mw["ms_total"] / args.steps, "windows": window_stats(mw, wl, W),
                                "roofline": rooflines(wl, mw, peaks, peak_src, fused_pack=args.pack_overlap > 0),
                                "batch_cap": caps}
        mw["pipe"].close()
        torch.cuda.empty_cache()
    # perfect proxy: stages 3-5 on the ground-truth cell masks of the measured frames
    sc = video.make_scene(wl, clip=rank)
    masks = torch.from_numpy(np.stack([video.gt_mask(sc.gt_boxes(t), wl.src_w, wl.src_h, wl.cell)
                                       for t in range(n)])).to(dev)
    pp = {}
    for tag, W in [("default_W", list(wl.sizes))] + [(f"W*_k{k}", W) for k, (W, _) in wstar.items()]:
        caps = caps_for(wl, W, n)
        r = otif.otif_select_windows(None, masks, 0.0, wl.src_w, wl.src_h, wl.cell, W)
        otif.otif_pack_windows(src, wl.src_h, wl.src_w, r["windows"], r["total"], W, caps)
        torch.cuda.synchronize()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        sel_ms = pk_ms = 0.0
        for _ in range(args.steps):
            ev[0].record()
            r = otif.otif_select_windows(None, masks, 0.0, wl.src_w, wl.src_h, wl.cell, W)
            ev[1].record()
            bt, slot, scount = otif.otif_pack_windows(src, wl.src_h, wl.src_w, r["windows"], r["total"], W, caps)
            ev[2].record()
            torch.cuda.synchronize()
            sel_ms += ev[0].elapsed_time(ev[1])
            pk_ms += ev[1].elapsed_time(ev[2])
            del bt
        tot = int(r["total"].item())
        wins = r["windows"][:tot].cpu().numpy()
        px = int((wins[:, 3].astype(np.int64) * wins[:, 4]).sum()) if tot else 0
        full = int(((wins[:, 3] == wl.src_w) & (wins[:, 4] == wl.src_h)).sum()) if tot else 0
        sc_np = scount.cpu().numpy()
        e = {"W": [list(x) for x in W], "windows_per_frame": tot / n, "fallback_share": full / n,
             "window_area_fraction": px / (n * wl.src_w * wl.src_h), "per_size": sc_np.tolist(),
             "dropped_windows": int(np.maximum(sc_np - np.array(caps), 0).sum()),
             "select_ns_per_frame": sel_ms / args.steps * 1e6 / n,
             "select_ms_per_step": sel_ms / args.steps, "pack_ms_per_step": pk_ms / args.steps,
             "pack_gbs": 2 * 3 * px / (pk_ms / args.steps / 1e3) / 1e9 if pk_ms > 0 else None,
             "est_sum": int(r["est_sum"].item())}
        e["pack_hbm_frac"] = e["pack_gbs"] / float(peaks["hbm_gbs"]) if e["pack_gbs"] else None
        pp[tag] = e
    out["perfect_proxy"] = pp
    return out


# --------------------------------------------------------------------------- GPU leg
def run_otif(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    nccl = None
    if world > 1:
        # communicator init lines (rank count per communicator) go to stderr, not the JSON stdout
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        nccl = {"backend": dist.get_backend(), "comm_nranks": dist.get_world_size(),
                "nccl_version": ".".join(str(v) for v in torch.cuda.nccl.version())}
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)

    import paper_conf_sigmod_bastanim22_b200 as otif
    from paper_conf_sigmod_bastanim22_b200 import dist as odist
    from paper_conf_sigmod_bastanim22_b200 import tuning as otif_tuning
    from synth import configs, video, weights

    wl = configs.C2
    n = wl.n_frames
    blob = weights.proxy_weights()
    b = threshold_for(wl.name)
    peaks, peak_src = load_peaks()
    cores = len(os.sched_getaffinity(0))
    extras = (world == 1 or rank == 0) and not args.headline_only

    # this rank's shard: its own 4500-frame clip (weak scaling; clip seeds by rank)
    src = torch.empty((n, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device=dev)
    video.make_scene(wl, clip=rank).render(range(n), out=src)
    torch.cuda.synchronize()

    # ---- headline: C2, random-init proxy (north_star), one device batch of 4500 frames
    sampler = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    m = measure_pipeline(otif, wl, blob, b, src, args.steps, args.warmup, batch=args.batch or None,
                         overlap=args.pack_overlap)
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    ms_max = odist.max_over_ranks(m["ms_total"], dev)
    gathered = odist.gather_counters(m["ctr"])
    frames_total = int(gathered[:, 0].sum().item())
    value = frames_total / (ms_max / 1000.0)
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(prof):
        try:
            traffic = json.load(open(prof)).get("conv_dram_bytes_per_batch")
        except Exception:
            traffic = None
    rl = rooflines(wl, m, peaks, peak_src, traffic, fused_pack=args.pack_overlap > 0)
    launches = m["launches"]
    m["pipe"].close()
    # the same pipeline with the serial stage-5 schedule (pack_overlap 0, 10 steps): every
    # kernel alone on the GPU, so resize / pack / conv rooflines without the fused copy
    serial = None
    if extras and args.pack_overlap > 0:
        ms_ = measure_pipeline(otif, wl, blob, b, src, 10, args.warmup, batch=args.batch or None, overlap=0)
        rs_ = rooflines(wl, ms_, peaks, peak_src, traffic)
        serial = {"frames_per_s": ms_["frames"] / (ms_["ms_total"] / 1e3), "ms_per_step": ms_["ms_total"] / 10,
                  "rooflines": rs_, "note": "pack_overlap 0: stage 5 as its own kernel after the selection"}
        ms_["pipe"].close()

    objs = {}
    # ---- the other BASELINE configs, each with its own rooflines and oracle sample
    if extras and not args.no_configs:
        cfg = {}
        for cw, nfr in ((configs.C1, None), (configs.C3, None), (configs.C4_SWEEP[1], None), (configs.C4_SWEEP[3], None)):
            nn = nfr or cw.n_frames
            s2 = torch.empty((nn, cw.src_h, cw.src_w, 3), dtype=torch.uint8, device=dev)
            video.make_scene(cw).render(range(nn), out=s2)
            thr = threshold_for(cw.name)
            steps_c = max(args.steps, int(np.ceil(2000.0 / nn)) if nn < 1000 else args.steps)
            mc = measure_pipeline(otif, cw, blob, thr, s2, steps_c, args.warmup, overlap=args.pack_overlap)
            r = rooflines(cw, mc, peaks, peak_src, fused_pack=args.pack_overlap > 0)
            cfg[cw.name] = {"workload": f"{cw.src_w}x{cw.src_h} {cw.scene}, {nn} frames, proxy {cw.proxy_w}x{cw.proxy_h} "
                                        f"(S={cw.stride}), {cw.cell}-px cells, W={[list(x) for x in cw.sizes]}",
                            "frames_per_s": mc["frames"] / (mc["ms_total"] / 1e3),
                            "ms_per_step": mc["ms_total"] / steps_c, "steps": steps_c, "threshold_q": 0.7,
                            "roofline": r, "windows": window_stats(mc, cw, cw.sizes), "gpu_launches": mc["launches"],
                            "cpu_baseline": None if args.no_cpu_baseline else
                            cpu_baseline_for(cw, thr, min(args.oracle_frames, nn), cores)}
            mc["pipe"].close()
            del s2
            torch.cuda.empty_cache()
        objs["configs"] = cfg

    # ---- windowing active: the NEXT-3-trained proxy and the perfect proxy under W*, at the
    # headline density (C2) and off-peak (C2s, same camera, ~4 vehicles)
    if extras and not args.no_windowing:
        wa = {}
        for ww in (configs.C2, configs.C2S):
            if ww.name == wl.name:
                s_w = src
            else:
                s_w = torch.empty((n, ww.src_h, ww.src_w, 3), dtype=torch.uint8, device=dev)
                video.make_scene(ww, clip=rank).render(range(n), out=s_w)
            wa[ww.name] = windowing_scenario(otif, otif_tuning, ww, s_w, rank, dev, peaks, peak_src, args)
            del s_w
            torch.cuda.empty_cache()
        objs["windowing_active"] = wa

    # ---- C5: the 8-hour corpus (480 one-minute clips x 450 frames), contiguous
    # clip ranges per rank, per-clip device counters and hashes, strong scaling
    if not args.no_c5:
        objs["c5"] = run_c5(otif, odist, configs, video, blob, b, dev, world, rank, args)

    # ---- NEXT-4: track index over S* + refinement of gap-16 query tracks (C6)
    if extras and not args.no_next4:
        from scripts import tracks_bench
        objs["track_refinement"] = tracks_bench.run(tracks_bench.tracks.C6, reps=5)

    # ---- NEXT-3: proxy training steps (fp32 forward + backward + Adam)
    if extras and not args.no_next3:
        from paper_conf_sigmod_bastanim22_b200 import train as otif_train
        sc = video.make_scene(wl, clip=rank)
        tsel = [t for t in range(0, n, max(n // 64, 1)) if sc.gt_boxes(t)][:32]
        bx = np.array([(i, *bb) for i, t in enumerate(tsel) for bb in sc.gt_boxes(t) if bb[0] < bb[2] and bb[1] < bb[3]],
                      np.int32).reshape(-1, 5)
        gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
        lab = otif_train.otif_cell_labels(torch.from_numpy(bx).to(dev), len(tsel), (gh, gw), wl.src_w, wl.src_h,
                                          wl.cell)
        timg = otif.otif_resize(src[torch.tensor(tsel, device=dev)], wl.proxy_h, wl.proxy_w)
        tr = otif_train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights(), max_batch=len(tsel))
        l0 = float(tr.step(timg, lab, 1e-3).item())
        torch.cuda.synchronize()
        t0e, t1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0e.record()
        for _ in range(args.steps):
            lt = tr.step(timg, lab, 1e-3)
        t1e.record()
        torch.cuda.synchronize()
        tms = t0e.elapsed_time(t1e) / args.steps
        macs, head = conv_macs_per_frame(wl, configs.ENC_WIDTHS, configs.DEC_WIDTH)
        train_flop = 3 * 2 * (sum(macs) + head) * len(tsel)      # forward + dgrad + wgrad
        nx3 = {"what": "fp32 training step (forward, BCE head, dgrad, wgrad, Adam); convolution GEMMs on tcgen05 "
                       "(3xTF32, fp32-accurate)", "batch": len(tsel), "ms_per_step": tms,
               "train_frames_per_s": len(tsel) / (tms / 1e3), "tflops": train_flop / (tms / 1e3) / 1e12,
               "loss_first": l0, "loss_last": float(lt.item())}
        # tf32 peak = measured bf16 burst x the guide's nominal tf32/bf16 ratio (1.1 / 2.25);
        # 3xTF32 issues 3 MMAs per useful product
        tf32_peak = float(peaks.get("bf16_tflops")) * 1.1 / 2.25
        nx3["roofline"] = {"bound": "tensor", "unit": "TFLOP/s", "achieved": nx3["tflops"], "peak": tf32_peak / 3.0,
                           "frac": nx3["tflops"] / (tf32_peak / 3.0),
                           "peak_source": "measured bf16 burst x 1.1/2.25 (tf32), / 3 (3xTF32 useful rate); "
                                          "the step is bound by the implicit-GEMM gathers, not the MMAs"}
        objs["proxy_training"] = nx3
        del tr, timg, lab

    # ---- end to end through the C ABI with HOST frames: pinned H2D + D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        e2e_frames = n
        try:
            host = torch.empty(src.shape, dtype=torch.uint8, pin_memory=True)
        except RuntimeError:
            # the host cannot pin 7 GB per rank (8 ranks on one node): first 1024 frames
            e2e_frames = min(n, 1024)
            host = torch.empty((e2e_frames,) + tuple(src.shape[1:]), dtype=torch.uint8, pin_memory=True)
        host.copy_(src[:e2e_frames])
        del src
        torch.cuda.empty_cache()
        pipe = otif.Pipeline(wl, blob, b, max_batch=args.host_batch)
        pipe.run_host(host)  # warm-up (allocates the output arrays)
        times, last = [], None
        for _ in range(args.e2e_steps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            last = pipe.run_host(host)
            times.append(time.perf_counter() - t0)
        win_, counts, sc_, tot = last
        tmax = odist.max_over_ranks(max(times), dev)
        e2e = {"value": world * e2e_frames / tmax, "unit": "frames/s",
               "h2d_bytes_per_step": int(host.numel()),
               "d2h_bytes_per_step": int(4 + 4 * e2e_frames + 24 * tot + 8 * 15),
               "frames_per_step_per_gpu": e2e_frames,
               "api": "otif_pipeline_run_host (C ABI), pinned host frames, 2 streams (PCIe-bound)"}
        pipe.close()

    cpu_baseline = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu_baseline = cpu_baseline_for(wl, b, args.oracle_frames, cores)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {"workload": "C2: 960x540 traffic-camera clip, 10 min @30 fps sampled every 4th frame "
                                   "(4500 frames per GPU), proxy at 1/4 res (240x135), 32x32-px cells (17x30 grid)",
                       "frames_per_step_per_gpu": n, "batch": args.batch or n, "W": [list(s) for s in wl.sizes],
                       "threshold": b, "threshold_q": 0.7, "proxy": "E1-E5 (32,64,128,256,256) + D1 128 + D2 1, "
                       "random init PCG64(20220612)", "l2": "inputs (7.0 GB/GPU) exceed the 126 MB L2; no flush",
                       "parallelism": f"dp{world} (clip-sharded)"},
            "roofline": dict(rl["conv"], kernel=("proxy convs on tcgen05: e12s_umma_kernel (resize + E1 fused into "
                                                 "E2: reads the u8 frames) + conv_umma_kernel (E3..E5, D1+D2 head)"
                                                 if m.get("resize_fused") else
                                                 "proxy convs on tcgen05: e12_umma_kernel (E1 fused into E2) + "
                                                 "conv_umma_kernel (E3..E5, D1+D2 head)"),
                             per_launch="5 launches per batch of 4500 frames; achieved = algorithmic FLOPs of "
                                        "E1..D1 / CUDA-event time of those launches on the pipeline stream",
                             fused_work=("; ".join(x for x in (
                                 ("the E5 and D1 launches also copy the previous step's detector batches "
                                  f"({rl['pack']['bytes_per_step'] / 1e9:.1f} GB per step through HBM; pack_overlap 2)"
                                  if args.pack_overlap > 0 else None),
                                 (f"the E1+E2 launch also reads the frames ({rl['resize']['bytes_per_step'] / 1e9:.1f} GB "
                                  "per step: stage 1 fused in)" if m.get("resize_fused") else None)) if x)
                                 + ", which the tensor FLOP count does not credit") if (args.pack_overlap > 0 or
                                                                                      m.get("resize_fused")) else None,
                             frac_serial_schedule=(serial["rooflines"]["conv"]["frac"] if serial else None)),
            "stages": {k: v for k, v in rl.items() if k != "conv"},
            "serial_schedule": serial,
            **objs,
            "cpu_baseline": cpu_baseline,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clocks,
            "nccl": nccl,
            "counters": odist.combine(gathered),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_c5(otif, odist, configs, video, blob, b, dev, world, rank, args):
    """C5: 480 clips x 450 frames (216,000 frames, 336 GB of u8: larger than HBM), every rank
    renders the same 8-clip pool and clip k reads pool slot k mod 8; rank r
    takes clips shard_clips(480, G, r).  One pipeline call per clip (frame_base = the
    clip's global first frame, so window hashes are keyed by the global frame); its
    device counters are snapshotted per clip and reset.  Time = max over ranks."""
    import torch
    import torch.distributed as dist
    wl = configs.C5
    fpc = configs.C5_FRAMES_PER_CLIP
    n_clips = configs.C5_CLIPS if args.c5_clips <= 0 else args.c5_clips
    pool = torch.empty((configs.C5_POOL_CLIPS * fpc, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device=dev)
    for j in range(configs.C5_POOL_CLIPS):
        video.make_scene(wl, clip=j).render(range(fpc), out=pool[j * fpc:(j + 1) * fpc])
    pool_n = configs.C5_POOL_CLIPS
    pipe = otif.Pipeline(wl, blob, b, max_batch=pool_n * fpc, pack_overlap=args.pack_overlap)
    clips = odist.shard_clips(n_clips, world, rank)

    def run_group(r):
        # clips r (consecutive, pool-contiguous) in ONE pipeline call: frames of pool slots
        # [r.start mod pool, ...) with the global frame base of clip r.start
        j = r.start % pool_n
        pipe.run_device(pool[j * fpc:(j + len(r)) * fpc], frame_base=r.start * fpc)
        tot = pipe.counters()
        pipe.reset_counters()
        fh, fc = pipe.frame_results(len(r) * fpc)
        rows = torch.zeros((len(r), tot.numel()), dtype=torch.int64, device=tot.device)
        rows[0] = tot
        rows[:, 0] = fpc
        rows[:, 2] = fc.view(len(r), fpc).sum(1)
        rows[:, 4] = fh.view(len(r), fpc).sum(1)      # wrapping int64 sum = the clip's hash
        return rows

    def run_clip(k):
        return run_group(range(k, k + 1))

    for k in list(clips)[:2]:     # warm-up
        run_clip(k)
    pipe.flush()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    times, per_clip = [], None
    for _ in range(args.c5_passes):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        per_clip = odist.run_corpus_grouped(clips, pool_n, run_group)
        pipe.flush()              # the last call's pack (pack_overlap 2) inside the timed pass
        e1.record()
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    if world > 1:
        dist.barrier()
    ms = odist.max_over_ranks(float(np.mean(times)), dev)
    allc = odist.gather_clip_counters(per_clip.to(dev), n_clips, per_clip.shape[1])
    digest = odist.corpus_digest(allc)
    pipe.close()
    del pool
    torch.cuda.empty_cache()
    return {"what": f"{n_clips} one-minute 960x540 clips x {fpc} sampled frames (P:L99, P:L244), 8-clip pool, "
                    f"contiguous clip ranges per rank; one pipeline call per pool-contiguous run of up to "
                    f"{pool_n} clips (pack of call c under call c+1's proxy, pack_overlap {args.pack_overlap}); "
                    f"per-clip hashes from the per-frame hash terms",
            "frames_per_s": n_clips * fpc / (ms / 1e3), "ms_per_pass": ms, "passes": args.c5_passes,
            "scaling": "strong (fixed corpus)", "clips_per_rank": len(clips), "corpus": digest}


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["otif", "reference"], default="otif")
    ap.add_argument("--batch", type=int, default=0, help="device batch (0 = whole clip)")
    ap.add_argument("--pack-overlap", type=int, default=2, choices=[0, 1, 2],
                    help="pipeline pack_overlap (0 = serial pack; 2 = pack of step s under step s+1's proxy)")
    ap.add_argument("--host-batch", type=int, default=512, help="device batch of the host (e2e) path")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--oracle-frames", type=int, default=64)
    ap.add_argument("--train-steps", type=int, default=400)
    ap.add_argument("--c5-clips", type=int, default=0, help="C5 clips (0 = the full 480)")
    ap.add_argument("--c5-passes", type=int, default=2)
    ap.add_argument("--headline-only", action="store_true", help="only the C2 headline (+ e2e / cpu baseline)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the C1 / C3 / C4b / C4d objects")
    ap.add_argument("--no-windowing", action="store_true", help="skip the trained-proxy / perfect-proxy objects")
    ap.add_argument("--no-c5", action="store_true", help="skip the C5 corpus object")
    ap.add_argument("--no-next4", action="store_true", help="skip the NEXT-4 track-refinement line")
    ap.add_argument("--no-next3", action="store_true", help="skip the NEXT-3 proxy-training line")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: re-launch under torchrun on this node (NCCL over NVLink)
        env = dict(os.environ)
        env.setdefault("NCCL_DEBUG", "INFO")
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        env.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd, env=env)
    if args.impl == "reference":
        return run_reference(args)
    return run_otif(args)


if __name__ == "__main__":
    sys.exit(main())
