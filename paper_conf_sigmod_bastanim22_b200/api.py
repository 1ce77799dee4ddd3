"""Python binding with the ABI's names.  PyTorch supplies device memory and the
current CUDA stream; all compute happens in libotif.so (no CPU path)."""
from __future__ import annotations

import ctypes
from typing import Sequence

import numpy as np
import torch

from . import _lib
from ._lib import GridDesc, PipelineDesc, ProxyDesc, WSize, check, lib

WINDOW_FIELDS = ("frame", "x", "y", "w", "h", "size_idx")


def _ptr(t: torch.Tensor | None) -> ctypes.c_void_p:
    if t is None:
        return ctypes.c_void_p(0)
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream=None) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _require_cuda(*ts):
    for t in ts:
        if t is not None:
            if not t.is_cuda:
                raise ValueError("libotif operates on CUDA tensors (there is no CPU path)")
            if not t.is_contiguous():
                raise ValueError("tensors must be contiguous")


def wsizes(sizes: Sequence[tuple]) -> ctypes.Array:
    """[(w, h)] or [(w, h, cost)]; default cost w*h (reading R8)."""
    arr = (WSize * len(sizes))()
    for i, s in enumerate(sizes):
        arr[i].w, arr[i].h = int(s[0]), int(s[1])
        arr[i].cost = int(s[2]) if len(s) > 2 else int(s[0]) * int(s[1])
    return arr


def version() -> str:
    return lib().otif_version().decode()


# ---------------------------------------------------------------- stage 1
def otif_resize(src: torch.Tensor, dst_h: int, dst_w: int, out: torch.Tensor | None = None,
                stream=None) -> torch.Tensor:
    _require_cuda(src)
    n, sh, sw, c = src.shape
    assert src.dtype == torch.uint8 and c == 3
    if out is None:
        out = torch.empty((n, dst_h, dst_w, 3), dtype=torch.uint8, device=src.device)
    _require_cuda(out)
    check(lib().otif_resize(_ptr(src), n, sh, sw, _ptr(out), dst_h, dst_w, _stream(stream)), "otif_resize")
    return out


# ---------------------------------------------------------------- stage 2
class Proxy:
    """otif_proxy_create / _score / _destroy (P:L135 proxy CNN)."""

    def __init__(self, in_h: int, in_w: int, n_strided: int, weights: np.ndarray,
                 enc: Sequence[int] = (32, 64, 128, 256, 256), dec: int = 128):
        d = ProxyDesc()
        d.in_h, d.in_w, d.n_strided = in_h, in_w, n_strided
        for i, e in enumerate(enc):
            d.enc[i] = int(e)
        d.dec = int(dec)
        w = np.ascontiguousarray(weights, np.float32)
        self._w = w
        h = ctypes.c_void_p()
        check(lib().otif_proxy_create(ctypes.byref(d), ctypes.c_void_p(w.ctypes.data), w.size, ctypes.byref(h)),
              "otif_proxy_create")
        self.handle = h
        self.in_h, self.in_w = in_h, in_w
        gh, gw = ctypes.c_int32(), ctypes.c_int32()
        check(lib().otif_proxy_grid(h, ctypes.byref(gh), ctypes.byref(gw)), "otif_proxy_grid")
        self.grid = (gh.value, gw.value)
        self._ws = None

    def workspace_bytes(self, n: int) -> int:
        return int(lib().otif_proxy_workspace_bytes(self.handle, n))

    def workspace(self, n: int, device=None) -> torch.Tensor:
        need = self.workspace_bytes(n)
        if self._ws is None or self._ws.numel() < need:
            # zero-filled once; the library keeps the pad positions zero afterwards
            self._ws = torch.zeros(need + 256, dtype=torch.uint8, device=device or "cuda")
        return self._ws

    def score(self, img: torch.Tensor, out: torch.Tensor | None = None, workspace: torch.Tensor | None = None,
              stream=None) -> torch.Tensor:
        _require_cuda(img)
        n, h, w, c = img.shape
        assert (h, w, c) == (self.in_h, self.in_w, 3) and img.dtype == torch.uint8
        if out is None:
            out = torch.empty((n,) + self.grid, dtype=torch.float32, device=img.device)
        ws = workspace if workspace is not None else self.workspace(n, img.device)
        base = ws.data_ptr()
        aligned = (base + 255) & ~255
        avail = ws.numel() - (aligned - base)
        check(lib().otif_proxy_score(self.handle, _ptr(img), n, _ptr(out), ctypes.c_void_p(aligned), avail,
                                     _stream(stream)), "otif_proxy_score")
        return out

    def close(self):
        if getattr(self, "handle", None):
            lib().otif_proxy_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---------------------------------------------------------------- stages 3 + 4
def otif_select_windows(scores: torch.Tensor | None, mask_in: torch.Tensor | None, threshold: float,
                        frame_w: int, frame_h: int, cell: int, sizes, connectivity: int = 4,
                        capacity: int | None = None, want_mask: bool = False, stream=None):
    """-> dict(windows int32[capacity, 6], counts int32[n], offsets int32[n], total int32[1], mask u8|None,
    est_sum int64[1] = Σ_t est(R_t) (computed by the grouping kernel))."""
    t = scores if scores is not None else mask_in
    _require_cuda(t)
    n, gh, gw = t.shape
    dev = t.device
    if capacity is None:
        capacity = max(n * ((gh * gw + 1) // 2), 1)
    windows = torch.empty((max(capacity, 1), 6), dtype=torch.int32, device=dev)
    counts = torch.empty(n, dtype=torch.int32, device=dev)
    offsets = torch.empty(n, dtype=torch.int32, device=dev)
    total = torch.zeros(1, dtype=torch.int32, device=dev)
    mask = torch.empty((n, gh, gw), dtype=torch.uint8, device=dev) if want_mask else None
    est_sum = torch.zeros(1, dtype=torch.int64, device=dev)
    ws_bytes = int(lib().otif_select_workspace_bytes(n, gh, gw))
    ws = torch.empty(max(ws_bytes, 256) + 256, dtype=torch.uint8, device=dev)
    g = GridDesc(frame_w, frame_h, cell, connectivity)
    ws_sizes = wsizes(sizes)
    check(lib().otif_select_windows(_ptr(scores), _ptr(mask_in), ctypes.c_float(threshold), n, gh, gw,
                                    ctypes.byref(g), ws_sizes, len(sizes), _ptr(mask), _ptr(windows), capacity,
                                    _ptr(counts), _ptr(offsets), _ptr(total), _ptr(ws), ws.numel(),
                                    _stream(stream), _ptr(est_sum)), "otif_select_windows")
    return dict(windows=windows, counts=counts, offsets=offsets, total=total, mask=mask, est_sum=est_sum)


# ---------------------------------------------------------------- stage 5
def otif_pack_windows(src: torch.Tensor, det_h: int, det_w: int, windows: torch.Tensor, total: torch.Tensor,
                      sizes, batch_cap: Sequence[int], stream=None):
    """-> (batches list[u8 [cap_s, h_s, w_s, 3]], slot int32[capacity], size_count int32[k])."""
    _require_cuda(src, windows, total)
    n, sh, sw, _ = src.shape
    k = len(sizes)
    dev = src.device
    capacity = windows.shape[0]
    batches = [torch.empty((max(int(batch_cap[s]), 0), int(sizes[s][1]), int(sizes[s][0]), 3), dtype=torch.uint8,
                           device=dev) for s in range(k)]
    ptrs = (ctypes.c_void_p * k)(*[b.data_ptr() if b.numel() else 0 for b in batches])
    caps = (ctypes.c_int32 * k)(*[int(c) for c in batch_cap])
    slot = torch.empty(max(capacity, 1), dtype=torch.int32, device=dev)
    size_count = torch.empty(k, dtype=torch.int32, device=dev)
    check(lib().otif_pack_windows(_ptr(src), n, sh, sw, det_h, det_w, _ptr(windows), _ptr(total), capacity,
                                  wsizes(sizes), k, ptrs, caps, _ptr(slot), _ptr(size_count), _stream(stream)),
          "otif_pack_windows")
    return batches, slot, size_count


# ---------------------------------------------------------------- end to end
class Pipeline:
    """otif_pipeline_*: the whole path with host or device frames (native C++ runtime)."""

    def __init__(self, workload, weights: np.ndarray, threshold: float, max_batch: int = 256,
                 batch_cap: Sequence[int] | None = None, connectivity: int = 4,
                 enc=(32, 64, 128, 256, 256), dec=128, proxy_batch: int = 0, sizes=None, pack_overlap: int = 0):
        """sizes: W as [(w, h)] or [(w, h, cost)] (default: the workload's own W).
        pack_overlap: 0 / 1 / 2 (otif.h: pack of batch b copied under batch b+1's proxy)."""
        d = PipelineDesc()
        d.proxy_batch = int(proxy_batch)
        d.pack_overlap = int(pack_overlap)
        sizes = list(workload.sizes) if sizes is None else list(sizes)
        d.proxy.in_h, d.proxy.in_w, d.proxy.n_strided = workload.proxy_h, workload.proxy_w, workload.n_strided
        for i, e in enumerate(enc):
            d.proxy.enc[i] = int(e)
        d.proxy.dec = int(dec)
        d.src_h, d.src_w = workload.src_h, workload.src_w
        d.det_h, d.det_w = workload.src_h, workload.src_w
        d.grid = GridDesc(workload.src_w, workload.src_h, workload.cell, connectivity)
        d.threshold = float(threshold)
        d.k = len(sizes)
        for i, s in enumerate(sizes):
            d.sizes[i].w, d.sizes[i].h = int(s[0]), int(s[1])
            d.sizes[i].cost = int(s[2]) if len(s) > 2 else int(s[0]) * int(s[1])
        d.max_batch = int(max_batch)
        if batch_cap is None:
            # a full-frame window is the only window of its frame; smaller sizes get headroom
            caps = [max_batch if (int(w[0]), int(w[1])) == (workload.src_w, workload.src_h) else max_batch * 4
                    for w in sizes]
        else:
            caps = batch_cap
        for i in range(d.k):
            d.batch_cap[i] = int(caps[i])
        self.k = d.k
        self.sizes = sizes
        self.grid = (-(-workload.src_h // workload.cell), -(-workload.src_w // workload.cell))
        self.batch_cap = [int(c) for c in caps]
        self.desc = d
        w = np.ascontiguousarray(weights, np.float32)
        self._w = w
        h = ctypes.c_void_p()
        check(lib().otif_pipeline_create(ctypes.byref(d), ctypes.c_void_p(w.ctypes.data), w.size, ctypes.byref(h)),
              "otif_pipeline_create")
        self.handle = h

    def run_host(self, frames: torch.Tensor, cap_windows: int | None = None):
        """frames: host uint8 [n, H, W, 3] (pinned for overlap).  -> (windows np[total,6], counts np[n], size_count)."""
        assert not frames.is_cuda and frames.is_contiguous()
        n = frames.shape[0]
        gh = -(-self.desc.grid.frame_h // self.desc.grid.cell)
        gw = -(-self.desc.grid.frame_w // self.desc.grid.cell)
        cap = cap_windows if cap_windows is not None else n * ((gh * gw + 1) // 2)
        win = np.zeros((max(cap, 1), 6), np.int32)
        counts = np.zeros(n, np.int32)
        total = np.zeros(1, np.int32)
        sc = np.zeros(self.k, np.int32)
        check(lib().otif_pipeline_run_host(self.handle, ctypes.c_void_p(frames.data_ptr()), n,
                                           ctypes.c_void_p(win.ctypes.data), cap, ctypes.c_void_p(counts.ctypes.data),
                                           ctypes.c_void_p(total.ctypes.data), ctypes.c_void_p(sc.ctypes.data)),
              "otif_pipeline_run_host")
        t = int(total[0])
        return win[:min(t, cap)], counts, sc, t

    def run_device(self, frames: torch.Tensor, frame_base: int = 0, stream=None):
        """frames: device u8 [n, H, W, 3]; frame_base = global index of frames[0] (window hash key)."""
        _require_cuda(frames)
        check(lib().otif_pipeline_run_device(self.handle, _ptr(frames), frames.shape[0], int(frame_base),
                                             _stream(stream)), "otif_pipeline_run_device")

    def resize_fused(self) -> bool:
        """True if the last device batch's proxy read the frames itself (no stage-1 launch)."""
        return bool(lib().otif_pipeline_resize_fused(self.handle))

    def detector_batch(self, s: int) -> torch.Tensor:
        """Copy of the detector batch of size s ([batch_cap[s], h_s, w_s, 3] u8) as last packed."""
        ptr = lib().otif_pipeline_detector_batch(self.handle, s)
        w, h = int(self.sizes[s][0]), int(self.sizes[s][1])
        shape = (self.batch_cap[s], h, w, 3)
        out = torch.empty(shape, dtype=torch.uint8, device="cuda")
        if ptr and out.numel():
            class _CAI:
                __cuda_array_interface__ = {"shape": shape, "typestr": "|u1", "data": (ptr, False), "version": 3}
            out.copy_(torch.as_tensor(_CAI(), device="cuda"))
        return out

    def frame_results(self, n: int):
        """(window-hash terms int64 [n], window counts int32 [n]) of the first n frames of the
        last device batch (copies; the per-clip hash is the wrapping sum over a clip's frames)."""
        hp = lib().otif_pipeline_frame_hashes(self.handle)
        cp = lib().otif_pipeline_frame_counts(self.handle)

        def view(ptr, typestr, dtype):
            class _CAI:
                __cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3}
            out = torch.empty(n, dtype=dtype, device="cuda")
            out.copy_(torch.as_tensor(_CAI(), device="cuda"))
            return out
        return view(hp, "<i8", torch.int64), view(cp, "<i4", torch.int32)

    def scores(self, n: int) -> torch.Tensor:
        """Copy of the cell scores fp32 [n, gh, gw] of the first n frames of the last device batch."""
        ptr = lib().otif_pipeline_scores(self.handle)
        shape = (n, self.grid[0], self.grid[1])

        class _CAI:
            __cuda_array_interface__ = {"shape": shape, "typestr": "<f4", "data": (ptr, False), "version": 3}
        out = torch.empty(shape, dtype=torch.float32, device="cuda")
        out.copy_(torch.as_tensor(_CAI(), device="cuda"))
        return out

    def pack_units(self):
        """Pack copy units per proxy GEMM layer since the last call (timing on, pack_overlap):
        dict E2, E3, E4, E5, D1, drain, total."""
        u = (ctypes.c_uint64 * 7)()
        check(lib().otif_pipeline_pack_units(self.handle, u), "otif_pipeline_pack_units")
        return dict(zip(("E2", "E3", "E4", "E5", "D1", "drain", "total"), [int(x) for x in u]))

    def flush(self, stream=None):
        """Complete a pack left pending by pack_overlap = 2."""
        check(lib().otif_pipeline_flush(self.handle, _stream(stream)), "otif_pipeline_flush")

    def counters(self) -> torch.Tensor:
        """int64 [15] device counters: frames, positive cells, windows, window pixels, window hash,
        windows per size [8], windows dropped for batch_cap, pixels of the windows packed."""
        ptr = lib().otif_pipeline_counters(self.handle)
        n = 15
        # wrap the device pointer without copying (read via a torch tensor view)
        return _device_view_i64(ptr, n)

    def set_timing(self, enable: bool = True):
        check(lib().otif_pipeline_set_timing(self.handle, int(enable)), "otif_pipeline_set_timing")

    def stage_ms(self):
        """-> (dict stage -> ms accumulated since the last call, kernel launches)."""
        ms = (ctypes.c_float * len(_lib.STAGES))()
        launches = ctypes.c_int64()
        check(lib().otif_pipeline_stage_ms(self.handle, ms, len(_lib.STAGES), ctypes.byref(launches)),
              "otif_pipeline_stage_ms")
        return dict(zip(_lib.STAGES, list(ms))), launches.value

    def reset_counters(self, stream=None):
        check(lib().otif_pipeline_reset_counters(self.handle, _stream(stream)), "otif_pipeline_reset_counters")

    def close(self):
        if getattr(self, "handle", None):
            lib().otif_pipeline_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _device_view_i64(ptr: int, n: int) -> torch.Tensor:
    out = torch.empty(n, dtype=torch.int64, device="cuda")
    # cudaMemcpy through torch: build a tensor from the raw pointer via __cuda_array_interface__
    class _CAI:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<i8", "data": (ptr, False), "version": 3}
    src = torch.as_tensor(_CAI(), device="cuda")
    out.copy_(src)
    return out
