"""§8(f) NEXT-3 — proxy training labels and training on top of the C ABI.
Argument marshalling only: labels, the forward/backward convolutions, the loss and Adam
run in libotif (csrc/train.cu).

    tr = Trainer(in_h, in_w, n_strided, weights)        # fp32 master weights on the device
    labels = otif_cell_labels(boxes, n, grid, frame_w, frame_h, cell)
    loss = tr.step(img, labels, lr=1e-3)                 # backward + Adam
    proxy = Proxy(in_h, in_w, n_strided, tr.weights())   # inference with the trained model
"""
from __future__ import annotations

import ctypes
from typing import Sequence

import numpy as np
import torch

from .api import _ptr, _require_cuda, _stream
from ._lib import GridDesc, ProxyDesc, check, lib


def otif_cell_labels(boxes: torch.Tensor, n: int, grid: tuple, frame_w: int, frame_h: int, cell: int,
                     out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """P:L139 labels: boxes int32 [nb, 5] (frame, x0, y0, x1, y1) on the device -> u8 [n, gh, gw]."""
    _require_cuda(boxes)
    assert boxes.dtype == torch.int32 and boxes.shape[-1] == 5
    gh, gw = grid
    if out is None:
        out = torch.empty((n, gh, gw), dtype=torch.uint8, device=boxes.device)
    g = GridDesc(frame_w, frame_h, cell, 4)
    check(lib().otif_cell_labels(_ptr(boxes), boxes.shape[0], n, gh, gw, ctypes.byref(g), _ptr(out),
                                 _stream(stream)), "otif_cell_labels")
    return out


def otif_adam_step(w: torch.Tensor, m: torch.Tensor, v: torch.Tensor, g: torch.Tensor, t: int, lr: float,
                   b1: float = 0.9, b2: float = 0.999, eps: float = 1e-8, stream=None):
    """Reading R27 Adam step on fp32 device tensors, in place."""
    _require_cuda(w, m, v, g)
    check(lib().otif_adam_step(_ptr(w), _ptr(m), _ptr(v), _ptr(g), w.numel(), t, lr, b1, b2, eps, _stream(stream)),
          "otif_adam_step")


class Trainer:
    """otif_trainer_*: fp32 training of the proxy CNN (BCE vs cell labels, Adam)."""

    def __init__(self, in_h: int, in_w: int, n_strided: int, weights: np.ndarray, max_batch: int = 32,
                 enc: Sequence[int] = (32, 64, 128, 256, 256), dec: int = 128):
        d = ProxyDesc()
        d.in_h, d.in_w, d.n_strided = in_h, in_w, n_strided
        for i, e in enumerate(enc):
            d.enc[i] = int(e)
        d.dec = int(dec)
        w = np.ascontiguousarray(weights, np.float32)
        h = ctypes.c_void_p()
        check(lib().otif_trainer_create(ctypes.byref(d), ctypes.c_void_p(w.ctypes.data), w.size, max_batch,
                                        ctypes.byref(h)), "otif_trainer_create")
        self.handle = h
        self.enc, self.dec, self.n_strided = tuple(enc), dec, n_strided
        self.in_h, self.in_w, self.max_batch = in_h, in_w, max_batch
        pw, pg, nw = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_size_t()
        gh, gw = ctypes.c_int32(), ctypes.c_int32()
        check(lib().otif_trainer_params(h, ctypes.byref(pw), ctypes.byref(pg), ctypes.byref(nw), ctypes.byref(gh),
                                        ctypes.byref(gw)), "otif_trainer_params")
        self.n_weights = nw.value
        self.grid = (gh.value, gw.value)
        self._pw, self._pg = pw.value, pg.value
        self._loss = torch.zeros(1, dtype=torch.float32, device="cuda")

    def _view(self, ptr: int) -> torch.Tensor:
        """Device tensor aliasing trainer-owned memory (no copy)."""
        class _CAI:
            __cuda_array_interface__ = {"shape": (self.n_weights,), "typestr": "<f4", "data": (ptr, False),
                                        "version": 3, "strides": None}
        return torch.as_tensor(_CAI(), device="cuda")

    def weights_tensor(self) -> torch.Tensor:
        return self._view(self._pw)

    def grads_tensor(self) -> torch.Tensor:
        return self._view(self._pg)

    def weights(self) -> np.ndarray:
        torch.cuda.synchronize()
        return self.weights_tensor().cpu().numpy().copy()

    def backward(self, img: torch.Tensor, labels: torch.Tensor, stream=None) -> torch.Tensor:
        """Forward + loss + gradients; returns the device loss (1-element tensor, no sync)."""
        _require_cuda(img, labels)
        n = img.shape[0]
        assert img.dtype == torch.uint8 and tuple(img.shape[1:]) == (self.in_h, self.in_w, 3)
        assert labels.dtype == torch.uint8 and tuple(labels.shape) == (n,) + self.grid
        check(lib().otif_trainer_backward(self.handle, _ptr(img), _ptr(labels), n, _ptr(self._loss),
                                          _stream(stream)), "otif_trainer_backward")
        return self._loss

    def adam(self, lr: float, stream=None):
        check(lib().otif_trainer_adam(self.handle, lr, _stream(stream)), "otif_trainer_adam")

    def step(self, img: torch.Tensor, labels: torch.Tensor, lr: float = 1e-3, stream=None) -> torch.Tensor:
        loss = self.backward(img, labels, stream)
        self.adam(lr, stream)
        return loss

    def __del__(self):
        h = getattr(self, "handle", None)
        if h is not None and h.value:
            try:
                lib().otif_trainer_destroy(h)
            except Exception:
                pass
            self.handle = None
