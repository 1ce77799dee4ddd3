"""§8(f) NEXT-4 — track refinement on top of the C ABI.  Argument
marshalling only: resampling, the DBSCAN neighbourhood bitmap, components, centres and
the k-nearest-cluster refinement all run in libotif (csrc/tracks.cu).

    idx = TrackIndex.build(pts, offsets, eps, min_pts)     # S*, offline
    out, used = idx.refine(qpts, qoffsets, k=10, rho=32)   # inference
"""
from __future__ import annotations

import dataclasses

import torch

from .api import _ptr, _require_cuda, _stream
from ._lib import check, lib


def _tracks(pts: torch.Tensor, offsets: torch.Tensor):
    _require_cuda(pts, offsets)
    assert pts.dtype == torch.float32 and pts.shape[-1] == 2, "pts: float32 [total, 2]"
    assert offsets.dtype == torch.int64 and offsets.dim() == 1, "offsets: int64 [n + 1]"
    return offsets.shape[0] - 1


def otif_track_resample(pts: torch.Tensor, offsets: torch.Tensor, npts: int = 20, out: torch.Tensor | None = None,
                        stream=None) -> torch.Tensor:
    """P:L196 arc-length resampling -> float32 [n, npts, 2] (reading R21)."""
    n = _tracks(pts, offsets)
    if out is None:
        out = torch.empty((n, npts, 2), dtype=torch.float32, device=pts.device)
    check(lib().otif_track_resample(_ptr(pts), _ptr(offsets), n, npts, _ptr(out), _stream(stream)),
          "otif_track_resample")
    return out


def otif_track_dbscan(P: torch.Tensor, eps: float, min_pts: int, workspace: torch.Tensor | None = None,
                      stream=None):
    """P:L198 DBSCAN over resampled tracks [n, npts, 2] (reading R23).
    -> (labels int32 [n], core uint8 [n], n_clusters int32 [1]) on the device (no sync)."""
    _require_cuda(P)
    n, npts = P.shape[0], P.shape[1]
    labels = torch.empty(n, dtype=torch.int32, device=P.device)
    core = torch.empty(n, dtype=torch.uint8, device=P.device)
    nc = torch.zeros(1, dtype=torch.int32, device=P.device)
    need = int(lib().otif_dbscan_workspace_bytes(n))
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(max(need, 1), dtype=torch.uint8, device=P.device)
    check(lib().otif_track_dbscan(_ptr(P), n, npts, float(eps), int(min_pts), _ptr(labels), _ptr(core), _ptr(nc),
                                  _ptr(workspace), workspace.numel(), _stream(stream)), "otif_track_dbscan")
    return labels, core, nc


def otif_track_centers(P: torch.Tensor, labels: torch.Tensor, nc: int, stream=None):
    """P:L198 cluster centres -> (centers float32 [nc, npts, 2], sizes int32 [nc])."""
    _require_cuda(P, labels)
    n, npts = P.shape[0], P.shape[1]
    centers = torch.empty((nc, npts, 2), dtype=torch.float32, device=P.device)
    sizes = torch.empty(nc, dtype=torch.int32, device=P.device)
    ws = torch.empty(max(int(lib().otif_centers_workspace_bytes(n, nc)), 1), dtype=torch.uint8, device=P.device)
    check(lib().otif_track_centers(_ptr(P), _ptr(labels), n, npts, nc, _ptr(centers), _ptr(sizes), _ptr(ws),
                                   ws.numel(), _stream(stream)), "otif_track_centers")
    return centers, sizes


def otif_track_refine(pts: torch.Tensor, offsets: torch.Tensor, centers: torch.Tensor, sizes: torch.Tensor,
                      k: int = 10, rho: float = 0.0, stream=None):
    """P:L200 refinement -> (out float32 [m, 4] = start x, y, end x, y; used int32 [m])."""
    m = _tracks(pts, offsets)
    _require_cuda(centers, sizes)
    nc, npts = centers.shape[0], centers.shape[1]
    out = torch.empty((m, 4), dtype=torch.float32, device=pts.device)
    used = torch.empty(m, dtype=torch.int32, device=pts.device)
    check(lib().otif_track_refine(_ptr(pts), _ptr(offsets), m, npts, _ptr(centers), _ptr(sizes), nc, int(k),
                                  float(rho), _ptr(out), _ptr(used), _stream(stream)), "otif_track_refine")
    return out, used


@dataclasses.dataclass
class TrackIndex:
    """Clusters of S* and their centres."""
    centers: torch.Tensor
    sizes: torch.Tensor
    labels: torch.Tensor
    core: torch.Tensor
    npts: int

    @classmethod
    def build(cls, pts: torch.Tensor, offsets: torch.Tensor, eps: float, min_pts: int, npts: int = 20,
              stream=None) -> "TrackIndex":
        """Resample, DBSCAN, centres.  One device->host read of the cluster count."""
        P = otif_track_resample(pts, offsets, npts, stream=stream)
        labels, core, nc = otif_track_dbscan(P, eps, min_pts, stream=stream)
        n_clusters = int(nc.item())
        centers, sizes = otif_track_centers(P, labels, n_clusters, stream=stream)
        return cls(centers, sizes, labels, core, npts)

    def refine(self, pts: torch.Tensor, offsets: torch.Tensor, k: int = 10, rho: float = 0.0, stream=None):
        return otif_track_refine(pts, offsets, self.centers, self.sizes, k, rho, stream=stream)
