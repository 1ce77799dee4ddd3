"""ctypes binding of libotif.so (include/otif.h).  Argument marshalling only: every
step of the path runs in the library's sm_100a kernels.  There is no fallback: if the
library is missing or the device is not sm_100, calls raise."""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("OTIF_LIB_OVERRIDE") or os.path.join(HERE, "libotif.so")

OK, EINVAL, ENOMEM, ECUDA, EUNSUPPORTED = 0, 1, 2, 3, 4


class OtifError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: status {status}: {detail}")
        self.status = status


class WSize(ctypes.Structure):
    _fields_ = [("w", ctypes.c_int32), ("h", ctypes.c_int32), ("cost", ctypes.c_int64)]


class Window(ctypes.Structure):
    _fields_ = [("frame", ctypes.c_int32), ("x", ctypes.c_int32), ("y", ctypes.c_int32),
                ("w", ctypes.c_int32), ("h", ctypes.c_int32), ("size_idx", ctypes.c_int32)]


class ProxyDesc(ctypes.Structure):
    _fields_ = [("in_h", ctypes.c_int32), ("in_w", ctypes.c_int32), ("n_strided", ctypes.c_int32),
                ("enc", ctypes.c_int32 * 5), ("dec", ctypes.c_int32)]


class GridDesc(ctypes.Structure):
    _fields_ = [("frame_w", ctypes.c_int32), ("frame_h", ctypes.c_int32), ("cell", ctypes.c_int32),
                ("connectivity", ctypes.c_int32)]


class PipelineDesc(ctypes.Structure):
    _fields_ = [("proxy", ProxyDesc), ("src_h", ctypes.c_int32), ("src_w", ctypes.c_int32),
                ("det_h", ctypes.c_int32), ("det_w", ctypes.c_int32), ("grid", GridDesc),
                ("threshold", ctypes.c_float), ("k", ctypes.c_int32), ("sizes", WSize * 8),
                ("max_batch", ctypes.c_int32), ("batch_cap", ctypes.c_int32 * 8), ("proxy_batch", ctypes.c_int32),
                ("pack_overlap", ctypes.c_int32)]


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libotif.so not built at {LIB_PATH}: run __graft_entry__.build() "
                           "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, i32, sz, st = ctypes.c_void_p, ctypes.c_int32, ctypes.c_size_t, ctypes.c_int
    L.otif_status_str.restype = ctypes.c_char_p
    L.otif_status_str.argtypes = [st]
    L.otif_last_error.restype = ctypes.c_char_p
    L.otif_version.restype = ctypes.c_char_p
    L.otif_resize.argtypes = [P, i32, i32, i32, P, i32, i32, P]
    L.otif_resize.restype = st
    L.otif_proxy_create.argtypes = [ctypes.POINTER(ProxyDesc), P, sz, ctypes.POINTER(P)]
    L.otif_proxy_create.restype = st
    L.otif_proxy_destroy.argtypes = [P]
    L.otif_proxy_destroy.restype = None
    L.otif_proxy_grid.argtypes = [P, P, P]
    L.otif_proxy_grid.restype = st
    L.otif_proxy_workspace_bytes.argtypes = [P, i32]
    L.otif_proxy_workspace_bytes.restype = sz
    L.otif_proxy_score.argtypes = [P, P, i32, P, P, sz, P]
    L.otif_proxy_score.restype = st
    L.otif_select_workspace_bytes.argtypes = [i32, i32, i32]
    L.otif_select_workspace_bytes.restype = sz
    L.otif_select_windows.argtypes = [P, P, ctypes.c_float, i32, i32, i32, ctypes.POINTER(GridDesc), P, i32,
                                      P, P, i32, P, P, P, P, sz, P, P]
    L.otif_select_windows.restype = st
    L.otif_pack_windows.argtypes = [P, i32, i32, i32, i32, i32, P, P, i32, P, i32, P, P, P, P, P]
    L.otif_pack_windows.restype = st
    L.otif_choose_workspace_bytes.argtypes = [i32, i32, i32, i32]
    L.otif_choose_workspace_bytes.restype = sz
    L.otif_choose_window_sizes.argtypes = [P, i32, i32, i32, ctypes.POINTER(GridDesc), P, i32, ctypes.c_int64, i32,
                                           P, P, P, sz, P]
    L.otif_choose_window_sizes.restype = st
    L.otif_window_recall.argtypes = [P, ctypes.c_int64, P, P, P, i32, P, P]
    L.otif_window_recall.restype = st
    i64, f32 = ctypes.c_int64, ctypes.c_float
    L.otif_track_resample.argtypes = [P, P, i64, i32, P, P]
    L.otif_track_resample.restype = st
    L.otif_dbscan_workspace_bytes.argtypes = [i64]
    L.otif_dbscan_workspace_bytes.restype = sz
    L.otif_track_dbscan.argtypes = [P, i64, i32, f32, i32, P, P, P, P, sz, P]
    L.otif_track_dbscan.restype = st
    L.otif_centers_workspace_bytes.argtypes = [i64, i32]
    L.otif_centers_workspace_bytes.restype = sz
    L.otif_track_centers.argtypes = [P, P, i64, i32, i32, P, P, P, sz, P]
    L.otif_track_centers.restype = st
    L.otif_track_refine.argtypes = [P, P, i64, i32, P, P, i32, i32, f32, P, P, P]
    L.otif_track_refine.restype = st
    L.otif_cell_labels.argtypes = [P, i64, i32, i32, i32, ctypes.POINTER(GridDesc), P, P]
    L.otif_cell_labels.restype = st
    L.otif_adam_step.argtypes = [P, P, P, P, i64, i32, f32, f32, f32, f32, P]
    L.otif_adam_step.restype = st
    L.otif_trainer_create.argtypes = [ctypes.POINTER(ProxyDesc), P, sz, i32, ctypes.POINTER(P)]
    L.otif_trainer_create.restype = st
    L.otif_trainer_destroy.argtypes = [P]
    L.otif_trainer_destroy.restype = None
    L.otif_trainer_params.argtypes = [P, ctypes.POINTER(P), ctypes.POINTER(P), ctypes.POINTER(sz),
                                      ctypes.POINTER(i32), ctypes.POINTER(i32)]
    L.otif_trainer_params.restype = st
    L.otif_trainer_backward.argtypes = [P, P, P, i32, P, P]
    L.otif_trainer_backward.restype = st
    L.otif_trainer_adam.argtypes = [P, f32, P]
    L.otif_trainer_adam.restype = st
    if hasattr(L, "otif_pipeline_create"):
        L.otif_pipeline_create.argtypes = [ctypes.POINTER(PipelineDesc), P, sz, ctypes.POINTER(P)]
        L.otif_pipeline_create.restype = st
        L.otif_pipeline_destroy.argtypes = [P]
        L.otif_pipeline_destroy.restype = None
        L.otif_pipeline_run_host.argtypes = [P, P, i32, P, i32, P, P, P]
        L.otif_pipeline_run_host.restype = st
        L.otif_pipeline_run_device.argtypes = [P, P, i32, ctypes.c_int64, P]
        L.otif_pipeline_run_device.restype = st
        L.otif_pipeline_frame_hashes.argtypes = [P]
        L.otif_pipeline_frame_hashes.restype = P
        L.otif_pipeline_frame_counts.argtypes = [P]
        L.otif_pipeline_frame_counts.restype = P
        L.otif_pipeline_scores.argtypes = [P]
        L.otif_pipeline_scores.restype = P
        L.otif_pipeline_pack_units.argtypes = [P, ctypes.POINTER(ctypes.c_uint64)]
        L.otif_pipeline_pack_units.restype = ctypes.c_int
        L.otif_pipeline_resize_fused.argtypes = [P]
        L.otif_pipeline_resize_fused.restype = i32
        L.otif_pipeline_detector_batch.argtypes = [P, i32]
        L.otif_pipeline_detector_batch.restype = P
        L.otif_pipeline_flush.argtypes = [P, P]
        L.otif_pipeline_flush.restype = st
        L.otif_pipeline_counters.argtypes = [P]
        L.otif_pipeline_counters.restype = P
        L.otif_pipeline_reset_counters.argtypes = [P, P]
        L.otif_pipeline_reset_counters.restype = st
        L.otif_pipeline_set_timing.argtypes = [P, i32]
        L.otif_pipeline_set_timing.restype = st
        L.otif_pipeline_stage_ms.argtypes = [P, P, i32, P]
        L.otif_pipeline_stage_ms.restype = st
    _lib = L
    return L


def check(status: int, where: str) -> None:
    if status != OK:
        raise OtifError(status, where, lib().otif_last_error().decode(errors="replace"))


# symbols include/otif.h declares (tests check the library exports every one)
EXPORTED = ("otif_status_str", "otif_last_error", "otif_version", "otif_resize", "otif_proxy_create",
            "otif_proxy_destroy", "otif_proxy_grid", "otif_proxy_workspace_bytes", "otif_proxy_score",
            "otif_select_workspace_bytes", "otif_select_windows", "otif_pack_windows",
            "otif_pipeline_create", "otif_pipeline_destroy", "otif_pipeline_run_host",
            "otif_pipeline_run_device", "otif_pipeline_flush", "otif_pipeline_resize_fused", "otif_pipeline_detector_batch", "otif_pipeline_frame_hashes",
            "otif_pipeline_frame_counts", "otif_pipeline_scores", "otif_pipeline_pack_units", "otif_pipeline_counters", "otif_pipeline_reset_counters",
            "otif_pipeline_set_timing", "otif_pipeline_stage_ms", "otif_choose_workspace_bytes",
            "otif_choose_window_sizes", "otif_window_recall", "otif_track_resample", "otif_dbscan_workspace_bytes",
            "otif_track_dbscan", "otif_centers_workspace_bytes", "otif_track_centers", "otif_track_refine",
            "otif_cell_labels", "otif_adam_step", "otif_trainer_create", "otif_trainer_destroy", "otif_trainer_params",
            "otif_trainer_backward", "otif_trainer_adam")
STAGES = ("resize", "proxy_prep_e1", "conv_e2", "conv_e3", "conv_e4", "conv_e5", "conv_d1_head", "select",
          "pack", "append")
