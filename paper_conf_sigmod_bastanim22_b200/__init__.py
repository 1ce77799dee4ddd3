"""B200-native (sm_100a) OTIF proxy + windowing hot path.

OTIF (Bastani & Madden, SIGMOD'22) scores every grid cell of a sampled video frame
with a small segmentation proxy CNN, thresholds the scores, groups the positive cells
into windows of a few fixed sizes and runs the object detector only on those windows,
batched per size.  This package is that per-frame path as hand-written CUDA kernels
behind a C ABI (include/otif.h, libotif.so) plus this thin Python binding.
"""
from .api import (Pipeline, Proxy, otif_pack_windows, otif_resize, otif_select_windows,  # noqa: F401
                  version, wsizes)
