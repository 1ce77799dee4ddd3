"""Seeded synthetic inputs (video frames, ground truth, proxy weights, workloads).

Shared by the oracle tests and the CUDA path; holds none of the method's arithmetic.
"""
from . import configs, video, weights  # noqa: F401
