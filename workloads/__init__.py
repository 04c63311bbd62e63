"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

Holds none of the method's arithmetic.  See ``images`` and ``filters``.
"""
from . import filters, images  # noqa: F401
from .images import fig5_statistic, frames, image, periodic, uniform_noise  # noqa: F401

# BASELINE.json configs (workload descriptors only)
CONFIGS = {
    "c1": dict(n=1, h=512, w=512, filter="gauss3", metric="mre"),
    "c2": dict(n=1, h=4096, w=4096, filter="mean5", metric="mre"),
    "c3": dict(n=256, h=2160, w=3840, filter="sep7", metric="l2"),
    "c4": dict(n=1, h=32768, w=32768, filter="conv9", metric="l2"),
}
