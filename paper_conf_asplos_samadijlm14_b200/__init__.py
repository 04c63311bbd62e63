"""B200-native Paraprox Stencil & Partition approximation (Samadi et al.,
ASPLOS'14, §3.2).

The product is ``libparaprox.so`` (C ABI, include/paraprox.h) with hand-written
sm_100a kernels; ``paraprox`` is its thin ctypes binding and ``dist`` the
multi-GPU orchestration (frame sharding, row stripes with NCCL halo exchange).
Importing this package loads the library and fails loudly if it is missing.
"""
from . import paraprox  # noqa: F401
from .paraprox import (  # noqa: F401
    Filter,
    ParaproxError,
    filter_create,
    filter_create_separable,
    quality,
    quality_from_partials,
    quality_partials,
    run_host,
    stencil_approx,
    stencil_approx_xy,
    stencil_exact,
    tune,
    tune_candidates,
    tune_decide,
    tune_partials,
)

__all__ = [n for n in dir() if not n.startswith("_")]
