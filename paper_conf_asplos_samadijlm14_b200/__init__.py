"""B200-native Paraprox Stencil & Partition approximation (Samadi et al.,
ASPLOS'14, §3.2).

The product is ``libparaprox.so`` (C ABI, include/paraprox.h) with hand-written
sm_100a kernels; ``paraprox`` is its thin ctypes binding and ``dist`` the
multi-GPU orchestration (frame sharding, row stripes with NCCL halo exchange,
HotSpot stripes).  Beyond the per-window schemes: the global-lattice reading
(``stencil_lattice``), the reduction schemes (``stencil_skip_xy``,
``tune_ex``), the runtime loop (``Runtime``) and HotSpot (``hotspot``).
Importing this package loads the library and fails loudly if it is missing.
"""
from . import paraprox  # noqa: F401
from .paraprox import (  # noqa: F401
    Filter,
    HotspotParams,
    ParaproxError,
    Prepared,
    Runtime,
    hotspot,
    prepare,
    quality_partials_async,
    stencil_lattice,
    stencil_lattice_xy,
    stencil_skip_xy,
    tune_candidates_ex,
    tune_decide_ex,
    tune_ex,
    tune_lattice,
    tune_lattice_decide,
    tune_lattice_partials,
    tune_partials_ex,
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
