// knobs.cpp -- the library's environment settings, read once per process.
//
// Every setting keeps results bit-identical (stencil outputs) or within the
// 1e-12 quality bound (PARAPROX_FUSED_QUALITY); they select slower or
// alternative code paths for tests, sanitizers and measurements.  Defaults
// are the product configuration (README.md):
//
//   PARAPROX_FORCE_GENERIC=1   one-thread-per-output kernels instead of the
//                              tile / map / lattice kernels (default 0)
//   PARAPROX_FUSED_QUALITY=0   tuner candidates and runtime checks stored,
//                              then scored by the quality kernel (default 1)
//   PARAPROX_TMA_STORE=0       128-bit register stores instead of one TMA
//                              tensor store per tile (default 1)
//   PARAPROX_TILE_CHUNK=N      tiles per CTA of the tile kernels, 0 = fully
//                              persistent (default per instance: 4 for
//                              4-warp CTAs, 16 for 8-warp CTAs)
//   PARAPROX_LATTICE_CHUNK=N   the same for the lattice kernels (default 4;
//                              r02 sweep of 2, 4, 8, 16: 4 is +3..+8 % on
//                              c1 and c3 against 8, within +-3 % elsewhere)
//   PARAPROX_HOTSPOT_TB=0      HotSpot: one tile-kernel pass per step instead
//                              of the temporally blocked kernel (default 1)
#include <climits>
#include <cstdlib>

#include "internal.h"

namespace ppx {

static bool flag(const char* name, bool dflt) {
    const char* e = std::getenv(name);
    if (!e || !e[0]) return dflt;
    return e[0] != '0';
}

static int chunk(const char* name, int dflt) {
    const char* e = std::getenv(name);
    if (!e || !e[0]) return dflt;
    const int c = std::atoi(e);
    return c > 0 ? c : INT_MAX;
}

const Knobs& knobs() {
    static const Knobs k = [] {
        Knobs v;
        v.force_generic = flag("PARAPROX_FORCE_GENERIC", false);
        v.fused_quality = flag("PARAPROX_FUSED_QUALITY", true);
        v.tma_store = flag("PARAPROX_TMA_STORE", true);
        v.tile_chunk = chunk("PARAPROX_TILE_CHUNK", 0);  // 0: the instance's default
        v.lattice_chunk = chunk("PARAPROX_LATTICE_CHUNK", 4);
        v.hotspot_tb = flag("PARAPROX_HOTSPOT_TB", true);
        return v;
    }();
    return k;
}

}  // namespace ppx
