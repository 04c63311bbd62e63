"""ctypes wrapper over ``liboracle.so`` (plain C, fp64; see ``oracle.h``).

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).  Every function cites
the PAPER.md passage it follows in ``oracle.c``.  Inputs are fp32 numpy
arrays (the seeded generators in ``workloads/``); outputs are fp64.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

EXACT, ROW, COL, CENTER = 0, 1, 2, 3
SKIP_ROW, SKIP_COL, SKIP_BOTH = 4, 5, 6
MRE, L2, PSNR = 0, 1, 2
SCHEMES = {"exact": EXACT, "row": ROW, "col": COL, "center": CENTER, "centre": CENTER,
           "skip_row": SKIP_ROW, "skip_col": SKIP_COL, "skip_both": SKIP_BOTH}
METRICS = {"mre": MRE, "l2": L2, "psnr": PSNR}
SCHEME_NAMES = {EXACT: "exact", ROW: "row", COL: "col", CENTER: "center", SKIP_ROW: "skip_row",
                SKIP_COL: "skip_col", SKIP_BOTH: "skip_both"}


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2, OpenMP, no fast-math)."""
    stale = not os.path.exists(_LIB) or max(os.path.getmtime(_SRC), os.path.getmtime(_HDR)) > os.path.getmtime(_LIB)
    if force or stale:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-Wall", "-Wextra", "-Wno-unused-parameter",
                               _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.POINTER
        f32, f64, i32 = P(C.c_float), P(C.c_double), P(C.c_int)
        _lib.oracle_index_map.argtypes = [C.c_int, C.c_int, i32]
        _lib.oracle_scheme_reaches.argtypes = [C.c_int, C.c_int, i32, i32]
        _lib.oracle_stencil_exact.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, C.c_int, f64]
        _lib.oracle_stencil_approx.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, C.c_int,
                                               C.c_int, C.c_int, f64]
        _lib.oracle_stencil_sep.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                            C.c_int, C.c_int, f64]
        _lib.oracle_quality.argtypes = [f64, f64, C.c_longlong, C.c_int, f64]
        _lib.oracle_lattice_map.argtypes = [C.c_int, C.c_int, i32]
        _lib.oracle_stencil_lattice.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, C.c_int,
                                                C.c_int, C.c_int, f64]
        _lib.oracle_stencil_lattice_sep.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                                    C.c_int, C.c_int, f64]
        _lib.oracle_tune_candidates.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, i32, i32]
        _lib.oracle_tune.argtypes = [f32, C.c_int, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                     C.c_double, C.c_int, C.c_int, f64, i32, i32, i32, f64]
        _lib.oracle_tune_lattice.argtypes = [f32, C.c_int, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                             C.c_double, C.c_int, f64, i32, i32, f64]
        _lib.oracle_scheme_skips.argtypes = [C.c_int, C.c_int, i32, i32]
        _lib.oracle_stencil_skip.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, C.c_int,
                                             C.c_int, C.c_int, f64]
        _lib.oracle_stencil_skip_sep.argtypes = [f32, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                                 C.c_int, C.c_int, f64]
        _lib.oracle_tune_candidates_ex.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, i32, i32]
        _lib.oracle_tune_ex.argtypes = [f32, C.c_int, C.c_int, C.c_int, C.c_int, f32, C.c_int, f32, C.c_int,
                                        C.c_int, C.c_double, C.c_int, C.c_int, f64, i32, i32, i32, f64]
        _lib.oracle_hotspot.argtypes = [f32, f32, C.c_int, C.c_int, C.c_int, C.c_double, C.c_double, C.c_double,
                                        C.c_double, C.c_double, C.c_int, C.c_int, C.c_int, f64]
        _lib.oracle_runtime_ladder.argtypes = [C.c_int, f64, C.c_double, C.c_int, i32]
        _lib.oracle_runtime_trace.argtypes = [C.c_int, C.c_int, C.c_double, C.c_int, f64, i32, i32,
                                              P(C.c_longlong), P(C.c_longlong)]
        for name in ("oracle_runtime_ladder", "oracle_runtime_trace", "oracle_hotspot", "oracle_scheme_skips", "oracle_stencil_skip", "oracle_stencil_skip_sep",
                     "oracle_tune_candidates_ex", "oracle_tune_ex", "oracle_tune_lattice", "oracle_lattice_map", "oracle_stencil_lattice", "oracle_stencil_lattice_sep",
                     "oracle_index_map", "oracle_scheme_reaches", "oracle_stencil_exact",
                     "oracle_stencil_approx", "oracle_stencil_sep", "oracle_quality",
                     "oracle_tune_candidates", "oracle_tune"):
            getattr(_lib, name).restype = C.c_int
    return _lib


def _fp(a):
    return a.ctypes.data_as(C.POINTER(C.c_float))


def _dp(a):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _frames(x):
    x = np.ascontiguousarray(x, dtype=np.float32)
    if x.ndim == 2:
        return x[None], True
    if x.ndim != 3:
        raise ValueError("expected [h, w] or [n, h, w]")
    return x, False


def _ok(rc, what):
    if rc != 0:
        raise ValueError(f"oracle: {what} rejected its arguments")


def index_map(r: int, d: int) -> np.ndarray:
    """m[i + r] for i in [-r, r] (§3.2.3; reading S5)."""
    m = np.zeros(2 * r + 1, dtype=np.int32)
    _ok(lib().oracle_index_map(r, d, m.ctypes.data_as(C.POINTER(C.c_int))), "index_map")
    return m


def scheme_reaches(scheme, reach: int):
    s = SCHEMES[scheme] if isinstance(scheme, str) else int(scheme)
    dy, dx = C.c_int(), C.c_int()
    _ok(lib().oracle_scheme_reaches(s, reach, C.byref(dy), C.byref(dx)), "scheme_reaches")
    return dy.value, dx.value


def stencil_exact(x, w) -> np.ndarray:
    """E = sum_ij w[i][j] X(clamp(y+i), clamp(x+j)) in fp64."""
    x, squeeze = _frames(x)
    w = np.ascontiguousarray(w, dtype=np.float32)
    out = np.empty(x.shape, dtype=np.float64)
    n, h, ww = x.shape
    _ok(lib().oracle_stencil_exact(_fp(x), n, h, ww, _fp(w), w.shape[0], w.shape[1], _dp(out)),
        "stencil_exact")
    return out[0] if squeeze else out


def stencil_approx_xy(x, w, dy: int, dx: int) -> np.ndarray:
    """Literal per-window substitution with per-axis reaches (dy, dx)."""
    x, squeeze = _frames(x)
    w = np.ascontiguousarray(w, dtype=np.float32)
    out = np.empty(x.shape, dtype=np.float64)
    n, h, ww = x.shape
    _ok(lib().oracle_stencil_approx(_fp(x), n, h, ww, _fp(w), w.shape[0], w.shape[1], dy, dx, _dp(out)),
        "stencil_approx")
    return out[0] if squeeze else out


def stencil_approx(x, w, scheme, reach: int) -> np.ndarray:
    dy, dx = scheme_reaches(scheme, reach)
    return stencil_approx_xy(x, w, dy, dx)


def stencil_sep(x, wy, wx, dy: int = 0, dx: int = 0) -> np.ndarray:
    x, squeeze = _frames(x)
    wy = np.ascontiguousarray(wy, dtype=np.float32).ravel()
    wx = np.ascontiguousarray(wx, dtype=np.float32).ravel()
    out = np.empty(x.shape, dtype=np.float64)
    n, h, ww = x.shape
    _ok(lib().oracle_stencil_sep(_fp(x), n, h, ww, _fp(wy), wy.size, _fp(wx), wx.size, dy, dx, _dp(out)),
        "stencil_sep")
    return out[0] if squeeze else out


def lattice_map(length: int, d: int) -> np.ndarray:
    """Global-lattice map of one axis (reading G): g[t] for t in [0, length)."""
    g = np.zeros(max(length, 1), dtype=np.int32)
    _ok(lib().oracle_lattice_map(int(length), int(d), g.ctypes.data_as(C.POINTER(C.c_int))), "lattice_map")
    return g[:length]


def stencil_lattice_xy(x, w, dy: int, dx: int) -> np.ndarray:
    """Exact stencil on the replicated array X~ (reading G).
    ``w`` is a 2-D array (dense) or a (wy, wx) pair (separable)."""
    x, squeeze = _frames(x)
    out = np.empty(x.shape, dtype=np.float64)
    n, h, ww = x.shape
    if isinstance(w, (tuple, list)):
        wy = np.ascontiguousarray(w[0], dtype=np.float32).ravel()
        wx = np.ascontiguousarray(w[1], dtype=np.float32).ravel()
        _ok(lib().oracle_stencil_lattice_sep(_fp(x), n, h, ww, _fp(wy), wy.size, _fp(wx), wx.size, dy, dx,
                                             _dp(out)), "stencil_lattice_sep")
    else:
        w = np.ascontiguousarray(w, dtype=np.float32)
        _ok(lib().oracle_stencil_lattice(_fp(x), n, h, ww, _fp(w), w.shape[0], w.shape[1], dy, dx, _dp(out)),
            "stencil_lattice")
    return out[0] if squeeze else out


def stencil_lattice(x, w, scheme, reach: int) -> np.ndarray:
    dy, dx = scheme_reaches(scheme, reach)
    return stencil_lattice_xy(x, w, dy, dx)


def stencil_sep_scheme(x, wy, wx, scheme, reach: int) -> np.ndarray:
    dy, dx = scheme_reaches(scheme, reach)
    return stencil_sep(x, wy, wx, dy, dx)


def quality(e, a, metric="mre") -> float:
    """1 - MRE / 1 - L2 (Table 1) or PSNR dB (not a paper metric)."""
    m = METRICS[metric] if isinstance(metric, str) else int(metric)
    e = np.ascontiguousarray(e, dtype=np.float64).ravel()
    a = np.ascontiguousarray(a, dtype=np.float64).ravel()
    if e.size != a.size:
        raise ValueError("size mismatch")
    q = C.c_double()
    _ok(lib().oracle_quality(_dp(e), _dp(a), e.size, m, C.byref(q)), "quality")
    return q.value


def tune_candidates(ky: int, kx: int, separable: bool = False):
    cap = 64
    s = np.zeros(cap, dtype=np.int32)
    r = np.zeros(cap, dtype=np.int32)
    n = lib().oracle_tune_candidates(ky, kx, int(separable), cap,
                                     s.ctypes.data_as(C.POINTER(C.c_int)),
                                     r.ctypes.data_as(C.POINTER(C.c_int)))
    if n < 0:
        raise ValueError("tune_candidates rejected its arguments")
    return [(SCHEME_NAMES[int(s[i])], int(r[i])) for i in range(n)]


def tune(x, w, toq: float, metric="mre", all_qualities: bool = False):
    """Oracle tuner.  ``w`` is a 2-D array (dense) or a (wy, wx) pair
    (separable).  Returns dict(scheme, reach, quality, qualities)."""
    x, _ = _frames(x)
    m = METRICS[metric] if isinstance(metric, str) else int(metric)
    n, h, ww = x.shape
    if isinstance(w, (tuple, list)):
        wy = np.ascontiguousarray(w[0], dtype=np.float32).ravel()
        wx = np.ascontiguousarray(w[1], dtype=np.float32).ravel()
        sep, ky, kx, wa, wb = 1, wy.size, wx.size, wy, wx
    else:
        wa = np.ascontiguousarray(w, dtype=np.float32)
        sep, ky, kx, wb = 0, wa.shape[0], wa.shape[1], wa
    cap = 64
    qs = np.full(cap, np.nan)
    nev, sc, rc = C.c_int(), C.c_int(), C.c_int()
    q = C.c_double()
    _ok(lib().oracle_tune(_fp(x), n, h, ww, sep, _fp(wa), ky, _fp(wb), kx, float(toq), m, cap,
                          _dp(qs) if all_qualities else None, C.byref(nev), C.byref(sc), C.byref(rc),
                          C.byref(q)), "tune")
    return dict(scheme=SCHEME_NAMES[sc.value], reach=rc.value, quality=q.value,
                qualities=[float(v) for v in qs[:nev.value]] if all_qualities else None)


def tune_lattice(x, w, toq: float, metric="mre"):
    """Oracle lattice tuner: row lattice reach 4, 3, 2, 1, first with quality
    >= toq, else exact.  Returns dict(scheme, reach, quality, qualities)."""
    x, _ = _frames(x)
    m = METRICS[metric] if isinstance(metric, str) else int(metric)
    n, h, ww = x.shape
    if isinstance(w, (tuple, list)):
        wa = np.ascontiguousarray(w[0], dtype=np.float32).ravel()
        wb = np.ascontiguousarray(w[1], dtype=np.float32).ravel()
        sep, ky, kx = 1, wa.size, wb.size
    else:
        wa = np.ascontiguousarray(w, dtype=np.float32)
        sep, ky, kx, wb = 0, wa.shape[0], wa.shape[1], wa
    qs = np.full(4, np.nan)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _ok(lib().oracle_tune_lattice(_fp(x), n, h, ww, sep, _fp(wa), ky, _fp(wb), kx, float(toq), m, _dp(qs),
                                  C.byref(sc), C.byref(rc), C.byref(q)), "tune_lattice")
    return dict(scheme=SCHEME_NAMES[sc.value], reach=rc.value, quality=q.value, qualities=[float(v) for v in qs])


def stencil_skip_xy(x, w, ny: int, nx: int) -> np.ndarray:
    """Reduction approximation of the stencil loops:
    every ny-th filter row / nx-th filter column, each loop scaled by its rate.
    ``w`` is a 2-D array (dense) or a (wy, wx) pair (separable)."""
    x, squeeze = _frames(x)
    out = np.empty(x.shape, dtype=np.float64)
    n, h, ww = x.shape
    if isinstance(w, (tuple, list)):
        wy = np.ascontiguousarray(w[0], dtype=np.float32).ravel()
        wx = np.ascontiguousarray(w[1], dtype=np.float32).ravel()
        _ok(lib().oracle_stencil_skip_sep(_fp(x), n, h, ww, _fp(wy), wy.size, _fp(wx), wx.size, ny, nx, _dp(out)),
            "stencil_skip_sep")
    else:
        w = np.ascontiguousarray(w, dtype=np.float32)
        _ok(lib().oracle_stencil_skip(_fp(x), n, h, ww, _fp(w), w.shape[0], w.shape[1], ny, nx, _dp(out)),
            "stencil_skip")
    return out[0] if squeeze else out


def scheme_skips(scheme, rate: int):
    ny, nx = C.c_int(), C.c_int()
    s = SCHEMES[scheme] if isinstance(scheme, str) else int(scheme)
    _ok(lib().oracle_scheme_skips(s, int(rate), C.byref(ny), C.byref(nx)), "scheme_skips")
    return ny.value, nx.value


def stencil_scheme(x, w, scheme, reach: int) -> np.ndarray:
    """Any scheme of the library (stencil or reduction), dense or separable."""
    s = SCHEMES[scheme] if isinstance(scheme, str) else int(scheme)
    if s >= SKIP_ROW:
        return stencil_skip_xy(x, w, *scheme_skips(s, reach))
    if isinstance(w, (tuple, list)):
        return stencil_sep_scheme(x, w[0], w[1], s, reach)
    return stencil_approx(x, w, s, reach)


def tune_candidates_ex(ky: int, kx: int, separable: bool = False, flags: int = 3):
    cap = 128
    s = np.zeros(cap, dtype=np.int32)
    r = np.zeros(cap, dtype=np.int32)
    n = lib().oracle_tune_candidates_ex(ky, kx, int(separable), int(flags), cap,
                                        s.ctypes.data_as(C.POINTER(C.c_int)), r.ctypes.data_as(C.POINTER(C.c_int)))
    if n < 0:
        raise ValueError("tune_candidates_ex rejected its arguments")
    return [(SCHEME_NAMES[int(s[i])], int(r[i])) for i in range(n)]


def tune_ex(x, w, toq: float, metric="mre", flags: int = 3, all_qualities: bool = False):
    """Extended oracle tuner over stencil (bit 0) and reduction (bit 1) schemes."""
    x, _ = _frames(x)
    m = METRICS[metric] if isinstance(metric, str) else int(metric)
    n, h, ww = x.shape
    if isinstance(w, (tuple, list)):
        wa = np.ascontiguousarray(w[0], dtype=np.float32).ravel()
        wb = np.ascontiguousarray(w[1], dtype=np.float32).ravel()
        sep, ky, kx = 1, wa.size, wb.size
    else:
        wa = np.ascontiguousarray(w, dtype=np.float32)
        sep, ky, kx, wb = 0, wa.shape[0], wa.shape[1], wa
    cap = 128
    qs = np.full(cap, np.nan)
    nev, sc, rc = C.c_int(), C.c_int(), C.c_int()
    q = C.c_double()
    _ok(lib().oracle_tune_ex(_fp(x), n, h, ww, sep, _fp(wa), ky, _fp(wb), kx, int(flags), float(toq), m, cap,
                             _dp(qs) if all_qualities else None, C.byref(nev), C.byref(sc), C.byref(rc),
                             C.byref(q)), "tune_ex")
    return dict(scheme=SCHEME_NAMES[sc.value], reach=rc.value, quality=q.value,
                qualities=[float(v) for v in qs[:nev.value]] if all_qualities else None)


def hotspot(temp, power, params, dy: int = 0, dx: int = 0, iterations: int = 1) -> np.ndarray:
    """HotSpot steps (Table 1; S25).  params = dict(c, gx, gy,
    gz, tamb); per-axis reaches (dy, dx) substitute the 3x3 tile of T."""
    t, squeeze = _frames(temp)
    p, _ = _frames(power)
    if t.shape != p.shape:
        raise ValueError("temp and power shapes differ")
    n, h, w = t.shape
    out = np.empty(t.shape, dtype=np.float64)
    _ok(lib().oracle_hotspot(_fp(t), _fp(p), n, h, w, float(params["c"]), float(params["gx"]), float(params["gy"]),
                             float(params["gz"]), float(params["tamb"]), int(dy), int(dx), int(iterations), _dp(out)),
        "hotspot")
    return out[0] if squeeze else out


def runtime_ladder(train_q, toq: float):
    """R1-R2 (oracle.h): candidate indices of the ladder's rungs, -1 = EXACT."""
    q = np.ascontiguousarray(train_q, dtype=np.float64)
    cap = q.size + 1
    r = np.zeros(cap, dtype=np.int32)
    n = lib().oracle_runtime_ladder(q.size, _dp(q), float(toq), cap, r.ctypes.data_as(C.POINTER(C.c_int)))
    _ok(0 if n > 0 else -1, "runtime_ladder")
    return [int(v) for v in r[:n]]


def runtime_trace(q, check_every: int, toq: float):
    """R3-R4 (oracle.h): q[t][k] = quality a check of invocation t measures on
    rung k.  Returns dict(rungs=[rung used per invocation], checked=[0/1],
    checks, backoffs)."""
    q = np.ascontiguousarray(q, dtype=np.float64)
    t_count, rungs = q.shape
    used = np.zeros(max(1, t_count), dtype=np.int32)
    chk = np.zeros(max(1, t_count), dtype=np.int32)
    nc, nb = C.c_longlong(), C.c_longlong()
    _ok(lib().oracle_runtime_trace(rungs, int(check_every), float(toq), t_count, _dp(q),
                                   used.ctypes.data_as(C.POINTER(C.c_int)), chk.ctypes.data_as(C.POINTER(C.c_int)),
                                   C.byref(nc), C.byref(nb)), "runtime_trace")
    return dict(rungs=[int(v) for v in used[:t_count]], checked=[int(v) for v in chk[:t_count]],
                checks=nc.value, backoffs=nb.value)


def runtime_simulate(train, frames, w, toq: float, metric="mre", check_every: int = 1):
    """The whole runtime loop on the oracle's own stencils: ladder from the
    oracle tuner's training qualities, then each invocation's check quality
    = quality(exact, approx of the rung) on that frame, both rounded to fp32
    (what the user gets), and the back-off trace.  `w` dense 2-D or (wy, wx).
    Returns dict(ladder=[(scheme, reach, train_q)], trace=..., q=[[...]])."""
    sep = isinstance(w, (tuple, list))
    ky, kx = (np.asarray(w[0]).size, np.asarray(w[1]).size) if sep else np.asarray(w).shape
    cands = tune_candidates(ky, kx, sep)
    tq = tune(train, w, 2.0, metric, all_qualities=True)["qualities"]
    idx = runtime_ladder(tq, toq)
    ladder = [(cands[k][0], cands[k][1], tq[k]) if k >= 0 else ("exact", 0, 1.0) for k in idx]
    frames, _ = _frames(frames)
    q = np.ones((frames.shape[0], len(ladder)))
    for t in range(frames.shape[0]):
        x = frames[t:t + 1]
        run = (lambda s, r: stencil_sep_scheme(x, w[0], w[1], s, r)) if sep else \
            (lambda s, r: stencil_approx(x, w, s, r))
        e = run("exact", 0).astype(np.float32)
        for k, (s, r, _) in enumerate(ladder[:-1]):
            q[t, k] = quality(e, run(s, r).astype(np.float32), metric)
    return dict(ladder=ladder, trace=runtime_trace(q, check_every, toq), q=q.tolist())
