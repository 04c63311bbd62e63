"""Thin Python binding over the libparaprox C ABI (include/paraprox.h).

Argument marshalling only: every step of the path runs in the library's
sm_100a kernels.  torch supplies device memory and the current CUDA stream.
The names follow the C entry points without the ``paraprox_`` prefix.

There is no CPU fallback: if ``libparaprox.so`` is missing this module raises
at import, and every stencil call requires CUDA tensors.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PARAPROX_LIB") or os.path.join(_HERE, "libparaprox.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'`")

_lib = C.CDLL(LIB_PATH)

OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_CUDA, ERR_ALLOC = range(5)
EXACT, ROW, COL, CENTER = 0, 1, 2, 3
SKIP_ROW, SKIP_COL, SKIP_BOTH = 4, 5, 6
MRE, L2, PSNR = 0, 1, 2
SCHEMES = {"exact": EXACT, "row": ROW, "col": COL, "column": COL, "center": CENTER, "centre": CENTER,
           "skip_row": SKIP_ROW, "skip_col": SKIP_COL, "skip_both": SKIP_BOTH}
SCHEME_NAMES = {EXACT: "exact", ROW: "row", COL: "col", CENTER: "center", SKIP_ROW: "skip_row",
                SKIP_COL: "skip_col", SKIP_BOTH: "skip_both"}
METRICS = {"mre": MRE, "l2": L2, "psnr": PSNR}
MAX_K = 17


class HotspotParams(C.Structure):
    _fields_ = [("step_div_cap", C.c_double), ("rx_inv", C.c_double), ("ry_inv", C.c_double),
                ("rz_inv", C.c_double), ("t_amb", C.c_double)]


class Image(C.Structure):
    _fields_ = [("n", C.c_int), ("h", C.c_int), ("w", C.c_int), ("pitch", C.c_longlong),
                ("frame_stride", C.c_longlong), ("halo_top", C.c_int), ("halo_bottom", C.c_int)]


_P = C.c_void_p
_I = C.POINTER(C.c_int)
_D = C.POINTER(C.c_double)
_F = C.POINTER(C.c_float)
_IMG = C.POINTER(Image)
_SIGS = {
    "paraprox_filter_create": [C.c_int, C.c_int, _F, C.POINTER(_P)],
    "paraprox_filter_create_separable": [C.c_int, _F, C.c_int, _F, C.POINTER(_P)],
    "paraprox_filter_shape": [_P, _I, _I, _I],
    "paraprox_plan_info": [_P, C.c_int, C.c_int, _I, _I, _I, _I, _I],
    "paraprox_stencil_exact": [_P, _P, _P, _IMG, _P],
    "paraprox_stencil_approx": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_stencil_approx_xy": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_run_host": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_stencil_lattice": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_stencil_skip_xy": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_hotspot": [C.POINTER(HotspotParams), C.c_int, C.c_int, _P, _P, _P, _IMG, C.c_int, _P],
    "paraprox_stencil_peer": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P, C.c_int, _P, C.c_int, C.c_longlong, _P],
    "paraprox_ipc_export": [_P, _P, C.POINTER(C.c_longlong)],
    "paraprox_hotspot_peer": [C.POINTER(HotspotParams), C.c_int, C.c_int, _P, _P, _P, _IMG, C.c_int, _P, _P, C.c_int,
                              _P, _P, C.c_int, C.c_longlong, _P],
    "paraprox_flag_wait": [_P, C.c_longlong, _P],
    "paraprox_flag_set": [_P, C.c_longlong, _P],
    "paraprox_ipc_open": [_P, C.POINTER(_P)],
    "paraprox_ipc_close": [_P],
    "paraprox_tune_ex": [_P, C.c_int, _P, _IMG, C.c_double, C.c_int, _I, _I, _D, _P],
    "paraprox_tune_candidates_ex": [_P, C.c_int, C.c_int, _I, _I, _I],
    "paraprox_tune_partials_ex": [_P, C.c_int, _P, _IMG, C.c_int, _D, _P],
    "paraprox_tune_decide_ex": [_P, C.c_int, _D, C.c_int, C.c_double, _I, _I, _D],
    "paraprox_stencil_lattice_xy": [_P, C.c_int, C.c_int, _P, _P, _IMG, _P],
    "paraprox_tune_lattice": [_P, _P, _IMG, C.c_double, C.c_int, _I, _I, _D, _P],
    "paraprox_tune_lattice_partials": [_P, _P, _IMG, C.c_int, _D, _P],
    "paraprox_tune_lattice_decide": [_D, C.c_int, C.c_double, _I, _I, _D],
    "paraprox_runtime_create": [_P, C.c_double, C.c_int, C.c_int, C.POINTER(_P)],
    "paraprox_runtime_train": [_P, _P, _IMG, _P],
    "paraprox_runtime_run": [_P, _P, _P, _IMG, _P],
    "paraprox_runtime_sync": [_P],
    "paraprox_runtime_state": [_P, _I, _I, C.POINTER(C.c_longlong), C.POINTER(C.c_longlong),
                               C.POINTER(C.c_longlong), _D],
    "paraprox_runtime_ladder": [_P, C.c_int, _I, _I, _I, _D],
    "paraprox_runtime_set_profiled": [_P, C.c_int],
    "paraprox_runtime_timings": [_P, C.c_int, _I, _D],
    "paraprox_quality": [_P, _P, _IMG, C.c_int, _D, _P],
    "paraprox_quality_partials": [_P, _P, _IMG, C.c_int, _D, _P],
    "paraprox_quality_partials_async": [_P, _P, _IMG, C.c_int, _P, _P],
    "paraprox_quality_from_partials": [_D, C.c_int, _D],
    "paraprox_tune": [_P, _P, _IMG, C.c_double, C.c_int, _I, _I, _D, _P],
    "paraprox_tune_candidates": [_P, C.c_int, _I, _I, _I],
    "paraprox_tune_partials": [_P, _P, _IMG, C.c_int, _D, _P],
    "paraprox_tune_decide": [_P, _D, C.c_int, C.c_double, _I, _I, _D],
}
for _name, _args in _SIGS.items():
    getattr(_lib, _name).argtypes = _args
    getattr(_lib, _name).restype = C.c_int
_lib.paraprox_filter_destroy.argtypes = [_P]
_lib.paraprox_filter_destroy.restype = None
_lib.paraprox_runtime_destroy.argtypes = [_P]
_lib.paraprox_runtime_destroy.restype = None
_lib.paraprox_status_string.argtypes = [C.c_int]
_lib.paraprox_status_string.restype = C.c_char_p
_lib.paraprox_last_error.restype = C.c_char_p
_lib.paraprox_last_kernel.restype = C.c_char_p
_lib.paraprox_version.restype = C.c_int
_lib.paraprox_launch_count.restype = C.c_ulonglong

ABI_SYMBOLS = sorted(list(_SIGS) + ["paraprox_filter_destroy", "paraprox_runtime_destroy", "paraprox_status_string", "paraprox_last_error",
                                    "paraprox_last_kernel", "paraprox_version", "paraprox_launch_count"])


class ParaproxError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        detail = _lib.paraprox_last_error().decode()
        super().__init__(f"{what}: {_lib.paraprox_status_string(status).decode()} ({detail})")


def _check(rc: int, what: str):
    if rc != OK:
        raise ParaproxError(rc, what)


def version() -> int:
    return _lib.paraprox_version()


def launch_count() -> int:
    return int(_lib.paraprox_launch_count())


def last_kernel() -> str:
    return _lib.paraprox_last_kernel().decode()


def _scheme(s) -> int:
    if isinstance(s, str):
        return SCHEMES[s.lower()]
    return int(s)


def _metric(m) -> int:
    if isinstance(m, str):
        return METRICS[m.lower()]
    return int(m)


class Filter:
    """A filter handle (paraprox_filter_create / _separable)."""

    def __init__(self, w=None, *, wy=None, wx=None):
        h = _P()
        if w is not None:
            a = np.ascontiguousarray(np.asarray(w, dtype=np.float32))
            if a.ndim == 1:
                a = a[None]
            if a.ndim != 2:
                raise ValueError("dense weights must be 2-D")
            _check(_lib.paraprox_filter_create(a.shape[0], a.shape[1], a.ctypes.data_as(_F), C.byref(h)),
                   "filter_create")
            self.ky, self.kx, self.separable = a.shape[0], a.shape[1], False
        else:
            ay = np.ascontiguousarray(np.asarray(wy, dtype=np.float32).ravel())
            ax = np.ascontiguousarray(np.asarray(wx, dtype=np.float32).ravel())
            _check(_lib.paraprox_filter_create_separable(ay.size, ay.ctypes.data_as(_F), ax.size,
                                                         ax.ctypes.data_as(_F), C.byref(h)),
                   "filter_create_separable")
            self.ky, self.kx, self.separable = ay.size, ax.size, True
        self._h = h

    @classmethod
    def separable_(cls, wy, wx):
        return cls(wy=wy, wx=wx)

    @property
    def handle(self):
        return self._h

    def close(self):
        if self._h:
            _lib.paraprox_filter_destroy(self._h)
            self._h = _P()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def plan_info(self, reach_y: int, reach_x: int):
        taps, hy, hx = C.c_int(), C.c_int(), C.c_int()
        my = (C.c_int * self.ky)()
        mx = (C.c_int * self.kx)()
        _check(_lib.paraprox_plan_info(self._h, reach_y, reach_x, C.byref(taps), C.byref(hy), C.byref(hx),
                                       my, mx), "plan_info")
        return dict(taps=taps.value, halo_y=hy.value, halo_x=hx.value, map_y=list(my), map_x=list(mx))


def filter_create(w) -> Filter:
    return Filter(w)


def filter_create_separable(wy, wx) -> Filter:
    return Filter(wy=wy, wx=wx)


def _stream(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


def image_of(x: torch.Tensor, halo_top: int = 0, halo_bottom: int = 0) -> Image:
    """Descriptor of a [h, w] or [n, h_total, w] fp32 tensor with unit column
    stride; h = h_total - halo_top - halo_bottom."""
    if x.dtype != torch.float32:
        raise TypeError("paraprox images are fp32")
    if x.dim() == 2:
        n, ht, w = 1, x.shape[0], x.shape[1]
        pitch, fs = x.stride(0), x.shape[0] * x.stride(0)
    elif x.dim() == 3:
        n, ht, w = x.shape
        pitch, fs = x.stride(1), x.stride(0)
    else:
        raise ValueError("expected [h, w] or [n, h, w]")
    if w > 1 and x.stride(-1) != 1:
        raise ValueError("rows must be contiguous (unit column stride)")
    if n > 1 and fs < ht * pitch:
        raise ValueError("frames overlap")
    return Image(n, ht - halo_top - halo_bottom, w, pitch, fs if n > 1 else ht * pitch, halo_top, halo_bottom)


def _need_cuda(*ts):
    for t in ts:
        if not (isinstance(t, torch.Tensor) and t.is_cuda):
            raise TypeError("paraprox device entry points take CUDA tensors (there is no CPU path)")


def _out_like(x: torch.Tensor, halo_top: int, halo_bottom: int, out):
    if out is not None:
        return out
    if x.dim() == 2:
        return torch.empty((x.shape[0] - halo_top - halo_bottom, x.shape[1]), dtype=x.dtype, device=x.device)
    if halo_top or halo_bottom:
        # same pitch and frame stride as the input (the ABI shares the layout)
        buf = torch.empty_like(x)
        return buf[:, halo_top:x.shape[1] - halo_bottom]
    return torch.empty_like(x)


def _dp(t, halo_top=0):
    return C.c_void_p(t.data_ptr() + 4 * halo_top * (t.stride(-2) if t.dim() >= 2 else 0))


def _check_out(out, img):
    if out.dim() == 2:
        ok = img.n == 1 and out.shape[0] == img.h and out.shape[1] == img.w and out.stride(0) == img.pitch
    else:
        ok = (tuple(out.shape) == (img.n, img.h, img.w) and out.stride(1) == img.pitch
              and (img.n == 1 or out.stride(0) == img.frame_stride))
    if not ok or out.dtype != torch.float32 or (img.w > 1 and out.stride(-1) != 1):
        raise ValueError("out must match the input's shape, pitch and frame stride")


def stencil_exact(x, f: Filter, out=None, *, halo_top=0, halo_bottom=0, stream=None):
    _need_cuda(x)
    img = image_of(x, halo_top, halo_bottom)
    out = _out_like(x, halo_top, halo_bottom, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_exact(f.handle, _dp(x, halo_top), _dp(out), C.byref(img), _stream(stream)),
           "stencil_exact")
    return out


def stencil_approx(x, f: Filter, scheme, reach: int, out=None, *, halo_top=0, halo_bottom=0, stream=None):
    _need_cuda(x)
    img = image_of(x, halo_top, halo_bottom)
    out = _out_like(x, halo_top, halo_bottom, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_approx(f.handle, _scheme(scheme), int(reach), _dp(x, halo_top), _dp(out),
                                        C.byref(img), _stream(stream)), "stencil_approx")
    return out


def stencil_approx_xy(x, f: Filter, reach_y: int, reach_x: int, out=None, *, halo_top=0, halo_bottom=0,
                      stream=None):
    _need_cuda(x)
    img = image_of(x, halo_top, halo_bottom)
    out = _out_like(x, halo_top, halo_bottom, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_approx_xy(f.handle, int(reach_y), int(reach_x), _dp(x, halo_top), _dp(out),
                                           C.byref(img), _stream(stream)), "stencil_approx_xy")
    return out


def stencil_lattice(x, f: Filter, scheme, reach: int, out=None, *, stream=None):
    """Global-lattice reading: the exact stencil on the
    array rebuilt from every (2*reach+1)-th row / column / both."""
    _need_cuda(x)
    img = image_of(x)
    out = _out_like(x, 0, 0, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_lattice(f.handle, _scheme(scheme), int(reach), _dp(x), _dp(out), C.byref(img),
                                         _stream(stream)), "stencil_lattice")
    return out


def stencil_lattice_xy(x, f: Filter, reach_y: int, reach_x: int, out=None, *, stream=None):
    _need_cuda(x)
    img = image_of(x)
    out = _out_like(x, 0, 0, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_lattice_xy(f.handle, int(reach_y), int(reach_x), _dp(x), _dp(out), C.byref(img),
                                            _stream(stream)), "stencil_lattice_xy")
    return out


def stencil_skip_xy(x, f: Filter, skip_y: int, skip_x: int, out=None, *, halo_top=0, halo_bottom=0, stream=None):
    """Reduction approximation of the filter loops: every
    skip_y-th filter row / skip_x-th filter column, scaled by the rates."""
    _need_cuda(x)
    img = image_of(x, halo_top, halo_bottom)
    out = _out_like(x, halo_top, halo_bottom, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_skip_xy(f.handle, int(skip_y), int(skip_x), _dp(x, halo_top), _dp(out),
                                         C.byref(img), _stream(stream)), "stencil_skip_xy")
    return out


class Prepared:
    """A stencil call with its arguments marshalled once (for tight loops and
    graph capture): calling it re-issues paraprox_stencil_approx on the
    stream given at preparation time."""

    def __init__(self, x, f: Filter, scheme, reach: int, out, *, halo_top=0, halo_bottom=0, stream=None,
                 lattice=False):
        _need_cuda(x, out)
        self._img = image_of(x, halo_top, halo_bottom)
        _check_out(out, self._img)
        self._keep = (x, out, f)
        self._args = (f.handle, _scheme(scheme), int(reach), _dp(x, halo_top), _dp(out), C.byref(self._img),
                      _stream(stream))
        self._fn = _lib.paraprox_stencil_lattice if lattice else _lib.paraprox_stencil_approx

    def __call__(self):
        rc = self._fn(*self._args)
        if rc != OK:
            raise ParaproxError(rc, "stencil_approx")


def prepare(x, f: Filter, scheme, reach: int, out, **kw) -> Prepared:
    return Prepared(x, f, scheme, reach, out, **kw)


def run_host(x: torch.Tensor, f: Filter, scheme, reach: int, out=None, *, stream=None):
    """End-to-end over host (ideally pinned) tensors: H2D, kernel, D2H inside
    the library, overlapped chunk by chunk.  Returns the host output."""
    if x.is_cuda:
        raise TypeError("run_host takes host tensors")
    img = image_of(x)
    if out is None:
        out = torch.empty_like(x, pin_memory=x.is_pinned())
    _check_out(out, img)
    _check(_lib.paraprox_run_host(f.handle, _scheme(scheme), int(reach), _dp(x), _dp(out), C.byref(img),
                                  _stream(stream)), "run_host")
    return out


def quality(exact, approx, metric="mre", *, stream=None) -> float:
    _need_cuda(exact, approx)
    img = image_of(exact)
    if exact.shape != approx.shape or exact.stride() != approx.stride():
        raise ValueError("exact and approx must share shape and strides")
    q = C.c_double()
    _check(_lib.paraprox_quality(_dp(exact), _dp(approx), C.byref(img), _metric(metric), C.byref(q),
                                 _stream(stream)), "quality")
    return q.value


def quality_partials(exact, approx, metric="mre", *, stream=None) -> np.ndarray:
    _need_cuda(exact, approx)
    img = image_of(exact)
    if exact.shape != approx.shape or exact.stride() != approx.stride():
        raise ValueError("exact and approx must share shape and strides")
    p = np.zeros(3, dtype=np.float64)
    _check(_lib.paraprox_quality_partials(_dp(exact), _dp(approx), C.byref(img), _metric(metric),
                                          p.ctypes.data_as(_D), _stream(stream)), "quality_partials")
    return p


def quality_partials_async(exact, approx, metric="mre", out=None, *, stream=None) -> torch.Tensor:
    """The 3 fp64 partials into a device tensor, stream-ordered, no sync."""
    _need_cuda(exact, approx)
    img = image_of(exact)
    if exact.shape != approx.shape or exact.stride() != approx.stride():
        raise ValueError("exact and approx must share shape and strides")
    if out is None:
        out = torch.empty(3, dtype=torch.float64, device=exact.device)
    if out.dtype != torch.float64 or out.numel() < 3 or not out.is_contiguous():
        raise ValueError("out must be a contiguous float64 device tensor of >= 3 elements")
    _need_cuda(out)
    _check(_lib.paraprox_quality_partials_async(_dp(exact), _dp(approx), C.byref(img), _metric(metric),
                                                C.c_void_p(out.data_ptr()), _stream(stream)), "quality_partials_async")
    return out


def quality_from_partials(p, metric="mre") -> float:
    p = np.ascontiguousarray(p, dtype=np.float64)
    q = C.c_double()
    _check(_lib.paraprox_quality_from_partials(p.ctypes.data_as(_D), _metric(metric), C.byref(q)),
           "quality_from_partials")
    return q.value


def tune_candidates(f: Filter):
    n = C.c_int()
    _check(_lib.paraprox_tune_candidates(f.handle, 0, C.byref(n), None, None), "tune_candidates")
    s = (C.c_int * max(1, n.value))()
    r = (C.c_int * max(1, n.value))()
    _check(_lib.paraprox_tune_candidates(f.handle, n.value, C.byref(n), s, r), "tune_candidates")
    return [(SCHEME_NAMES[s[i]], r[i]) for i in range(n.value)]


def tune(frames, f: Filter, toq: float, metric="mre", *, stream=None):
    """Returns (scheme name, reach, quality)."""
    _need_cuda(frames)
    img = image_of(frames)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune(f.handle, _dp(frames), C.byref(img), float(toq), _metric(metric), C.byref(sc),
                              C.byref(rc), C.byref(q), _stream(stream)), "tune")
    return SCHEME_NAMES[sc.value], rc.value, q.value


def tune_partials(frames, f: Filter, metric="mre", *, stream=None) -> np.ndarray:
    _need_cuda(frames)
    img = image_of(frames)
    n = len(tune_candidates(f))
    p = np.zeros(3 * max(n, 1), dtype=np.float64)
    _check(_lib.paraprox_tune_partials(f.handle, _dp(frames), C.byref(img), _metric(metric),
                                       p.ctypes.data_as(_D), _stream(stream)), "tune_partials")
    return p[:3 * n]


def tune_decide(f: Filter, partials, toq: float, metric="mre"):
    p = np.ascontiguousarray(partials, dtype=np.float64)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune_decide(f.handle, p.ctypes.data_as(_D) if p.size else None, _metric(metric),
                                     float(toq), C.byref(sc), C.byref(rc), C.byref(q)), "tune_decide")
    return SCHEME_NAMES[sc.value], rc.value, q.value


def tune_lattice(frames, f: Filter, toq: float, metric="mre", *, stream=None):
    """Lattice tuner: returns (scheme name, reach, quality)."""
    _need_cuda(frames)
    img = image_of(frames)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune_lattice(f.handle, _dp(frames), C.byref(img), float(toq), _metric(metric),
                                      C.byref(sc), C.byref(rc), C.byref(q), _stream(stream)), "tune_lattice")
    return SCHEME_NAMES[sc.value], rc.value, q.value


def tune_lattice_partials(frames, f: Filter, metric="mre", *, stream=None) -> np.ndarray:
    _need_cuda(frames)
    img = image_of(frames)
    p = np.zeros(12, dtype=np.float64)
    _check(_lib.paraprox_tune_lattice_partials(f.handle, _dp(frames), C.byref(img), _metric(metric),
                                               p.ctypes.data_as(_D), _stream(stream)), "tune_lattice_partials")
    return p


def tune_lattice_decide(partials, toq: float, metric="mre"):
    p = np.ascontiguousarray(partials, dtype=np.float64)
    if p.size != 12:
        raise ValueError("12 partials expected")
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune_lattice_decide(p.ctypes.data_as(_D), _metric(metric), float(toq), C.byref(sc),
                                             C.byref(rc), C.byref(q)), "tune_lattice_decide")
    return SCHEME_NAMES[sc.value], rc.value, q.value


class Runtime:
    """The runtime loop (paraprox_runtime_*): train once, then run the current
    rung; every ``check_every``-th invocation is checked against the exact
    stencil on the device and a quality below ``toq`` moves one rung down the
    ladder."""

    def __init__(self, f: Filter, toq: float, metric="mre", check_every: int = 40, profiled: bool = False):
        self._f = f
        h = _P()
        _check(_lib.paraprox_runtime_create(f.handle, float(toq), _metric(metric), int(check_every), C.byref(h)),
               "runtime_create")
        self._h = h
        if profiled:
            _check(_lib.paraprox_runtime_set_profiled(h, 1), "runtime_set_profiled")

    def timings(self):
        """Measured ms per candidate (tuner order), then exact; NaN = not timed."""
        n = C.c_int()
        _check(_lib.paraprox_runtime_timings(self._h, 0, C.byref(n), None), "runtime_timings")
        ms = (C.c_double * max(1, n.value))()
        _check(_lib.paraprox_runtime_timings(self._h, n.value, C.byref(n), ms), "runtime_timings")
        return [ms[i] for i in range(n.value)]

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            _lib.paraprox_runtime_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def train(self, frames, *, stream=None):
        _need_cuda(frames)
        img = image_of(frames)
        _check(_lib.paraprox_runtime_train(self._h, _dp(frames), C.byref(img), _stream(stream)), "runtime_train")
        return self.state()

    def run(self, x, out=None, *, halo_top=0, halo_bottom=0, stream=None):
        _need_cuda(x)
        img = image_of(x, halo_top, halo_bottom)
        out = _out_like(x, halo_top, halo_bottom, out)
        _need_cuda(out)
        _check_out(out, img)
        _check(_lib.paraprox_runtime_run(self._h, _dp(x, halo_top), _dp(out), C.byref(img), _stream(stream)),
               "runtime_run")
        return out

    def sync(self):
        _check(_lib.paraprox_runtime_sync(self._h), "runtime_sync")

    def state(self):
        sc, r = C.c_int(), C.c_int()
        inv, chk, bo = C.c_longlong(), C.c_longlong(), C.c_longlong()
        q = C.c_double()
        _check(_lib.paraprox_runtime_state(self._h, C.byref(sc), C.byref(r), C.byref(inv), C.byref(chk),
                                           C.byref(bo), C.byref(q)), "runtime_state")
        return dict(scheme=SCHEME_NAMES[sc.value], reach=r.value, invocations=inv.value, checks=chk.value,
                    backoffs=bo.value, last_quality=q.value)

    def ladder(self):
        n = C.c_int()
        _check(_lib.paraprox_runtime_ladder(self._h, 0, C.byref(n), None, None, None), "runtime_ladder")
        k = max(1, n.value)
        s, r, q = (C.c_int * k)(), (C.c_int * k)(), (C.c_double * k)()
        _check(_lib.paraprox_runtime_ladder(self._h, k, C.byref(n), s, r, q), "runtime_ladder")
        return [(SCHEME_NAMES[s[i]], r[i], q[i]) for i in range(n.value)]


STENCIL, REDUCTION = 1, 2  # tune_ex flags


def tune_candidates_ex(f: Filter, flags: int = 3):
    n = C.c_int()
    _check(_lib.paraprox_tune_candidates_ex(f.handle, int(flags), 0, C.byref(n), None, None), "tune_candidates_ex")
    s = (C.c_int * max(1, n.value))()
    r = (C.c_int * max(1, n.value))()
    _check(_lib.paraprox_tune_candidates_ex(f.handle, int(flags), n.value, C.byref(n), s, r), "tune_candidates_ex")
    return [(SCHEME_NAMES[s[i]], r[i]) for i in range(n.value)]


def tune_ex(frames, f: Filter, toq: float, metric="mre", flags: int = 3, *, stream=None):
    """Extended tuner over stencil (flags & 1) and reduction (flags & 2)
    schemes.  Returns (scheme name, reach or skipping rate, quality)."""
    _need_cuda(frames)
    img = image_of(frames)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune_ex(f.handle, int(flags), _dp(frames), C.byref(img), float(toq), _metric(metric),
                                 C.byref(sc), C.byref(rc), C.byref(q), _stream(stream)), "tune_ex")
    return SCHEME_NAMES[sc.value], rc.value, q.value


def tune_partials_ex(frames, f: Filter, metric="mre", flags: int = 3, *, stream=None) -> np.ndarray:
    _need_cuda(frames)
    img = image_of(frames)
    n = len(tune_candidates_ex(f, flags))
    p = np.zeros(3 * max(n, 1), dtype=np.float64)
    _check(_lib.paraprox_tune_partials_ex(f.handle, int(flags), _dp(frames), C.byref(img), _metric(metric),
                                          p.ctypes.data_as(_D), _stream(stream)), "tune_partials_ex")
    return p[:3 * n]


def tune_decide_ex(f: Filter, partials, toq: float, metric="mre", flags: int = 3):
    p = np.ascontiguousarray(partials, dtype=np.float64)
    sc, rc, q = C.c_int(), C.c_int(), C.c_double()
    _check(_lib.paraprox_tune_decide_ex(f.handle, int(flags), p.ctypes.data_as(_D) if p.size else None,
                                        _metric(metric), float(toq), C.byref(sc), C.byref(rc), C.byref(q)),
           "tune_decide_ex")
    return SCHEME_NAMES[sc.value], rc.value, q.value


def hotspot(temp, power, params, scheme="exact", reach: int = 0, iterations: int = 1, out=None, *, halo_top=0,
            halo_bottom=0, stream=None):
    """HotSpot steps (paraprox_hotspot).  params: dict(c, gx, gy, gz, tamb)."""
    _need_cuda(temp, power)
    img = image_of(temp, halo_top, halo_bottom)
    out = _out_like(temp, halo_top, halo_bottom, out)
    _need_cuda(out)
    _check_out(out, img)
    _check_out(power, img)
    prm = HotspotParams(float(params["c"]), float(params["gx"]), float(params["gy"]), float(params["gz"]),
                        float(params["tamb"]))
    _check(_lib.paraprox_hotspot(C.byref(prm), _scheme(scheme), int(reach), _dp(temp, halo_top), _dp(power), _dp(out),
                                 C.byref(img), int(iterations), _stream(stream)), "hotspot")
    return out


def stencil_peer(x, f: Filter, scheme, reach: int, out=None, *, top=None, top_rows: int = 0, bot=None,
                 bot_rows: int = 0, src_pitch: int = 0, stream=None):
    """A row stripe whose halo rows are read inside the kernel from device
    pointers (ints) `top` (the top_rows rows right above row 0) and `bot`
    (the bot_rows rows right below the last row), e.g. CUDA-IPC mappings of
    the neighbours' stripes (dist.PeerStripe)."""
    _need_cuda(x)
    img = image_of(x)
    out = _out_like(x, 0, 0, out)
    _need_cuda(out)
    _check_out(out, img)
    _check(_lib.paraprox_stencil_peer(f.handle, _scheme(scheme), int(reach), _dp(x), _dp(out), C.byref(img),
                                      C.c_void_p(top or 0), int(top_rows), C.c_void_p(bot or 0), int(bot_rows),
                                      int(src_pitch), _stream(stream)), "stencil_peer")
    return out


def ipc_export(t: torch.Tensor):
    """(64-byte handle, byte offset) of the CUDA allocation holding t."""
    _need_cuda(t)
    h = (C.c_char * 64)()
    off = C.c_longlong()
    _check(_lib.paraprox_ipc_export(C.c_void_p(t.data_ptr()), h, C.byref(off)), "ipc_export")
    return bytes(h), off.value


def ipc_open(handle: bytes) -> int:
    buf = (C.c_char * 64).from_buffer_copy(handle)
    p = _P()
    _check(_lib.paraprox_ipc_open(buf, C.byref(p)), "ipc_open")
    return p.value


def ipc_close(base: int):
    _check(_lib.paraprox_ipc_close(C.c_void_p(base)), "ipc_close")


def hotspot_peer(temp, power, params, scheme, reach: int, steps: int, out, *, top_t=None, top_p=None,
                 top_rows: int = 0, bot_t=None, bot_p=None, bot_rows: int = 0, src_pitch: int = 0, stream=None):
    """One HotSpot pass (<= 8 steps) of a row stripe reading its neighbours'
    rows (device pointers as ints) inside the blocked kernel."""
    _need_cuda(temp, power, out)
    img = image_of(temp)
    _check_out(out, img)
    _check_out(power, img)
    prm = HotspotParams(float(params["c"]), float(params["gx"]), float(params["gy"]), float(params["gz"]),
                        float(params["tamb"]))
    _check(_lib.paraprox_hotspot_peer(C.byref(prm), _scheme(scheme), int(reach), _dp(temp), _dp(power), _dp(out),
                                      C.byref(img), int(steps), C.c_void_p(top_t or 0), C.c_void_p(top_p or 0),
                                      int(top_rows), C.c_void_p(bot_t or 0), C.c_void_p(bot_p or 0), int(bot_rows),
                                      int(src_pitch), _stream(stream)), "hotspot_peer")
    return out


def flag_wait(flag_ptr: int, target: int, *, stream=None):
    _check(_lib.paraprox_flag_wait(C.c_void_p(flag_ptr), int(target), _stream(stream)), "flag_wait")


def flag_set(flag_ptr: int, value: int, *, stream=None):
    _check(_lib.paraprox_flag_set(C.c_void_p(flag_ptr), int(value), _stream(stream)), "flag_set")
