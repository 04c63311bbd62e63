"""Host-side checks of the C ABI (no GPU needed): the library loads, exports
every symbol include/paraprox.h declares, validates its arguments, and its
host logic (index maps, folded-plan sizes, candidate order, decision,
quality from partials) agrees with the independently written oracle."""
import ctypes as C
import math
import os
import re

import numpy as np
import pytest

from workloads import filters as F

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def P():
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "paraprox.h")).read()
    return sorted(set(re.findall(r"PARAPROX_API[^;]*?\b(paraprox_\w+)\s*\(", src, flags=re.S)))


def test_exports_every_declared_symbol(P):
    decl = declared_symbols()
    assert len(decl) >= 20
    for name in decl:
        assert hasattr(P._lib, name), name
    assert sorted(P.ABI_SYMBOLS) == decl
    assert P.version() == 1


def test_no_torch_in_header():
    src = open(os.path.join(ROOT, "include", "paraprox.h")).read()
    assert "torch" not in src.lower().replace("torch types", "")
    assert "#include" not in src


def test_library_is_sm100a():
    import subprocess
    lib = os.path.join(ROOT, "paper_conf_asplos_samadijlm14_b200", "libparaprox.so")
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_filter_create_errors(P):
    with pytest.raises(P.ParaproxError) as e:
        P.Filter(np.ones((2, 3), np.float32))
    assert e.value.status == P.ERR_INVALID_ARG
    with pytest.raises(P.ParaproxError) as e:
        P.Filter(np.ones((19, 19), np.float32))
    assert e.value.status == P.ERR_UNSUPPORTED
    h = C.c_void_p()
    assert P._lib.paraprox_filter_create(3, 3, None, C.byref(h)) == P.ERR_INVALID_ARG
    f = P.Filter(F.gaussian(3))
    ky, kx, sep = C.c_int(), C.c_int(), C.c_int()
    assert P._lib.paraprox_filter_shape(f.handle, C.byref(ky), C.byref(kx), C.byref(sep)) == 0
    assert (ky.value, kx.value, sep.value) == (3, 3, 0)


@pytest.mark.parametrize("k", [1, 3, 5, 7, 9, 11, 17])
def test_plan_maps_match_oracle(P, O, k):
    f = P.Filter(np.ones((k, k), np.float32) / (k * k))
    r = k // 2
    for dy in range(0, r + 3):
        for dx in (0, min(dy, r), r + 1):
            info = f.plan_info(dy, dx)
            assert info["map_y"] == list(O.index_map(r, dy))
            assert info["map_x"] == list(O.index_map(r, dx))
            ry = set(info["map_y"])
            rx = set(info["map_x"])
            assert info["taps"] == len(ry) * len(rx)
            assert info["halo_y"] == max(abs(a) for a in ry)
            assert info["halo_x"] == max(abs(b) for b in rx)


def test_plan_separable_taps(P):
    wy, wx = F.separable(7)
    f = P.Filter(wy=wy, wx=wx)
    assert f.plan_info(0, 0)["taps"] == 14
    assert f.plan_info(3, 3)["taps"] == 2
    assert f.plan_info(1, 0)["taps"] == 3 + 7


@pytest.mark.parametrize("ky,kx", [(1, 1), (1, 5), (3, 3), (5, 5), (3, 7), (7, 7), (9, 9), (9, 3), (17, 17),
                                   (1, 17), (17, 1), (13, 5)])
@pytest.mark.parametrize("sep", [False, True])
def test_candidates_match_oracle(P, O, ky, kx, sep):
    if sep:
        f = P.Filter(wy=np.ones(ky, np.float32), wx=np.ones(kx, np.float32))
    else:
        f = P.Filter(np.ones((ky, kx), np.float32))
    assert P.tune_candidates(f) == O.tune_candidates(ky, kx, sep)


def test_decide_first_passing(P):
    f = P.Filter(F.mean(5))
    cands = P.tune_candidates(f)
    assert len(cands) == 6
    # MRE partials: (sum of relative errors, count, 0); qualities .80 .85 .93 .95 .97 .99
    errs = [0.20, 0.15, 0.07, 0.05, 0.03, 0.01]
    parts = np.array([[e * 1000.0, 1000.0, 0.0] for e in errs]).ravel()
    assert P.tune_decide(f, parts, 0.90, "mre")[:2] == cands[2]
    assert P.tune_decide(f, parts, 0.95, "mre")[:2] == cands[3]
    assert P.tune_decide(f, parts, 0.80, "mre")[:2] == cands[0]
    s, r, q = P.tune_decide(f, parts, 0.995, "mre")
    assert (s, r, q) == ("exact", 0, 1.0)
    q = P.tune_decide(f, parts, 0.92, "mre")[2]
    assert q == pytest.approx(0.93, abs=1e-15)
    for bad in (0.0, 1.5, float("nan")):
        with pytest.raises(P.ParaproxError):
            P.tune_decide(f, parts, bad, "mre")


def test_quality_from_partials(P):
    assert P.quality_from_partials([5.0, 100.0, 0.0], "mre") == pytest.approx(0.95)
    assert P.quality_from_partials([1.0, 100.0, 10.0], "l2") == pytest.approx(0.9)
    assert P.quality_from_partials([0.0, 0.0, 10.0], "l2") == 1.0
    assert P.quality_from_partials([40.0, 10.0, 0.0], "psnr") == pytest.approx(20 * math.log10(255 / 2))
    assert P.quality_from_partials([0.0, 10.0, 0.0], "psnr") == math.inf


def _img(P, n=1, h=8, w=8, pitch=8, fs=64, ht=0, hb=0):
    return P.Image(n, h, w, pitch, fs, ht, hb)


def test_stencil_argument_validation(P):
    """Every rejected argument returns INVALID_ARG before any CUDA call."""
    f = P.Filter(F.gaussian(3))
    lib = P._lib
    a, b = C.c_void_p(0x10000), C.c_void_p(0x90000)
    s = C.c_void_p(0)
    good = _img(P)
    assert lib.paraprox_stencil_exact(None, a, b, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_exact(f.handle, None, b, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_exact(f.handle, a, None, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_exact(f.handle, a, b, None, s) == P.ERR_INVALID_ARG
    for bad in (_img(P, n=0), _img(P, h=0), _img(P, w=0), _img(P, pitch=7), _img(P, n=2, fs=63),
                _img(P, ht=-1), _img(P, n=2, fs=64, ht=1)):
        assert lib.paraprox_stencil_exact(f.handle, a, b, C.byref(bad), s) == P.ERR_INVALID_ARG
    # in-place / overlapping output
    assert lib.paraprox_stencil_exact(f.handle, a, a, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_exact(f.handle, a, C.c_void_p(0x10000 + 4 * 60), C.byref(good), s) == \
        P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_approx(f.handle, 7, 1, a, b, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_approx(f.handle, P.ROW, -1, a, b, C.byref(good), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_stencil_approx_xy(f.handle, 1, -2, a, b, C.byref(good), s) == P.ERR_INVALID_ARG
    q = C.c_double()
    assert lib.paraprox_quality(a, b, C.byref(good), 9, C.byref(q), s) == P.ERR_INVALID_ARG
    assert lib.paraprox_quality(a, b, C.byref(good), P.MRE, None, s) == P.ERR_INVALID_ARG
    sc, rc = C.c_int(), C.c_int()
    assert lib.paraprox_tune(f.handle, a, C.byref(good), 1.5, P.MRE, C.byref(sc), C.byref(rc), C.byref(q), s) == \
        P.ERR_INVALID_ARG
    assert lib.paraprox_run_host(f.handle, P.ROW, 1, a, a, C.byref(good), s) == P.ERR_INVALID_ARG
    assert "overlap" in lib.paraprox_last_error().decode()


def test_status_strings(P):
    for st in range(5):
        assert P._lib.paraprox_status_string(st)


def test_device_calls_refuse_cpu_tensors(P):
    import torch
    f = P.Filter(F.gaussian(3))
    with pytest.raises(TypeError):
        P.stencil_exact(torch.zeros(8, 8), f)


def test_runtime_argument_errors(P):
    import ctypes as C
    from workloads import filters as F
    f = P.Filter(F.mean(5))
    h = C.c_void_p()
    assert P._lib.paraprox_runtime_create(f.handle, 1.5, P.MRE, 40, C.byref(h)) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_runtime_create(f.handle, 0.9, P.MRE, -1, C.byref(h)) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_runtime_create(None, 0.9, P.MRE, 40, C.byref(h)) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_runtime_create(f.handle, 0.9, P.MRE, 40, C.byref(h)) == P.OK
    img = P.Image(1, 8, 8, 8, 64, 0, 0)
    # untrained: refused before any device work
    assert P._lib.paraprox_runtime_run(h, None, None, C.byref(img), None) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_runtime_state(h, None, None, None, None, None, None) == P.ERR_INVALID_ARG
    n = C.c_int()
    assert P._lib.paraprox_runtime_ladder(h, 0, C.byref(n), None, None, None) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_runtime_sync(h) == P.OK
    P._lib.paraprox_runtime_destroy(h)
    P._lib.paraprox_runtime_destroy(None)


@pytest.mark.parametrize("ky,kx", [(1, 1), (1, 5), (3, 3), (5, 5), (3, 7), (9, 9), (9, 1), (17, 17), (15, 3)])
@pytest.mark.parametrize("sep", [False, True])
@pytest.mark.parametrize("flags", [1, 2, 3])
def test_candidates_ex_match_oracle(P, O, ky, kx, sep, flags):
    rng = np.random.default_rng(ky * 31 + kx)
    if sep:
        f = P.Filter(wy=rng.uniform(0, 1, ky).astype(np.float32), wx=rng.uniform(0, 1, kx).astype(np.float32))
    else:
        f = P.Filter(rng.uniform(0, 1, (ky, kx)).astype(np.float32))
    assert P.tune_candidates_ex(f, flags) == O.tune_candidates_ex(ky, kx, sep, flags)
    if flags == 1:
        assert P.tune_candidates_ex(f, 1) == P.tune_candidates(f)


def test_skip_argument_errors(P):
    import ctypes as C
    from workloads import filters as F
    f = P.Filter(F.mean(5))
    img = P.Image(1, 8, 8, 8, 64, 0, 0)
    buf = C.c_void_p(16)
    out = C.c_void_p(1 << 20)
    assert P._lib.paraprox_stencil_skip_xy(f.handle, 0, 1, buf, out, C.byref(img), None) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_stencil_approx(f.handle, P.SKIP_ROW, 0, buf, out, C.byref(img), None) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_stencil_approx(f.handle, 7, 1, buf, out, C.byref(img), None) == P.ERR_INVALID_ARG
    n = C.c_int()
    assert P._lib.paraprox_tune_candidates_ex(f.handle, 0, 0, C.byref(n), None, None) == P.ERR_INVALID_ARG
    assert P._lib.paraprox_tune_candidates_ex(f.handle, 4, 0, C.byref(n), None, None) == P.ERR_INVALID_ARG
