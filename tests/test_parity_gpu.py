"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.

Tolerance (reading S18): per output,
|gpu - oracle| <= 1e-5 * sum_ij |w_ij| |X~_ij| (the oracle run on |w|, |X|),
i.e. a 1e-5 relative error for non-negative filters, guarded against
cancellation for signed ones.  Integer-valued decisions (the tuner) must be
identical."""
import numpy as np
import pytest
import torch

import workloads as W
from workloads import filters as F

pytestmark = pytest.mark.gpu

RTOL = 1e-5


@pytest.fixture(scope="module")
def P():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def assert_dense(P, O, x, w, dy, dx, f=None):
    f = f or P.Filter(w)
    g = P.stencil_approx_xy(dev(x), f, dy, dx).cpu().numpy()
    o = O.stencil_approx_xy(x, w, dy, dx)
    bound = RTOL * O.stencil_approx_xy(np.abs(x), np.abs(w), dy, dx) + 1e-30
    err = np.abs(g - o)
    assert np.all(err <= bound), (dy, dx, float((err / bound).max()), P.last_kernel())
    return g


def assert_sep(P, O, x, wy, wx, dy, dx, f=None):
    f = f or P.Filter(wy=wy, wx=wx)
    g = P.stencil_approx_xy(dev(x), f, dy, dx).cpu().numpy()
    o = O.stencil_sep(x, wy, wx, dy, dx)
    bound = RTOL * O.stencil_sep(np.abs(x), np.abs(wy), np.abs(wx), dy, dx) + 1e-30
    err = np.abs(g - o)
    assert np.all(err <= bound), (dy, dx, float((err / bound).max()), P.last_kernel())
    return g


DENSE = [
    ("gauss3", F.gaussian(3)),
    ("mean5", F.mean(5)),
    ("conv7", F.conv(7, seed=3)),
    ("conv9", F.conv(9)),
    ("signed5", F.conv_signed(5)),
    ("rect3x7", F.conv(7, seed=11, ky=3)),
    ("rect9x1", F.conv(1, seed=12, ky=9)),
    ("conv17", F.conv(17, seed=13)),
    ("one", np.ones((1, 1), np.float32)),
]


@pytest.mark.parametrize("name,w", DENSE, ids=[d[0] for d in DENSE])
@pytest.mark.parametrize("shape", [(2, 77, 300), (1, 257, 513)], ids=["2x77x300", "1x257x513"])
def test_dense_all_reaches(P, O, name, w, shape):
    """Every (dy, dx) pair, over several tiles with ragged tails."""
    x = W.frames(*shape, seed0=1)
    f = P.Filter(w)
    ky, kx = w.shape
    ry, rx = ky // 2, kx // 2
    pairs = {(dy, dx) for dy in range(ry + 2) for dx in range(rx + 2)}
    if len(pairs) > 40:  # 17x17: schemes x reaches only
        pairs = {(d, d) for d in range(ry + 2)} | {(d, 0) for d in range(ry + 2)} | {(0, d) for d in range(rx + 2)}
    for dy, dx in sorted(pairs):
        assert_dense(P, O, x, w, dy, dx, f)


@pytest.mark.parametrize("ky,kx", [(7, 7), (3, 5), (1, 17), (17, 1), (9, 9), (17, 17), (5, 11)])
@pytest.mark.parametrize("shape", [(2, 77, 300), (1, 190, 700)], ids=["2x77x300", "1x190x700"])
def test_separable_all_reaches(P, O, ky, kx, shape):
    wy = F.conv(1, seed=40 + ky, ky=ky).ravel()
    wx = F.conv(kx, seed=50 + kx, ky=1).ravel()
    x = W.frames(*shape, seed0=2)
    f = P.Filter(wy=wy, wx=wx)
    for dy in range(ky // 2 + 2):
        for dx in range(kx // 2 + 2):
            assert_sep(P, O, x, wy, wx, dy, dx, f)


@pytest.mark.parametrize("shape", [(1, 1, 1), (3, 1, 1), (1, 1, 700), (1, 700, 1), (1, 5, 5), (2, 8, 8),
                                   (1, 3, 129), (1, 33, 4), (1, 31, 127)])
def test_degenerate_shapes(P, O, shape):
    x = W.images.random_integers(shape, seed=3, lo=0, hi=255)
    for w in (F.gaussian(3), F.mean(5), F.conv(9)):
        for d in range(0, w.shape[0] // 2 + 2):
            for dy, dx in ((d, 0), (0, d), (d, d)):
                assert_dense(P, O, x, w, dy, dx)
    wy, wx = F.separable(7)
    for d in range(5):
        assert_sep(P, O, x, wy, wx, d, d)


@pytest.mark.parametrize("k", [3, 5, 7])
def test_bruteforce_8x8_all_schemes(P, O, k):
    w = F.conv(k, seed=100 + k)
    for seed in range(3):
        x = W.images.random_integers((8, 8), seed)
        for scheme in ("exact", "row", "col", "center"):
            for d in range(0, k // 2 + 2):
                dy, dx = O.scheme_reaches(scheme, d)
                assert_dense(P, O, x, w, dy, dx)


def test_scheme_entry_points_agree(P, O):
    x = W.frames(2, 70, 140, 4)
    w = F.conv(9)
    f = P.Filter(w)
    xd = dev(x)
    e = P.stencil_exact(xd, f)
    assert torch.equal(e, P.stencil_approx(xd, f, "exact", 3))
    assert torch.equal(e, P.stencil_approx(xd, f, "row", 0))
    for scheme in ("row", "col", "center"):
        for d in range(1, 6):
            dy, dx = O.scheme_reaches(scheme, d)
            assert torch.equal(P.stencil_approx(xd, f, scheme, d), P.stencil_approx_xy(xd, f, dy, dx))


def test_invariants_on_gpu(P):
    f = P.Filter(F.mean(5))
    c = torch.full((1, 100, 200), 77.0, device="cuda")
    for d in range(3):
        for s in ("row", "col", "center"):
            torch.testing.assert_close(P.stencil_approx(c, f, s, d), c, rtol=1e-6, atol=0)
    yc = dev(np.repeat(W.image(1, 300, 5), 90, axis=0))
    e = P.stencil_exact(yc, f)
    for d in (1, 2):
        torch.testing.assert_close(P.stencil_approx(yc, f, "row", d), e, rtol=2e-6, atol=0)


def test_pitched_and_strided_layouts(P, O):
    """pitch > w, frame_stride > h*pitch, and a misaligned base pointer."""
    x = W.frames(3, 50, 130, 6)
    w = F.conv(5, seed=8)
    f = P.Filter(w)
    o = O.stencil_exact(x, w)
    big = torch.zeros((3, 60, 141), device="cuda")
    big[:, 3:53, 5:135] = dev(x)
    view = big[:, 3:53, 5:135]  # pitch 141, frame stride 60*141, offset 3*141+5 floats
    out = torch.zeros_like(big)[:, 3:53, 5:135]
    g = P.stencil_exact(view, f, out=out).cpu().numpy()
    bound = RTOL * O.stencil_exact(np.abs(x), np.abs(w))
    assert np.all(np.abs(g - o) <= bound)


def test_stripes_with_halos_bitwise(P, O):
    """Row stripes with halo rows reproduce the whole-image output bitwise
    (same kernel, same tap order): the multi-GPU row-stripe decomposition."""
    x = W.image(1000, 777, 7)
    w = F.conv(9)
    f = P.Filter(w)
    xd = dev(x)
    for dy, dx in [(0, 0), (1, 1), (4, 0), (0, 4), (2, 2)]:
        full = P.stencil_approx_xy(xd, f, dy, dx)
        hy = f.plan_info(dy, dx)["halo_y"]
        for g in (2, 3, 8):
            bounds = [1000 * k // g for k in range(g + 1)]
            for k in range(g):
                r0, r1 = bounds[k], bounds[k + 1]
                ht, hb = min(hy, r0), min(hy, 1000 - r1)
                stripe = xd[r0 - ht:r1 + hb].clone()
                got = P.stencil_approx_xy(stripe, f, dy, dx, halo_top=ht, halo_bottom=hb)
                assert torch.equal(got, full[r0:r1]), (dy, dx, g, k)


def test_quality_matches_oracle_and_is_deterministic(P, O):
    x = W.frames(3, 300, 400, 9)
    f = P.Filter(F.mean(5))
    xd = dev(x)
    e = P.stencil_exact(xd, f)
    a = P.stencil_approx(xd, f, "center", 1)
    en, an = e.cpu().numpy().astype(np.float64), a.cpu().numpy().astype(np.float64)
    for m in ("mre", "l2", "psnr"):
        q1 = P.quality(e, a, m)
        q2 = P.quality(e, a, m)
        assert q1 == q2
        qo = O.quality(en, an, m)
        assert abs(q1 - qo) <= 1e-12 * max(1.0, abs(qo)), (m, q1, qo)
    assert P.quality(e, e, "mre") == 1.0
    # partials add across disjoint pixel sets
    p0 = P.quality_partials(e[:1], a[:1], "l2")
    p1 = P.quality_partials(e[1:], a[1:], "l2")
    assert P.quality_from_partials(p0 + p1, "l2") == pytest.approx(P.quality(e, a, "l2"), abs=1e-14)


TUNE_CASES = [
    ("gauss3", F.gaussian(3), "mre", (10, 256, 256)),
    ("mean5", F.mean(5), "mre", (10, 256, 256)),
    ("conv9", F.conv(9), "l2", (10, 256, 256)),
    ("sep7", F.separable(7), "l2", (10, 216, 384)),
    ("sep17", F.separable(17, 3, 4), "l2", (6, 200, 300)),  # the wide separable path (ConvSep loops)
]


@pytest.mark.parametrize("name,w,metric,shape", TUNE_CASES, ids=[t[0] for t in TUNE_CASES])
def test_tuner_bit_identical(P, O, name, w, metric, shape):
    x = W.frames(*shape, seed0=0)
    f = P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)
    xd = dev(x)
    parts = P.tune_partials(xd, f, metric)
    ref_all = O.tune(x, w, 2.0 if metric != "psnr" else 1e9, metric, all_qualities=True)["qualities"]
    qs = [P.quality_from_partials(parts[3 * k:3 * k + 3], metric) for k in range(len(ref_all))]
    np.testing.assert_allclose(qs, ref_all, rtol=0, atol=1e-7)
    for toq in (0.80, 0.90, 0.95, 0.99):
        got = P.tune(xd, f, toq, metric)
        ref = O.tune(x, w, toq, metric)
        margin = min(abs(q - toq) for q in ref_all)
        assert got[:2] == (ref["scheme"], ref["reach"]), (toq, got, ref, margin)
        assert P.tune_decide(f, parts, toq, metric) == got
        print(f"{name} toq={toq}: {got[0]}:{got[1]} q={got[2]:.6f} (oracle {ref['quality']:.6f}), "
              f"min |q-toq| = {margin:.2e}")


def test_tuner_tpins_on_gpu(P):
    f = P.Filter(F.mean(5))
    yc = dev(np.repeat(W.image(1, 128, 3), 64, axis=0)[None])
    assert P.tune(yc, f, 1 - 1e-6, "mre")[:2] == ("row", 2)
    const = torch.full((2, 64, 64), 120.0, device="cuda")
    assert P.tune(const, f, 1 - 1e-6, "l2")[:2] == ("center", 2)
    noise = dev(W.uniform_noise(128, 128, 5)[None])
    assert P.tune(noise, f, 0.95, "mre") == ("exact", 0, 1.0)


def test_run_host_matches_device_path(P):
    # single-chunk shapes, then shapes that take the ramped chunk schedule
    # (row bands of 64/128/256 rows at both ends of a 2048 x 4096 image with a
    # 4-row halo; 1/1/2-frame chunks at both ends of a 40-frame batch)
    for shape, w in [((1, 1500, 900), F.conv(9)), ((5, 120, 256), F.mean(5)), ((1, 2048, 4096), F.conv(9)),
                     ((40, 256, 2048), F.mean(5))]:
        x = torch.from_numpy(W.frames(*shape, seed0=12)).pin_memory()
        f = P.Filter(w)
        for scheme, d in [("exact", 0), ("row", 1), ("center", 2)]:
            host = P.run_host(x[0] if shape[0] == 1 else x, f, scheme, d)
            ref = P.stencil_approx(x.cuda(), f, scheme, d).cpu()
            assert torch.equal(host, ref[0] if shape[0] == 1 else ref), (shape, scheme, d)


def test_launches_counted(P):
    f = P.Filter(F.gaussian(3))
    x = torch.rand(1, 64, 64, device="cuda")
    n0 = P.launch_count()
    P.stencil_exact(x, f)
    P.stencil_approx(x, f, "row", 1)
    torch.cuda.synchronize()
    assert P.launch_count() - n0 == 2


@pytest.mark.parametrize("kind,w", [("dense", F.gaussian(3)), ("dense", F.mean(5)), ("dense", F.conv(9)),
                                    ("dense", F.conv(7, seed=3)), ("sep", F.separable(7))])
def test_fast_path_taken(P, kind, w):
    """Aligned layouts of every BASELINE filter take the TMA tile kernels."""
    f = P.Filter(wy=w[0], wx=w[1]) if kind == "sep" else P.Filter(w)
    x = torch.rand(2, 200, 260, device="cuda")
    r = f.ky // 2
    for dy, dx in [(0, 0), (r, r), (1, 0), (0, 1), (r, 0), (0, r)]:
        P.stencil_approx_xy(x, f, dy, dx)
        assert P.last_kernel().startswith(kind + "_"), (dy, dx, P.last_kernel())


@pytest.mark.parametrize("w", [F.mean(5), F.conv(9), F.conv_signed(5), F.gaussian(3)])
def test_generic_and_tile_kernels_bitwise(P, w):
    """The tile kernel and the generic kernel sum the folded taps in the same
    order: an aligned (tile / map path) and a misaligned (generic / row-map
    path) copy of the same image give identical bits."""
    f = P.Filter(w)
    x = dev(W.frames(2, 150, 336, 30))
    buf = torch.zeros(2 * 150 * 336 + 1, device="cuda")
    mis = buf[1:].view(2, 150, 336)
    mis.copy_(x)
    r = w.shape[0] // 2
    for dy, dx in [(0, 0), (1, 1), (r, 0), (0, r), (r, r)]:
        a = P.stencil_approx_xy(x, f, dy, dx)
        ka = P.last_kernel()
        ob = torch.zeros(2 * 150 * 336 + 1, device="cuda")[1:].view(2, 150, 336)
        b = P.stencil_approx_xy(mis, f, dy, dx, out=ob)
        kb = P.last_kernel()
        # centre-only plans are maps: the misaligned copy takes the row-wise map
        assert ka != "generic" and kb in ("generic", "dense_map_rows"), (ka, kb)
        assert torch.equal(a, b), (dy, dx)


def test_fused_tuner_partials_match_unfused(P):
    """The tuner scores candidates with the fused stencil + quality epilogue;
    the unfused path (PARAPROX_FUSED_QUALITY=0: stencil stored, then the
    quality kernel) gives the same qualities to rounding and the same
    decisions."""
    import json
    import os
    import subprocess
    import sys
    code = r'''
import json, sys, torch
sys.path.insert(0, %r)
import paper_conf_asplos_samadijlm14_b200 as pkg
import workloads as W
from workloads import filters as F
P = pkg.paraprox
out = {}
for name, w, m in [("mean5", F.mean(5), "mre"), ("conv9", F.conv(9), "l2"), ("sep7", F.separable(7), "l2"),
                   ("sep17", F.separable(17, 3, 4), "l2")]:
    f = P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)
    x = torch.from_numpy(W.frames(4, 160, 200, 3)).cuda()
    out[name] = P.tune_partials(x, f, m).tolist()
    # 6144 tiles: two waves of the bounded-persistence schedule
    xb = torch.from_numpy(W.frames(3, 4096, 4096, 5)).cuda()
    out[name + "_waves"] = P.tune_partials(xb, f, m).tolist()
print(json.dumps(out))
''' % (os.path.dirname(os.path.dirname(os.path.abspath(__file__))),)
    res = {}
    for flag in ("1", "0"):
        env = dict(os.environ, PARAPROX_FUSED_QUALITY=flag)
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr
        res[flag] = json.loads(r.stdout.strip().splitlines()[-1])
    metric = {"mean5": "mre", "conv9": "l2", "sep7": "l2", "sep17": "l2"}
    for name in res["1"]:
        a, b = np.array(res["1"][name]), np.array(res["0"][name])
        mt = metric[name.split("_")[0]]
        qa = [P.quality_from_partials(a[3 * k:3 * k + 3], mt) for k in range(len(a) // 3)]
        qb = [P.quality_from_partials(b[3 * k:3 * k + 3], mt) for k in range(len(b) // 3)]
        np.testing.assert_allclose(qa, qb, rtol=0, atol=1e-12)


def test_tile_schedules_bitwise():
    """Bounded persistence (default: 4 tiles per CTA for 4-warp instances,
    16 for 8-warp ones, 4 for the lattice), other chunk sizes and the fully
    persistent grid (PARAPROX_TILE_CHUNK=0 / PARAPROX_LATTICE_CHUNK=0) compute
    every tile with the same code: outputs are bit-identical, here on up to
    24 k tiles (several waves) with ragged edges."""
    import os
    import subprocess
    import sys
    code = r'''
import hashlib, sys, torch
sys.path.insert(0, %r)
import paper_conf_asplos_samadijlm14_b200 as pkg
import workloads as W
from workloads import filters as F
P = pkg.paraprox
x = torch.from_numpy(W.frames(3, 4090, 4093, 7)).cuda()
h = hashlib.sha256()
for w in (F.mean(5), F.conv(9), F.gaussian(3)):
    f = P.Filter(w)
    for scheme, d in (("exact", 0), ("row", 1), ("center", 1), ("col", 2)):
        h.update(P.stencil_approx(x, f, scheme, d).cpu().numpy().tobytes())
    h.update(P.stencil_lattice(x, f, "row", 1).cpu().numpy().tobytes())
fs = P.Filter(wy=F.separable(7)[0], wx=F.separable(7)[1])
h.update(P.stencil_approx(x, fs, "row", 1).cpu().numpy().tobytes())
print(h.hexdigest())
''' % (os.path.dirname(os.path.dirname(os.path.abspath(__file__))),)
    digests = []
    for chunk in ("", "16", "2", "0"):
        env = dict(os.environ, PARAPROX_TILE_CHUNK=chunk, PARAPROX_LATTICE_CHUNK="0" if chunk == "0" else chunk)
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr
        digests.append(r.stdout.strip().splitlines()[-1])
    assert len(set(digests)) == 1, digests


def test_tma_store_and_register_store_epilogues_bitwise():
    """Tile kernels send their outputs as one TMA tensor store per tile by
    default; PARAPROX_TMA_STORE=0 keeps 128-bit register stores.  Both write
    the same bits, including ragged edges (tiles clipped by the image) and a
    pitched layout whose padding columns must stay untouched."""
    import os
    import subprocess
    import sys
    code = r'''
import sys, hashlib, torch
sys.path.insert(0, %r)
import paper_conf_asplos_samadijlm14_b200 as pkg
import workloads as W
from workloads import filters as F
P = pkg.paraprox
h = hashlib.sha256()
for name, w in [("gauss3", F.gaussian(3)), ("mean5", F.mean(5)), ("conv9", F.conv(9)), ("sep7", F.separable(7))]:
    f = P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)
    x = torch.from_numpy(W.frames(3, 131, 300, 5)).cuda()
    r = f.ky // 2
    for dy, dx in [(0, 0), (1, 0), (0, 1), (r, 0), (1, 1)]:
        y = P.stencil_approx_xy(x, f, dy, dx)
        h.update(y.cpu().numpy().tobytes())
        xb = torch.zeros((3, 131, 308), device="cuda")
        xb[:, :, :300] = x
        big = torch.full((3, 131, 308), -7.0, device="cuda")
        P.stencil_approx_xy(xb[:, :, :300], f, dy, dx, out=big[:, :, :300])
        h.update(big.cpu().numpy().tobytes())
print(h.hexdigest(), P.last_kernel())
''' % (os.path.dirname(os.path.dirname(os.path.abspath(__file__))),)
    res = {}
    for flag in ("1", "0"):
        env = dict(os.environ, PARAPROX_TMA_STORE=flag)
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr
        res[flag] = r.stdout.strip().splitlines()[-1]
    assert res["1"] == res["0"], res
    assert not res["1"].endswith("generic"), res


def test_fused_quality_many_tiny_frames(P, O):
    """20 000 frames of 16 x 16: one tile per frame, so the tiles outnumber
    the scratch's partial pairs (sized from the pixel count, 1250 here) under
    the bounded-persistence schedule; the fused-quality launch keeps the
    persistent grid instead.  Qualities equal the oracle's on the GPU's own
    outputs to rounding, and the tuner's to 1e-8 (test_fullsize_tuner_gpu:
    the folded weights are rounded to fp32 once, a bias shared by all pixels)."""
    rng = np.random.default_rng(31)
    base = W.image(160, 2000, 3)  # smooth seeded field cut into 16x16 frames
    x = np.ascontiguousarray(base.reshape(10, 16, 125, 16).transpose(0, 2, 1, 3).reshape(1250, 16, 16))
    x = np.ascontiguousarray(np.concatenate([x] * 16)[rng.permutation(20000)])
    f = P.Filter(F.mean(5))
    xd = dev(x)
    cands = P.tune_candidates(f)
    parts = P.tune_partials(xd, f, "mre")
    qg = [P.quality_from_partials(parts[3 * k:3 * k + 3], "mre") for k in range(len(cands))]
    qo = O.tune(x, F.mean(5), 2.0, "mre", all_qualities=True)["qualities"]
    np.testing.assert_allclose(qg, qo, rtol=0, atol=1e-8)
    en = P.stencil_exact(xd, f).cpu().numpy()
    for k, (s, r) in enumerate(cands):
        an = P.stencil_approx(xd, f, s, r).cpu().numpy()
        assert abs(qg[k] - O.quality(en, an, "mre")) <= 1e-12, (s, r)


def test_wide_separable_layouts_and_stripes(P, O):
    """The wide separable path (17-tap loops, `sep_wide`): aligned pitched and
    strided layouts (pitch 532 > w, frame stride > h * pitch) against the
    oracle, and row stripes with halo rows bitwise equal to the whole image
    (the stripe-edge tiles clamp at their valid rows)."""
    wy = F.conv(1, seed=61, ky=17).ravel()
    wx = F.conv(17, seed=62, ky=1).ravel()
    f = P.Filter(wy=wy, wx=wx)
    x = W.frames(3, 150, 520, 8)
    big = torch.zeros((3, 170, 532), device="cuda")
    big[:, 4:154, 8:528] = dev(x)
    view = big[:, 4:154, 8:528]  # 16-byte aligned: the tile (TMA) path
    outb = torch.zeros_like(big)
    out = outb[:, 4:154, 8:528]
    for dy, dx in [(0, 0), (3, 3), (0, 8), (8, 0), (2, 5)]:
        g = P.stencil_approx_xy(view, f, dy, dx, out=out).cpu().numpy()
        assert P.last_kernel().startswith("sep8_") or (dy, dx) == (2, 5), P.last_kernel()
        o = O.stencil_sep(x, wy, wx, dy, dx)
        bound = RTOL * O.stencil_sep(np.abs(x), np.abs(wy), np.abs(wx), dy, dx) + 1e-30
        assert np.all(np.abs(g - o) <= bound), (dy, dx, P.last_kernel())
        assert torch.count_nonzero(outb[:, :4]) == 0 and torch.count_nonzero(outb[:, :, :8]) == 0  # no stray writes
    img = dev(W.image(700, 600, 9))
    for dy, dx in [(0, 0), (3, 3)]:
        full = P.stencil_approx_xy(img, f, dy, dx)
        hy = f.plan_info(dy, dx)["halo_y"]
        bounds = [0, 130, 333, 700]
        for k in range(3):
            r0, r1 = bounds[k], bounds[k + 1]
            ht, hb = min(hy, r0), min(hy, 700 - r1)
            got = P.stencil_approx_xy(img[r0 - ht:r1 + hb].clone(), f, dy, dx, halo_top=ht, halo_bottom=hb)
            assert torch.equal(got, full[r0:r1]), (dy, dx, k)


def test_concurrent_streams_and_threads(P):
    """The library keeps no global mutable state on the data path (scratch is
    stream-ordered, plans are cached behind a lock): four host threads, each
    on its own stream, run stencils, qualities and the tuner concurrently on
    different filters and frames; every result equals the sequential one."""
    import threading

    jobs = [(F.mean(5), "mre", 0), (F.conv(9), "l2", 1), (F.gaussian(3), "mre", 2), (F.separable(7), "l2", 3)]
    frames = [dev(W.frames(3, 512, 640, 10 * k)) for k in range(4)]
    torch.cuda.synchronize()

    def work(k, res):
        w, m, _ = jobs[k]
        f = P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            x = frames[k]
            out = []
            for _ in range(3):
                e = P.stencil_exact(x, f, stream=s)
                a = P.stencil_approx(x, f, "center", 1, stream=s)
                q = P.quality(e, a, m, stream=s)
                t = P.tune(x, f, 0.9, m, stream=s)
                s.synchronize()
                out.append((e.cpu(), a.cpu(), q, t))
            res[k] = out

    seq = {}
    for k in range(4):
        work(k, seq)
    par = {}
    ths = [threading.Thread(target=work, args=(k, par)) for k in range(4)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    for k in range(4):
        for (e0, a0, q0, t0), (e1, a1, q1, t1) in zip(seq[k], par[k]):
            assert torch.equal(e0, e1) and torch.equal(a0, a1), k
            assert q0 == q1 and t0 == t1, (k, q0, q1, t0, t1)


def test_generic_kernels_tall_images(P, O):
    """More than 65535 x 8 rows on the fallback kernels (pitch 5 is not
    TMA-describable): they grid-stride over rows."""
    x = W.images.random_integers((1, 600001, 5), seed=4, lo=16, hi=235)
    w = F.mean(5)
    f = P.Filter(w)
    for scheme, d in (("exact", 0), ("row", 1)):
        g = P.stencil_approx(dev(x), f, scheme, d).cpu().numpy()
        assert P.last_kernel() == "generic", P.last_kernel()
        o = O.stencil_approx(x, w, scheme, d)
        assert np.all(np.abs(g - o) <= RTOL * O.stencil_approx(np.abs(x), np.abs(w), scheme, d) + 1e-30), scheme
    g = P.stencil_lattice(dev(x), f, "col", 1).cpu().numpy()
    assert P.last_kernel() == "lattice_generic", P.last_kernel()
    o = O.stencil_lattice(x, w, "col", 1)
    assert np.all(np.abs(g - o) <= RTOL * O.stencil_lattice(np.abs(x), np.abs(w), "col", 1) + 1e-30)
