"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same shapes, same entry points), on outputs the oracle can compute:
whole frames where the oracle is quick, else sampled patches (corners, edges,
interior) computed by the oracle on crops that keep the true image borders
(so clamp-to-edge is exercised where it applies)."""
import numpy as np
import pytest
import torch

import workloads as W
from workloads import filters as F

pytestmark = pytest.mark.gpu
RTOL = 1e-5


@pytest.fixture(scope="module")
def P():
    assert torch.cuda.is_available()
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def patches(h, w, size=48):
    ys = [0, h // 2 - size // 2, h - size]
    xs = [0, w // 3, w - size]
    return [(y, x) for y in ys for x in xs]


def check_patches(O, x, gpu, w, dy, dx, r, sep=None, size=48):
    h, wd = x.shape
    for (y0, x0) in patches(h, wd, size):
        cy0, cx0 = max(0, y0 - r), max(0, x0 - r)
        cy1, cx1 = min(h, y0 + size + r), min(wd, x0 + size + r)
        crop = x[cy0:cy1, cx0:cx1]
        if sep is None:
            o = O.stencil_approx_xy(crop, w, dy, dx)
            b = RTOL * O.stencil_approx_xy(np.abs(crop), np.abs(w), dy, dx)
        else:
            o = O.stencil_sep(crop, sep[0], sep[1], dy, dx)
            b = RTOL * O.stencil_sep(np.abs(crop), np.abs(sep[0]), np.abs(sep[1]), dy, dx)
        sl = (slice(y0 - cy0, y0 - cy0 + size), slice(x0 - cx0, x0 - cx0 + size))
        g = gpu[y0:y0 + size, x0:x0 + size]
        assert np.all(np.abs(g - o[sl]) <= b[sl]), (y0, x0, dy, dx)


def test_c2_mean5_4096_full_frame(P, O):
    x = W.image(4096, 4096, 10)
    w = F.mean(5)
    f = P.Filter(w)
    xd = torch.from_numpy(x).cuda()
    for dy, dx in [(0, 0), (2, 2), (2, 0), (0, 2), (1, 1), (1, 0), (0, 1)]:
        g = P.stencil_approx_xy(xd, f, dy, dx).cpu().numpy()
        o = O.stencil_approx_xy(x, w, dy, dx)
        assert np.all(np.abs(g - o) <= RTOL * np.abs(o)), (dy, dx)


def test_c3_sep7_256_frames_sampled(P, O):
    wy, wx = F.separable(7)
    f = P.Filter(wy=wy, wx=wx)
    base = W.frames(2, 2160, 3840, 20)
    xd = torch.empty((256, 2160, 3840), device="cuda")
    for k in range(256):
        xd[k].copy_(torch.from_numpy(base[k % 2]))
    for dy, dx in [(0, 0), (3, 3), (1, 1), (3, 0), (0, 3)]:
        out = P.stencil_approx_xy(xd, f, dy, dx)
        for k in (0, 131, 255):
            g = out[k].cpu().numpy()
            o = O.stencil_sep(base[k % 2], wy, wx, dy, dx)
            b = RTOL * O.stencil_sep(base[k % 2], np.abs(wy), np.abs(wx), dy, dx)
            assert np.all(np.abs(g - o) <= b), (dy, dx, k)
        del out
    del xd
    torch.cuda.empty_cache()


def test_c4_conv9_32768_sampled(P, O):
    w = F.conv(9)
    f = P.Filter(w)
    x = W.periodic(32768, 32768, tile=4096, seed=0)
    xd = torch.from_numpy(x).cuda()
    for dy, dx in [(0, 0), (4, 4), (4, 0), (1, 1), (2, 2), (1, 0), (0, 1)]:
        g = P.stencil_approx_xy(xd, f, dy, dx).cpu().numpy()
        check_patches(O, x, g, w, dy, dx, 4)
        del g
    del xd
    torch.cuda.empty_cache()


def test_c1_gauss3_512_batch(P, O):
    x = W.frames(110, 512, 512, 0)
    w = F.gaussian(3)
    f = P.Filter(w)
    xd = torch.from_numpy(x).cuda()
    for s, d in [("exact", 0), ("center", 1), ("row", 1), ("col", 1), ("center", 2)]:
        g = P.stencil_approx(xd, f, s, d).cpu().numpy()
        o = O.stencil_approx(x, w, s, d)
        assert np.all(np.abs(g - o) <= RTOL * np.abs(o)), (s, d)


def test_c4_lattice_sampled(P, O):
    """NEXT-1 at c4's size: the row lattice (reach 1 and 4) on 32768^2, sampled
    patches against the exact stencil on the rebuilt array X~ (oracle lattice
    map + oracle exact stencil on crops with a radius margin)."""
    w = F.conv(9)
    f = P.Filter(w)
    h = wd = 32768
    x = W.periodic(h, wd, tile=4096, seed=0)
    xd = torch.from_numpy(x).cuda()
    size, r = 48, 4
    for d in (1, 4):
        g = P.stencil_lattice(xd, f, "row", d).cpu().numpy()
        assert P.last_kernel().startswith("lattice_dense"), P.last_kernel()
        gy = O.lattice_map(h, d)
        for (y0, x0) in patches(h, wd, size):
            cy0, cx0 = max(0, y0 - r), max(0, x0 - r)
            cy1, cx1 = min(h, y0 + size + r), min(wd, x0 + size + r)
            xt = x[gy[cy0:cy1]][:, cx0:cx1]  # rows replaced by their accessed rows
            o = O.stencil_exact(xt, w)
            b = RTOL * O.stencil_exact(np.abs(xt), np.abs(w))
            sl = (slice(y0 - cy0, y0 - cy0 + size), slice(x0 - cx0, x0 - cx0 + size))
            assert np.all(np.abs(g[y0:y0 + size, x0:x0 + size] - o[sl]) <= b[sl]), (d, y0, x0)
        del g
    del xd
    torch.cuda.empty_cache()


def test_c3_lattice_sampled_frames(P, O):
    wy, wx = F.separable(7)
    f = P.Filter(wy=wy, wx=wx)
    base = W.frames(2, 2160, 3840, 30)
    xd = torch.empty((256, 2160, 3840), device="cuda")
    for k in range(256):
        xd[k].copy_(torch.from_numpy(base[k % 2]))
    for d in (1, 4):
        out = P.stencil_lattice(xd, f, "row", d)
        for k in (0, 255):
            g = out[k].cpu().numpy()
            o = O.stencil_lattice_xy(base[k % 2], (wy, wx), d, 0)
            b = RTOL * O.stencil_lattice_xy(base[k % 2], (np.abs(wy), np.abs(wx)), d, 0)
            assert np.all(np.abs(g - o) <= b), (d, k)
        del out
    del xd
    torch.cuda.empty_cache()
