"""Small invocations of every kernel family for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck): tile kernels (dense and
separable, border tiles, ragged shapes), the map kernel, the generic kernel,
lattice (fast and generic), reduction schemes, quality (flat and rows),
HotSpot (single step, blocked, fused), the runtime check path.

    compute-sanitizer --tool memcheck python tools/sanitize_run.py
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402
from workloads import hotspot as H  # noqa: E402

P = pkg.paraprox


def main():
    x = torch.from_numpy(W.frames(2, 70, 200, 1)).cuda()
    for w in (F.gaussian(3), F.mean(5), F.conv(9)):
        f = P.Filter(w)
        r = w.shape[0] // 2
        for dy, dx in ((0, 0), (1, 0), (0, 1), (r, r), (1, 1)):
            P.stencil_approx_xy(x, f, dy, dx)
        for d in (1, 2):
            P.stencil_lattice(x, f, "row", d)
            P.stencil_lattice(x, f, "center", d)
        P.stencil_skip_xy(x, f, 2, 3)
        e = P.stencil_exact(x, f)
        a = P.stencil_approx(x, f, "center", 1)
        P.quality(e, a, "mre")
        P.quality(e, a, "l2")
        P.quality(e[:, :, :199], a[:, :, :199], "mre")  # rows path
        P.tune(x, f, 0.9, "mre")
    fs = P.Filter(wy=F.separable(17, 1, 2)[0], wx=F.separable(17, 1, 2)[1])
    for dy, dx in ((0, 0), (3, 3), (8, 0)):
        P.stencil_approx_xy(x, fs, dy, dx)
    P.stencil_skip_xy(x, fs, 3, 2)
    P.stencil_lattice(x, fs, "row", 2)
    mis = torch.zeros(2 * 70 * 200 + 1, device="cuda")[1:].view(2, 70, 200)
    mis.copy_(x)
    P.stencil_approx_xy(mis, P.Filter(F.mean(5)), 1, 1, out=torch.zeros(2 * 70 * 200 + 1, device="cuda")[1:].view(2, 70, 200))
    t, p = H.frames(1, 50, 140, 2)
    td, pd = torch.from_numpy(t).cuda(), torch.from_numpy(p).cuda()
    for scheme, reach in (("exact", 0), ("row", 1), ("col", 1), ("center", 1)):
        P.hotspot(td, pd, H.PARAMS, scheme, reach, 1)
        P.hotspot(td, pd, H.PARAMS, scheme, reach, 11)
    # a grid with interior tiles of the temporally blocked kernel (no clamp)
    t2, p2 = H.frames(1, 200, 300, 3)
    t2d, p2d = torch.from_numpy(t2).cuda(), torch.from_numpy(p2).cuda()
    for scheme, reach in (("exact", 0), ("row", 1), ("col", 1)):
        P.hotspot(t2d, p2d, H.PARAMS, scheme, reach, 8)
    rt = P.Runtime(P.Filter(F.mean(5)), 0.9, "mre", check_every=2)
    rt.train(x)
    out = torch.empty_like(x)
    for _ in range(5):
        rt.run(x, out=out)
    rt.sync()
    torch.cuda.synchronize()
    print("sanitize run ok", P.launch_count())


if __name__ == "__main__":
    main()
