"""Bit-identity of the wide separable path (r02) with the r01 separable path:
the same inputs through the in-tree library and an A/B build of the previous
source (PARAPROX_LIB_OLD=abship/lib_old.so, loaded in a subprocess), every
reach pair of a 17-tap separable filter, ragged shapes."""
import os
import subprocess
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def run(out_path):
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    res = {}
    for shape in ((2, 77, 300), (1, 190, 700), (3, 2048, 2048)):
        x = torch.from_numpy(W.frames(*shape, seed0=4)).cuda()
        for ky, kx in ((17, 17), (1, 17), (11, 13)):
            wy, wx = F.separable(17, 5, 6)
            wy = F.conv(1, seed=40 + ky, ky=ky).ravel()
            wx = F.conv(kx, seed=50 + kx, ky=1).ravel()
            f = P.Filter(wy=wy, wx=wx)
            for dy, dx in ((0, 0), (3, 3), (8, 0), (0, 8), (1, 2), (5, 5)):
                o = P.stencil_approx_xy(x, f, dy, dx)
                res[f"{shape}_{ky}x{kx}_{dy}_{dx}"] = (o.cpu().numpy(), P.last_kernel())
    np.savez(out_path, **{k: v[0] for k, v in res.items()})
    print({k: v[1] for k, v in list(res.items())[:6]})


if __name__ == "__main__":
    if len(sys.argv) > 1:
        run(sys.argv[1])
        sys.exit(0)
    env = dict(os.environ)
    subprocess.check_call([sys.executable, __file__, "/tmp/sep_new.npz"], env=env)
    env["PARAPROX_LIB"] = os.path.join(ROOT, "abship", "lib_old.so")
    subprocess.check_call([sys.executable, __file__, "/tmp/sep_old.npz"], env=env)
    a, b = np.load("/tmp/sep_new.npz"), np.load("/tmp/sep_old.npz")
    bad = [k for k in a.files if not np.array_equal(a[k], b[k])]
    print(f"sep_wide bitwise: {len(a.files) - len(bad)}/{len(a.files)} identical", bad[:5])
    sys.exit(1 if bad else 0)
