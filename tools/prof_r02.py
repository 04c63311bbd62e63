"""Launch one instance of each kernel the r02 verdict names, for one ncu
--set full capture (ncu -k regex:... -c N):

  c2 exact 5x5 (dense_f2_f2), c4 exact 9x9 (dense_f4_f4, a 8192-row band of
  the c4 image), ConvSep exact 1x17 + 17x1 (sep8_f8_f8, 16 x 2048^2), the
  c4 row lattice s = 3 (lattice_dense_s3_r4), HotSpot 8 blocked steps at
  8192^2 (hotspot_tb_f1_f1).

    python tools/prof_r02.py [--only name,name]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default="")
    ap.add_argument("--reps", type=int, default=2)
    args = ap.parse_args()
    import torch

    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    from workloads import hotspot as H
    P = pkg.paraprox
    only = set(filter(None, args.only.split(",")))

    def want(n):
        return not only or n in only

    if want("c2"):
        x = torch.from_numpy(W.image(4096, 4096, 0)).cuda().view(1, 4096, 4096)
        f = P.Filter(F.mean(5))
        for _ in range(args.reps):
            P.stencil_exact(x, f)
        torch.cuda.synchronize()
        print("c2", P.last_kernel(), flush=True)
        del x
    if want("c4") or want("lattice"):
        x = torch.from_numpy(W.periodic(8192, 32768, tile=4096, seed=0)).cuda().view(1, 8192, 32768)
        f = P.Filter(F.conv(9))
        if want("c4"):
            for _ in range(args.reps):
                P.stencil_exact(x, f)
            torch.cuda.synchronize()
            print("c4", P.last_kernel(), flush=True)
        if want("lattice"):
            for _ in range(args.reps):
                P.stencil_lattice(x, f, "row", 1)
            torch.cuda.synchronize()
            print("lattice", P.last_kernel(), flush=True)
        del x
    if want("convsep"):
        x = torch.from_numpy(W.frames(4, 2048, 2048, 0)).cuda().repeat(4, 1, 1)
        wy, wx = F.separable(17)
        f = P.Filter(wy=wy, wx=wx)
        for _ in range(args.reps):
            P.stencil_exact(x, f)
        torch.cuda.synchronize()
        print("convsep", P.last_kernel(), flush=True)
        del x
    if want("hotspot"):
        t, p = H.frames(1, 8192, 8192, 11)
        td, pd = torch.from_numpy(t).cuda(), torch.from_numpy(p).cuda()
        for _ in range(args.reps):
            P.hotspot(td, pd, H.PARAMS, "exact", 0, 8)
        torch.cuda.synchronize()
        print("hotspot", P.last_kernel(), flush=True)


if __name__ == "__main__":
    main()
