"""Launch a few stencil kernels of one workload for ncu captures.

    python tools/prof_run.py --workload c2 --schemes exact:0,center:2 --reps 3
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--schemes", default="exact:0,center:2")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--quality", action="store_true")
    ap.add_argument("--lattice", default="", help="lattice schemes, e.g. row:1,row:4")
    args = ap.parse_args()
    import torch

    import bench
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    P = pkg.paraprox
    wl = bench.WORKLOADS[args.workload]
    kind, w = bench.make_filter_arrays(wl["filter"])
    f = P.Filter(wy=w[0], wx=w[1]) if kind == "sep" else P.Filter(w)
    n, h, wd = wl["n"], wl["h"], wl["w"]
    if args.workload == "c4":
        x = torch.from_numpy(W.periodic(h, wd, tile=4096, seed=0)).cuda().view(1, h, wd)
    elif n == 1:
        x = torch.from_numpy(W.image(h, wd, 0)).cuda().view(1, h, wd)
    else:
        base = W.frames(min(n, 4), h, wd, 0)
        x = torch.empty((n, h, wd), device="cuda")
        for k in range(n):
            x[k].copy_(torch.from_numpy(base[k % len(base)]))
    out = torch.empty_like(x)
    e = torch.empty_like(x)
    P.stencil_exact(x, f, out=e)
    for spec in args.schemes.split(","):
        s, r = spec.split(":")
        for _ in range(args.reps):
            P.stencil_approx(x, f, s, int(r), out=out)
        torch.cuda.synchronize()
        print(spec, P.last_kernel())
        if args.quality:
            for _ in range(args.reps):
                P.quality(e, out, wl["metric"])
    for spec in filter(None, args.lattice.split(",")):
        s, r = spec.split(":")
        for _ in range(args.reps):
            P.stencil_lattice(x, f, s, int(r), out=out)
        torch.cuda.synchronize()
        print("lattice", spec, P.last_kernel())


if __name__ == "__main__":
    main()
