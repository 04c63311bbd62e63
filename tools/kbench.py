"""Kernel-level timing sweep (GPU box): every (workload, reach pair) of the
tile kernels plus the quality kernel, CUDA events over back-to-back launches
on rotating buffers larger than L2.  Prints one JSON object per line.

    python tools/kbench.py [--workloads c1,c2,c4] [--reps 20]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
SHAPES = {"c1": (110, 512, 512, "gauss3"), "c2": (1, 4096, 4096, "mean5"), "c3": (32, 2160, 3840, "sep7"),
          "c4": (1, 16384, 16384, "conv9")}


def timeit(fn, nbuf, reps, stream):
    for k in range(3):
        fn(k % nbuf)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for k in range(reps):
        fn(k % nbuf)
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workloads", default="c1,c2,c3,c4")
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    for wl in args.workloads.split(","):
        n, h, w, fname = SHAPES[wl]
        kind, wt = F.named(fname)
        f = P.Filter(wy=wt[0], wx=wt[1]) if kind == "sep" else P.Filter(wt)
        px = n * h * w
        nbuf = max(1, min(6, -(-(3 * l2) // (8 * px))))
        ins = [torch.rand((n, h, w), device=dev) * 200 + 16 for _ in range(nbuf)]
        outs = [torch.empty_like(ins[0]) for _ in range(nbuf)]
        r = f.plan_info(0, 0)
        ry = (len(r["map_y"]) - 1) // 2
        rx = (len(r["map_x"]) - 1) // 2
        seen = set()
        for dy in range(ry + 1):
            for dx in range(rx + 1):
                info = f.plan_info(dy, dx)
                key = (tuple(info["map_y"]), tuple(info["map_x"]))
                if key in seen:
                    continue
                seen.add(key)
                ops = [P.Prepared(ins[k], f, "exact", 0, outs[k], stream=stream) for k in range(nbuf)]
                for k in range(nbuf):  # bind reaches through the xy entry point
                    ops[k]._fn = P._lib.paraprox_stencil_approx_xy
                    a = ops[k]._args
                    ops[k]._args = (a[0], dy, dx) + a[3:]
                ms = timeit(lambda k: ops[k](), nbuf, args.reps, stream)
                print(json.dumps({"wl": wl, "dy": dy, "dx": dx, "kernel": P.last_kernel(), "taps": info["taps"],
                                  "us": round(1e3 * ms, 2), "gbs": round(8 * px / ms / 1e6, 1)}), flush=True)
        for d in (1, 2, 3, 4):  # global-lattice row scheme: 4/(2d+1) + 4 B per pixel
            ops = [P.Prepared(ins[k], f, "row", d, outs[k], stream=stream, lattice=True) for k in range(nbuf)]
            ms = timeit(lambda k: ops[k](), nbuf, args.reps, stream)
            alg = (4.0 / (2 * d + 1) + 4.0) * px
            print(json.dumps({"wl": wl, "lattice_dy": d, "kernel": P.last_kernel(), "us": round(1e3 * ms, 2),
                              "alg_bytes_px": round(alg / px, 3), "gbs": round(alg / ms / 1e6, 1),
                              "mpx_s": round(px / ms / 1e3, 1)}), flush=True)
        part = torch.empty(3, dtype=torch.float64, device=dev)
        for m in ("mre", "l2"):
            ms = timeit(lambda k: P.quality_partials_async(ins[k], outs[k], m, part, stream=stream), nbuf,
                        args.reps, stream)
            print(json.dumps({"wl": wl, "kernel": "quality_" + m, "us": round(1e3 * ms, 2),
                              "gbs": round(8 * px / ms / 1e6, 1)}), flush=True)
        del ins, outs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
