"""Tuner (row a5) timing on the GPU box: device time of one warm
`tune_partials` call per workload on its training frames (random-valued
frames of the same shape; the tuner's work is data-independent), with the
candidate count and the HBM bytes the call moves.  Run it under
`ncu --metrics gpu__time_duration.sum` to split the call into its launches.

    python tools/tuneprof.py [--workloads c1,c2,c3,c4] [--reps 3]
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
# training sets of bench.py: 10 frames (2 of 4096^2 for c4)
TRAIN = {"c1": (10, 512, 512, "gauss3", "mre"), "c2": (10, 4096, 4096, "mean5", "mre"),
         "c3": (10, 2160, 3840, "sep7", "l2"), "c4": (2, 4096, 4096, "conv9", "l2")}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workloads", default="c1,c2,c3,c4")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    stream = torch.cuda.current_stream()
    for wl in args.workloads.split(","):
        n, h, w, fname, metric = TRAIN[wl]
        kind, wt = F.named(fname)
        f = P.Filter(wy=wt[0], wx=wt[1]) if kind == "sep" else P.Filter(wt)
        x = torch.randint(16, 236, (n, h, w), device=dev).float()
        P.tune_partials(x, f, metric)  # warm (plans, kernels, scratch pool)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(args.reps):
            P.tune_partials(x, f, metric)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.reps
        nc = len(P.tune_candidates(f))
        px = n * h * w
        print(json.dumps({"wl": wl, "frames": n, "h": h, "w": w, "candidates": nc, "ms": round(ms, 4),
                          "px_per_s": px * (1 + nc) / (ms * 1e-3),
                          "training_px_per_s": px / (ms * 1e-3),
                          "unfused_equiv_gbs": 8.0 * px * (1 + nc) / (ms * 1e-3) / 1e9}), flush=True)


if __name__ == "__main__":
    main()
