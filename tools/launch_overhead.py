"""Fixed cost per launch vs steady-state cost per frame of the tile kernels:
time one launch over n = 1, 2, 4, 8, 16 frames of 4096^2 (5x5 mean: exact,
row 2, the centre map) and fit t(n) = t0 + n t1 (CUDA graphs of back-to-back
launches on rotating buffers larger than L2).  t0 is what a single-frame
launch (c2) pays on top of the streaming rate t1.

    python tools/launch_overhead.py [--out gpurun_out/launch_overhead.json]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox


def graph_time(make_ops, reps=40):
    s = torch.cuda.Stream()
    ops = make_ops(s)
    with torch.cuda.stream(s):
        for op in ops:
            op()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for k in range(reps):
            ops[k % len(ops)]()
    g.replay()
    torch.cuda.synchronize()
    best = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        best.append(e0.elapsed_time(e1) / reps)
    return float(np.median(best))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "launch_overhead.json"))
    ap.add_argument("--side", type=int, default=4096)
    args = ap.parse_args()
    f = P.Filter(F.mean(5))
    base = torch.from_numpy(W.image(args.side, args.side, 0)).cuda()
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6548.2
    rows = []
    for scheme, reach in (("exact", 0), ("row", 2), ("center", 2)):
        pts = []
        for n in (1, 2, 4, 8, 16):
            px = n * args.side * args.side
            nbuf = max(2, -(-(3 * 126 * 2 ** 20) // (8 * px)))
            ins = [base.expand(n, -1, -1).contiguous() for _ in range(nbuf)]
            outs = [torch.empty_like(ins[0]) for _ in range(nbuf)]
            ms = graph_time(lambda st: [P.Prepared(ins[k], f, scheme, reach, outs[k], stream=st)
                                        for k in range(nbuf)])
            kern = P.last_kernel()
            pts.append((n, ms))
            rows.append({"scheme": scheme, "reach": reach, "kernel": kern, "frames": n, "us": 1e3 * ms,
                         "frac": 8.0 * px / (ms * 1e-3) / 1e9 / peak})
            print(json.dumps(rows[-1]), flush=True)
            del ins, outs
        n_, t_ = np.array([p[0] for p in pts], float), np.array([p[1] for p in pts])
        t1, t0 = np.polyfit(n_, t_, 1)
        fit = {"scheme": scheme, "kernel": kern, "fixed_us_per_launch": 1e3 * t0, "us_per_frame": 1e3 * t1,
               "steady_frac": 8.0 * args.side ** 2 / (t1 * 1e-3) / 1e9 / peak}
        rows.append(fit)
        print(json.dumps(fit), flush=True)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(rows, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
