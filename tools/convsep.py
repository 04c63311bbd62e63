"""NEXT-3 measurement: the paper's Convolution Separable workload (2048^2,
two 1x17 loops, L2-norm; Table 1) with the
stencil approximation, the reduction approximation and both, as the paper
compares them ("stencil optimization 1.7x at 90 %", "reduction 1.6x").

For each TOQ and each candidate family (flags 1 = stencil, 2 = reduction,
3 = both) the library's extended tuner trains on 10 seeded frames; the chosen
kernel is timed on 16 held-out frames (CUDA events, buffers > L2) against the
exact fused separable kernel, its held-out quality measured, and the oracle
tuner's decision on a 2-frame subset compared with the GPU tuner's on the
same subset.

    python tools/convsep.py [--out gpurun_out/convsep.json]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (decision check only)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
FAMILY = {1: "stencil", 2: "reduction", 3: "stencil+reduction"}


def time_ms(fn, reps=20):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "convsep.json"))
    args = ap.parse_args()
    wy, wx = F.separable(17, seed_y=17, seed_x=71)
    f = P.Filter(wy=wy, wx=wx)
    train_np = W.frames(10, 2048, 2048, 0)
    held_np = W.frames(16, 2048, 2048, 10)
    train = torch.from_numpy(train_np).cuda()
    held = torch.from_numpy(held_np).cuda()
    out = torch.empty_like(held)
    exact = P.stencil_exact(held, f)
    ex_ms = time_ms(lambda: P.stencil_exact(held, f, out=out))
    px = held.numel()
    rows = []
    for toq in (0.80, 0.90, 0.95):
        for flags in (1, 2, 3):
            scheme, rate, q_train = P.tune_ex(train, f, toq, "l2", flags)
            g_sub = P.tune_ex(train[:2], f, toq, "l2", flags)
            o_sub = oracle.tune_ex(train_np[:2], (wy, wx), toq, "l2", flags=flags)
            row = {"toq": toq, "family": FAMILY[flags], "scheme": scheme, "rate_or_reach": rate, "q_train": q_train,
                   "exact_us": 1e3 * ex_ms, "decision_identical": g_sub[:2] == (o_sub["scheme"], o_sub["reach"]),
                   "gpu_subset": list(g_sub[:2]), "oracle_subset": [o_sub["scheme"], o_sub["reach"]]}
            if scheme == "exact":
                row.update(kernel="exact", approx_us=1e3 * ex_ms, speedup=1.0, q_heldout=1.0)
            else:
                a = P.stencil_approx(held, f, scheme, rate, out=out)
                row["kernel"] = P.last_kernel()
                row["q_heldout"] = P.quality(exact, a, "l2")
                ms = time_ms(lambda: P.stencil_approx(held, f, scheme, rate, out=out))
                row.update(approx_us=1e3 * ms, speedup=ex_ms / ms, gbs=8.0 * px / ms / 1e6)
            print(json.dumps(row), flush=True)
            rows.append(row)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(rows, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
