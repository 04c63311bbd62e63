"""Config c5 (BASELINE.json configs[4]): runtime TOQ sweep 80/90/95/99 % with
paraprox_tune selecting scheme and reach on the Gaussian, mean, 9x9 conv and
7x7 separable workloads.

Protocol: train on the first 10 seeded frames, then
measure the held-out frames.  For every filter x TOQ it reports the tuned
(scheme, reach), the training quality, the held-out quality (pooled, mean and
min per frame), the Fig. 13 analogue (share of output pixels whose relative
error is below 10 %), and the measured approx/exact speedup of
the chosen kernel on the held-out batch (CUDA events, buffers > L2).  The
oracle tuner runs on a training subset (the full 10 frames at 512^2, 2 frames
at the larger sizes) together with the GPU tuner on the same subset, and the
two decisions must be identical.

    python tools/toq_sweep.py [--out gpurun_out/toq_sweep.json] [--quick]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (test infrastructure: the decision check only)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
TOQS = (0.80, 0.90, 0.95, 0.99)
CASES = [
    # name, filter, metric, h, w, held-out frames, oracle-subset frames
    ("gauss3@512", "gauss3", "mre", 512, 512, 100, 10),
    ("mean5@4096", "mean5", "mre", 4096, 4096, 20, 2),
    ("conv9@4096", "conv9", "l2", 4096, 4096, 20, 2),
    ("sep7@3840x2160", "sep7", "l2", 2160, 3840, 20, 2),
]


def time_ms(fn, reps=10):
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
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "toq_sweep.json"))
    ap.add_argument("--quick", action="store_true", help="fewer held-out frames")
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    rows = []
    for name, fname, metric, h, w, nheld, nsub in CASES:
        if args.quick:
            nheld = min(nheld, 4)
        kind, wt = F.named(fname)
        f = P.Filter(wy=wt[0], wx=wt[1]) if kind == "sep" else P.Filter(wt)
        t0 = time.perf_counter()
        train_np = W.frames(10, h, w, 0)
        held_np = W.frames(nheld, h, w, 10)
        gen_s = time.perf_counter() - t0
        train = torch.from_numpy(train_np).to(dev)
        held = torch.from_numpy(held_np).to(dev)
        exact = P.stencil_exact(held, f)
        out = torch.empty_like(held)
        ex_ms = time_ms(lambda: P.stencil_exact(held, f, out=out))
        sub = train_np[:nsub]
        sub_d = train[:nsub]
        for toq in TOQS:
            t1 = time.perf_counter()
            scheme, reach, q_train = P.tune(train, f, toq, metric)
            tune_ms = 1e3 * (time.perf_counter() - t1)
            # decision check against the oracle tuner on the same subset
            g_sub = P.tune(sub_d, f, toq, metric)
            t2 = time.perf_counter()
            o_sub = oracle.tune(sub, wt, toq, metric)
            oracle_s = time.perf_counter() - t2
            same = g_sub[:2] == (o_sub["scheme"], o_sub["reach"])
            row = {"case": name, "metric": metric, "toq": toq, "scheme": scheme, "reach": reach,
                   "q_train": q_train, "tune_ms": tune_ms, "train_frames": 10, "heldout_frames": nheld,
                   "oracle_subset_frames": nsub, "gpu_subset": list(g_sub[:2]),
                   "oracle_subset": [o_sub["scheme"], o_sub["reach"]], "decision_identical": same,
                   "oracle_tune_s": oracle_s, "gen_s": gen_s}
            if scheme == "exact":
                row.update(q_heldout=1.0, q_heldout_min=1.0, fig13_lt10=1.0, speedup=1.0, exact_us=1e3 * ex_ms,
                           approx_us=1e3 * ex_ms)
            else:
                approx = P.stencil_approx(held, f, scheme, reach)
                row["q_heldout"] = P.quality(exact, approx, metric)
                per = [P.quality(exact[k:k + 1], approx[k:k + 1], metric) for k in range(nheld)]
                row["q_heldout_mean"] = float(np.mean(per))
                row["q_heldout_min"] = float(np.min(per))
                e = exact.cpu().numpy().astype(np.float64)
                a = approx.cpu().numpy().astype(np.float64)
                rel = np.abs(a - e) / np.maximum(np.abs(e), 1e-30)
                row["fig13_lt10"] = float(np.mean(rel < 0.10))
                ap_ms = time_ms(lambda: P.stencil_approx(held, f, scheme, reach, out=out))
                row.update(speedup=ex_ms / ap_ms, exact_us=1e3 * ex_ms, approx_us=1e3 * ap_ms)
                del approx
            print(json.dumps(row), flush=True)
            rows.append(row)
        del train, held, exact, out
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(rows, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
