"""NEXT-4 measurement: HotSpot (Table 1: 1024x1024,
Stencil-Partition, MRE) iterated with every scheme.  For each grid size and
scheme: the time of `iterations` steps (one paraprox_hotspot call, captured in
a CUDA graph and replayed, CUDA events), the per-step HBM figure (12 B/px:
read T and P, write T), the MRE quality against the exact iteration, and the
speedup.  The centre scheme at full reach reads no neighbour, so its steps fuse
into one pass (k_pointwise): 12 B/px for all the steps.

    python tools/hotspot.py [--out gpurun_out/hotspot.json]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import hotspot as H  # noqa: E402

P = pkg.paraprox


def graph_ms(fn, reps=10):
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        fn()
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "hotspot.json"))
    args = ap.parse_args()
    rows = []
    for n, side, iters in ((1, 1024, 100), (1, 8192, 20)):
        t, p = H.frames(n, side, side, 11)
        td, pd = torch.from_numpy(t).cuda(), torch.from_numpy(p).cuda()
        out = torch.empty_like(td)
        exact = P.hotspot(td, pd, H.PARAMS, "exact", 0, iters).clone()
        res = {}
        for scheme, reach in (("exact", 0), ("row", 1), ("col", 1), ("center", 1)):
            ms = graph_ms(lambda: P.hotspot(td, pd, H.PARAMS, scheme, reach, iters, out=out))
            kern = P.last_kernel()
            # unblocked: one paraprox_hotspot call (one tile-kernel pass) per step
            bufs = (out, torch.empty_like(td))

            def per_step():
                src = td
                for k in range(iters):
                    P.hotspot(src, pd, H.PARAMS, scheme, reach, 1, out=bufs[k % 2])
                    src = bufs[k % 2]
            ms1 = graph_ms(per_step)
            kern1 = P.last_kernel()
            q = 1.0 if scheme == "exact" else P.quality(exact, P.hotspot(td, pd, H.PARAMS, scheme, reach, iters), "mre")
            px = td.numel()
            passes = 1 if scheme == "center" else -(-iters // 8)  # k_hotspot_tb: 8 steps per pass
            res[scheme] = ms
            row = {"grid": f"{side}x{side}", "iterations": iters, "scheme": scheme, "kernel": kern, "ms": ms,
                   "us_per_step": 1e3 * ms / iters, "quality_mre": q, "hbm_passes": passes,
                   "algorithmic_gbs": 12.0 * px * passes / (ms * 1e-3) / 1e9,
                   "speedup_vs_exact": res["exact"] / ms,
                   "unblocked_kernel": kern1, "unblocked_us_per_step": 1e3 * ms1 / iters,
                   "unblocked_gbs": 12.0 * px * iters / (ms1 * 1e-3) / 1e9, "blocked_speedup": ms1 / ms}
            print(json.dumps(row), flush=True)
            rows.append(row)
        del td, pd, out, exact
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(rows, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
