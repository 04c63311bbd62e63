"""Time the map kernel (centre full collapse) and the exact 5x5 at c2 / c4
shapes for A/B of build variants (PARAPROX_LIB)."""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox


def t(fn, nbuf, reps=30):
    for k in range(3):
        fn(k % nbuf)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for k in range(reps):
        fn(k % nbuf)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for name, shape, nbuf in (("c2", (1, 4096, 4096), 3), ("c4", (1, 16384, 16384), 1), ("c4full", (1, 32768, 32768), 1)):
    ins = [torch.rand(shape, device="cuda") for _ in range(nbuf)]
    outs = [torch.empty_like(ins[0]) for _ in range(nbuf)]
    f = P.Filter(F.mean(5))
    res = {"lib": os.environ.get("PARAPROX_LIB", "default"), "wl": name}
    for sch, r in (("center", 2), ("exact", 0)):
        ops = [P.Prepared(ins[k], f, sch, r, outs[k]) for k in range(nbuf)]
        ms = t(lambda k: ops[k](), nbuf)
        res[sch + "_us"] = round(1e3 * ms, 2)
        res[sch + "_gbs"] = round(8 * ins[0].numel() / ms / 1e6, 1)
    print(json.dumps(res), flush=True)
    del ins, outs
    torch.cuda.empty_cache()
