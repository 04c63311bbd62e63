"""A/B of the column-strip streaming kernel (tools/ab/k_sepstream_ab.cu.txt,
copied into csrc/ as k_sepstream.cu with its dispatch hook and the
PARAPROX_SEP_STREAM knob; not in the product build: slower)
against the tile kernels' wide separable path: bitwise identity on
ragged shapes, halo stripes and pitched layouts, and the ConvSep timing
(16 x 2048^2, 1x17 + 17x1) of both.  Each side runs in its own process (the
setting is read once per process)."""
import json
import os
import subprocess
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def time_ms(fn, reps=20, regions=5):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(regions):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / reps)
    return float(np.median(ts))


def run(out_path):
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    res, kern = {}, {}
    wy17, wx17 = F.separable(17, seed_y=17, seed_x=71)
    filt = {"17x17": P.Filter(wy=wy17, wx=wx17)}
    for shape in ((2, 77, 300), (1, 190, 700), (1, 5, 130), (4, 33, 129), (1, 1, 17), (3, 601, 2048),
                  (2, 2048, 2048)):
        x = torch.from_numpy(W.frames(*shape, seed0=4)).cuda()
        for name, f in filt.items():
            for dy, dx in ((0, 0), (3, 3), (8, 0), (0, 8), (1, 2)):
                o = P.stencil_approx_xy(x, f, dy, dx)
                key = f"{shape}_{name}_{dy}_{dx}"
                res[key] = o.cpu().numpy()
                kern[key] = P.last_kernel()
    # halo stripe (rows 100..299 of a 400-row image, 8 halo rows each side)
    x = torch.from_numpy(W.frames(1, 400, 500, seed0=9)).cuda()
    o = P.stencil_exact(x[:, 92:308], filt["17x17"], halo_top=8, halo_bottom=8)
    res["stripe"] = o.cpu().numpy()
    kern["stripe"] = P.last_kernel()
    # pitched layout: a 300-column view of 512-column rows
    xb = torch.from_numpy(W.frames(2, 200, 512, seed0=11)).cuda()
    ob = torch.zeros_like(xb)
    o = P.stencil_exact(xb[:, :, 8:308], filt["17x17"], out=ob[:, :, 8:308])
    res["pitched"] = o.cpu().numpy()
    kern["pitched"] = P.last_kernel()
    held = torch.from_numpy(W.frames(16, 2048, 2048, 10)).cuda()
    out = torch.empty_like(held)
    t = {}
    for dy, dx in ((0, 0), (5, 5)):
        t[f"{dy}_{dx}"] = 1e3 * time_ms(lambda: P.stencil_approx_xy(held, filt["17x17"], dy, dx, out=out))
        t[f"{dy}_{dx}_kernel"] = P.last_kernel()
    np.savez(out_path, **res)
    print(json.dumps({"kernels": {k: kern[k] for k in list(kern)[:6]}, "stripe": kern["stripe"],
                      "pitched": kern["pitched"], "convsep_us": t}))


def time_only():
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    wy17, wx17 = F.separable(17, seed_y=17, seed_x=71)
    f = P.Filter(wy=wy17, wx=wx17)
    held = torch.from_numpy(W.frames(16, 2048, 2048, 10)).cuda()
    out = torch.empty_like(held)
    us = 1e3 * time_ms(lambda: P.stencil_exact(held, f, out=out))
    print(json.dumps({"env": {k: v for k, v in os.environ.items() if k.startswith(("PPX_", "PARAPROX_"))},
                      "kernel": P.last_kernel(), "convsep_exact_us": us}))


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--time":
        time_only()
        sys.exit(0)
    if len(sys.argv) > 1:
        run(sys.argv[1])
        sys.exit(0)
    env = dict(os.environ)
    env["PARAPROX_SEP_STREAM"] = "1"
    subprocess.check_call([sys.executable, __file__, "/tmp/ss_new.npz"], env=env)
    env["PARAPROX_SEP_STREAM"] = "0"
    subprocess.check_call([sys.executable, __file__, "/tmp/ss_old.npz"], env=env)
    a, b = np.load("/tmp/ss_new.npz"), np.load("/tmp/ss_old.npz")
    bad = [k for k in a.files if not np.array_equal(a[k], b[k])]
    for k in bad[:5]:
        d = np.abs(a[k].astype(np.float64) - b[k])
        print(k, "max diff", d.max(), "at", np.unravel_index(d.argmax(), d.shape), "n bad", int((d > 0).sum()))
    print(f"sepstream bitwise: {len(a.files) - len(bad)}/{len(a.files)} identical", bad[:8])
    sys.exit(1 if bad else 0)
