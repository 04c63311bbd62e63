"""Time one stencil under several environment settings (one subprocess per
setting; the library reads its settings once).

    python tools/ab/env_sweep.py c4exact 'PARAPROX_TMA_STORE=0' 'PARAPROX_TILE_CHUNK=16' ...
"""
import json
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

CASES = {
    # name: (n, h, w, filter, dy, dx)
    "c4exact": (1, 16384, 16384, "conv9", 0, 0),
    "c4lat": (1, 16384, 16384, "conv9", "lat", 1),
    "c2exact": (1, 4096, 4096, "mean5", 0, 0),
    "c3exact": (32, 2160, 3840, "sep7", 0, 0),
    "c1exact": (110, 512, 512, "gauss3", 0, 0),
    "convsep": (16, 2048, 2048, "sep17", 0, 0),
}


def run(case):
    import torch

    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    n, h, w, filt, dy, dx = CASES[case]
    if filt == "sep17":
        wy, wx = F.separable(17, seed_y=17, seed_x=71)
        f = P.Filter(wy=wy, wx=wx)
    else:
        kind, wts = F.named(filt)
        f = P.Filter(wy=wts[0], wx=wts[1]) if kind == "sep" else P.Filter(wts)
    nbuf = max(2, int(3 * 126e6 // (8 * n * h * w)) + 1)
    base = torch.from_numpy(W.periodic(h, w, tile=min(4096, h), seed=0) if n == 1 else W.frames(n, h, w, 0)).cuda()
    xs = [base.view(n, h, w).clone() for _ in range(nbuf)]
    outs = [torch.empty_like(xs[0]) for _ in range(nbuf)]
    if dy == "lat":
        fn = lambda k: P.stencil_lattice(xs[k], f, "row", dx, out=outs[k])  # noqa: E731
    else:
        fn = lambda k: P.stencil_approx_xy(xs[k], f, dy, dx, out=outs[k])  # noqa: E731
    for k in range(3):
        fn(k % nbuf)
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for k in range(20):
            fn(k % nbuf)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 20)
    ms = float(np.median(ts))
    print(json.dumps({"case": case, "env": {k: v for k, v in os.environ.items() if k.startswith(("PARAPROX_", "PPX_"))},
                      "kernel": P.last_kernel(), "us": 1e3 * ms, "gbs": 8 * n * h * w / ms / 1e6}), flush=True)


if __name__ == "__main__":
    if sys.argv[1] == "--run":
        run(sys.argv[2])
        sys.exit(0)
    case = sys.argv[1]
    for spec in [""] + sys.argv[2:]:
        env = dict(os.environ)
        for kv in spec.split(","):
            if kv:
                k, v = kv.split("=")
                env[k] = v
        subprocess.call([sys.executable, __file__, "--run", case], env=env)
