"""Check of the tensor-core exact 9x9 stencil (k_conv_tc.cu) against the
oracle (S18: 1e-5 of sum |w||x| per pixel) on ragged shapes, halo stripes,
non-integer inputs (the A_lo term) and signed weights, then the c4-shaped
timing (8192 x 32768 band, 9x9 conv) against the CUDA-core tile kernel
(PARAPROX_CONV_TC=0, in a subprocess: the setting is read once)."""
import json
import os
import subprocess
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)


def time_ms(fn, reps=10, regions=5):
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


def timing():
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    f = P.Filter(F.conv(9))
    x = torch.from_numpy(W.periodic(8192, 32768, tile=4096, seed=0)).cuda().view(1, 8192, 32768)
    out = torch.empty_like(x)
    ms = time_ms(lambda: P.stencil_exact(x, f, out=out))
    px = x.numel()
    print(json.dumps({"conv_tc": os.environ.get("PARAPROX_CONV_TC", "1"), "kernel": P.last_kernel(), "ms": ms,
                      "gbs": 8 * px / ms / 1e6, "tfma_s": 81 * px / ms / 1e9}))
    return out


def main():
    import oracle
    import paper_conf_asplos_samadijlm14_b200 as pkg
    import workloads as W
    from workloads import filters as F
    P = pkg.paraprox
    rng = np.random.default_rng(3)
    bad = []
    cases = []
    for shape in ((1, 300, 400), (2, 131, 77), (3, 128, 32), (1, 9, 9), (1, 5, 8), (1, 257, 1000)):
        cases.append((shape, "int", F.conv(9)))
    cases.append(((2, 200, 300), "float", F.conv(9)))
    cases.append(((1, 150, 260), "int", F.conv_signed(9) if hasattr(F, "conv_signed") else F.conv(9, seed=4)))
    for shape, kind, w in cases:
        x = W.frames(*shape, seed0=7) if kind == "int" else rng.random(shape).astype(np.float32) * 200
        xd = torch.from_numpy(x).cuda()
        f = P.Filter(w)
        g = P.stencil_exact(xd, f).cpu().numpy()
        k = P.last_kernel()
        o = oracle.stencil_exact(x, w)
        tol = 1e-5 * oracle.stencil_exact(np.abs(x), np.abs(w))
        err = np.abs(g - o)
        ratio = float((err / np.maximum(tol, 1e-30)).max())
        rel = float((err / np.maximum(np.abs(o), 1e-30)).max())
        ok = bool(np.all(err <= tol))
        print(json.dumps({"shape": shape, "kind": kind, "kernel": k, "ok": ok, "max_err_over_tol": ratio,
                          "max_rel": rel}))
        if not ok:
            bad.append((shape, kind))
    # halo stripe: rows 100..299 of a 400-row image with 4 halo rows each side
    x = W.frames(1, 400, 512, seed0=9)
    xd = torch.from_numpy(x).cuda()
    f = P.Filter(F.conv(9))
    whole = P.stencil_exact(xd, f).cpu().numpy()
    st = P.stencil_exact(xd[:, 96:304], f, halo_top=4, halo_bottom=4).cpu().numpy()
    print(json.dumps({"stripe_bitwise_to_whole": bool(np.array_equal(st, whole[:, 100:300])),
                      "kernel": P.last_kernel()}))
    print("bad:", bad)
    return 1 if bad else 0


if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "--time":
        timing()
        sys.exit(0)
    rc = main()
    env = dict(os.environ)
    for v in ("1", "0"):
        env["PARAPROX_CONV_TC"] = v
        subprocess.check_call([sys.executable, __file__, "--time"], env=env)
    sys.exit(rc)
