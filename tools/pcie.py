"""PCIe context for the e2e number: pinned H2D alone, D2H alone, both at once
(two streams), and paraprox_run_host on the same bytes (c2: 4096^2 fp32)."""
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox


def wall(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


def main():
    for mb in (64, 256, 1024):
        n = mb * 2**20 // 4
        h = torch.empty(n, pin_memory=True).uniform_()
        ho = torch.empty(n, pin_memory=True)
        d = torch.empty(n, device="cuda")
        d2 = torch.empty(n, device="cuda")
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

        def h2d():
            d.copy_(h, non_blocking=True)

        def d2h():
            ho.copy_(d2, non_blocking=True)

        def both():
            with torch.cuda.stream(s1):
                d.copy_(h, non_blocking=True)
            with torch.cuda.stream(s2):
                ho.copy_(d2, non_blocking=True)

        t_up, t_dn, t_both = wall(h2d), wall(d2h), wall(both)
        side = int(round((n) ** 0.5))
        x = h[: side * side].view(1, side, side)
        o = ho[: side * side].view(1, side, side)
        f = P.Filter(F.mean(5))
        t_run = wall(lambda: P.run_host(x, f, "center", 2, out=o))
        print(json.dumps({"MiB": mb, "h2d_gbs": n * 4 / t_up / 1e9, "d2h_gbs": n * 4 / t_dn / 1e9,
                          "both_gbs_each": n * 4 / t_both / 1e9, "run_host_ms": 1e3 * t_run,
                          "run_host_gbs_each_way": side * side * 4 / t_run / 1e9,
                          "ideal_duplex_ms": 1e3 * t_both}), flush=True)


if __name__ == "__main__":
    main()
