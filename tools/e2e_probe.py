"""A/B probe of paraprox_run_host (the e2e path): Mpixel/s over pinned host
buffers at c2 (1 x 4096^2) and c1 (110 x 512^2), beside the pinned H2D + D2H
duplex bound measured in the same process.  PARAPROX_LIB selects the library."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
res = {}
for name, shape, w, scheme, d in (("c2", (1, 4096, 4096), F.mean(5), "center", 2),
                                  ("c1", (110, 512, 512), F.gaussian(3), "center", 1),
                                  ("c2_exact", (1, 4096, 4096), F.mean(5), "exact", 0)):
    f = P.Filter(w)
    x = (torch.rand(shape) * 200 + 16).pin_memory()
    o = torch.empty_like(x).pin_memory()
    xx = x[0] if shape[0] == 1 else x
    oo = o[0] if shape[0] == 1 else o
    for _ in range(3):
        P.run_host(xx, f, scheme, d, out=oo)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(40):
        P.run_host(xx, f, scheme, d, out=oo)
    dt = (time.perf_counter() - t0) / 40
    n = x.numel()
    db, db2 = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
    hb = torch.empty(n, pin_memory=True)
    su, sd = torch.cuda.Stream(), torch.cuda.Stream()

    def duplex():
        with torch.cuda.stream(su):
            db.copy_(x.view(-1), non_blocking=True)
        with torch.cuda.stream(sd):
            hb.copy_(db2, non_blocking=True)
        torch.cuda.synchronize()
    duplex()
    t0 = time.perf_counter()
    for _ in range(20):
        duplex()
    bound = n / ((time.perf_counter() - t0) / 20) / 1e6
    res[name] = {"mpx_s": round(n / dt / 1e6), "bound_mpx_s": round(bound), "frac": round(n / dt / 1e6 / bound, 3)}
print(json.dumps(res))
