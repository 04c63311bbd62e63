"""Launch the exact 9x9 on an 8192 x 32768 band (c4-shaped) for ncu captures."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
f = P.Filter(F.conv(9))
x = torch.from_numpy(W.periodic(8192, 32768, tile=4096, seed=0)).cuda().view(1, 8192, 32768)
out = torch.empty_like(x)
for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 2):
    P.stencil_exact(x, f, out=out)
torch.cuda.synchronize()
print(P.last_kernel())
