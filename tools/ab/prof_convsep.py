"""Launch the ConvSep exact stencil (16 x 2048^2, 1x17 + 17x1) a few times
for ncu captures:  python tools/ab/prof_convsep.py [reps] [dy dx]"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
import workloads as W  # noqa: E402
from workloads import filters as F  # noqa: E402

P = pkg.paraprox
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
dy, dx = (int(sys.argv[2]), int(sys.argv[3])) if len(sys.argv) > 3 else (0, 0)
wy, wx = F.separable(17, seed_y=17, seed_x=71)
f = P.Filter(wy=wy, wx=wx)
x = torch.from_numpy(W.frames(16, 2048, 2048, 10)).cuda()
out = torch.empty_like(x)
for _ in range(reps):
    P.stencil_approx_xy(x, f, dy, dx, out=out)
torch.cuda.synchronize()
print(P.last_kernel())
