"""Launch HotSpot exact steps on 8192^2 (k_hotspot_tb) for ncu captures."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_asplos_samadijlm14_b200 as pkg  # noqa: E402
from workloads import hotspot as H  # noqa: E402

P = pkg.paraprox
t, p = H.frames(1, 8192, 8192, 0)
td, pd = torch.from_numpy(t).cuda(), torch.from_numpy(p).cuda()
out = P.hotspot(td, pd, H.PARAMS, "exact", 0, 16)
torch.cuda.synchronize()
print(P.last_kernel())
