"""A/B probe of the lattice kernels' tile schedule: row lattice reach 1 and 4 at
c3, c4 and c2 sizes.  Run once per PARAPROX_LATTICE_CHUNK setting.
"""
import sys, os, json, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_samadijlm14_b200 as pkg
from workloads import filters as F
P = pkg.paraprox
dev = torch.device("cuda", 0); st = torch.cuda.current_stream()
kind, wt = F.named("sep7"); fs = P.Filter(wy=wt[0], wx=wt[1])
fd = P.Filter(F.named("mean5")[1]); fc = P.Filter(F.named("conv9")[1])
def t(f, xs, os_, d, reps=10):
    ops = [P.Prepared(xs[k], f, "row", d, os_[k], stream=st, lattice=True) for k in range(len(xs))]
    for k in range(3): ops[k % len(xs)]()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record(st)
    for k in range(reps): ops[k % len(xs)]()
    e1.record(st); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    px = xs[0].numel()
    return round((4.0 / (2 * d + 1) + 4.0) * px / ms / 1e6, 1)
r = {}
x = [torch.rand((256, 2160, 3840), device=dev) * 200 + 16]; o = [torch.empty_like(x[0])]
r.update({"c3_r4": t(fs, x, o, 4), "c3_r1": t(fs, x, o, 1)}); del x, o
x = [torch.rand((1, 32768, 32768), device=dev) * 200 + 16]; o = [torch.empty_like(x[0])]
r.update({"c4_r4": t(fc, x, o, 4), "c4_r1": t(fc, x, o, 1)}); del x, o
x = [torch.rand((1, 4096, 4096), device=dev) * 200 + 16 for _ in range(4)]; o = [torch.empty_like(x[0]) for _ in range(4)]
r.update({"c2_r4": t(fd, x, o, 4, 200), "c2_r1": t(fd, x, o, 1, 200)})
print(json.dumps(r), flush=True)
