"""A/B probe of the tile schedule (bounded persistence): exact and approximate
stencils at c3 (256 x 2160 x 3840), c4 (32768^2) and c2 sizes, GB/s of
algorithmic bytes.  Run once per PARAPROX_TILE_CHUNK setting (read at load).
"""
import sys, os, json, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_samadijlm14_b200 as pkg
from workloads import filters as F
P = pkg.paraprox
dev = torch.device("cuda", 0)
st = torch.cuda.current_stream()
kind, wt = F.named("sep7")
fs = P.Filter(wy=wt[0], wx=wt[1])
fd = P.Filter(F.named("mean5")[1])
fc = P.Filter(F.named("conv9")[1])
def t(f, x, out, scheme="exact", d=0, reps=10):
    op = P.Prepared(x, f, scheme, d, out, stream=st)
    for _ in range(3): op()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record(st)
    for _ in range(reps): op()
    e1.record(st); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    return round(8 * x.numel() / ms / 1e6, 1)
big = torch.rand((256, 2160, 3840), device=dev) * 200 + 16
obig = torch.empty_like(big)
r = {"c3_sep_exact": t(fs, big, obig), "c3_sep_row1": t(fs, big, obig, "row", 1), "c3_mean5_exact": t(fd, big, obig)}
del big, obig
x = torch.rand((1, 32768, 32768), device=dev) * 200 + 16
o = torch.empty_like(x)
r.update({"c4_exact": t(fc, x, o, reps=5), "c4_row4": t(fc, x, o, "row", 4), "c4_center1": t(fc, x, o, "center", 1)})
del x, o
xs = [torch.rand((1, 4096, 4096), device=dev) * 200 + 16 for _ in range(4)]
os_ = [torch.empty_like(xs[0]) for _ in range(4)]
def tc(scheme, d, reps=200):
    ops = [P.Prepared(xs[k], fd, scheme, d, os_[k], stream=st) for k in range(4)]
    for k in range(8): ops[k % 4]()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record(st)
    for k in range(reps): ops[k % 4]()
    e1.record(st); torch.cuda.synchronize()
    return round(8 * xs[0].numel() / (e0.elapsed_time(e1) / reps) / 1e6, 1)
r.update({"c2_exact": tc("exact", 0), "c2_row1": tc("row", 1)})
print(json.dumps(r), flush=True)
