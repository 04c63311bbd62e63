"""HBM context for the roofline fractions: read-only, write-only and copy
bandwidth of torch's own kernels on 1 GiB (CUDA events, best of 10).  The
measured copy figure of MEASURED_PEAKS.json is the roofline peak; a kernel
that mostly writes (the lattice: 0.44 B/px read, 4 B/px written) is bounded by
the write figure, a read-only one (quality) by the read figure."""
import json

import torch


def best(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return min(ts)


def main():
    n = 1 << 28  # 1 GiB of fp32
    a = torch.rand(n, device="cuda")
    b = torch.empty_like(a)
    out = torch.empty(1, device="cuda")
    t_read = best(lambda: torch.sum(a, dim=0, out=out[0]))
    t_write = best(lambda: b.fill_(1.5))
    t_copy = best(lambda: b.copy_(a))
    gb = n * 4 / 1e9
    print(json.dumps({"read_only_gbs": gb / (t_read * 1e-3), "write_only_gbs": gb / (t_write * 1e-3),
                      "copy_gbs_read_plus_write": 2 * gb / (t_copy * 1e-3)}))


if __name__ == "__main__":
    main()
