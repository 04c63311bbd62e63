"""Per-kernel pipe / issue / stall table of an ncu --set full report (for
profiles/r02_*.md): duration, DRAM bytes, FMA-pipe and issue activity,
occupancy, and the top warp-stall reasons (share of sampled stalls).

    python tools/ncu_kernels.py gpurun_out/prof_r02a.ncu-rep [...]
"""
import csv
import io
import subprocess
import sys

from ncu_summary import UNIT_SCALE, short

COLS = [
    ("gpu__time_duration.sum", "us", 1e-6),
    ("dram__bytes_read.sum", "DRAM read GB", 1e9),
    ("dram__bytes_write.sum", "DRAM write GB", 1e9),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %", None),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue %", None),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %", None),
    ("smsp__inst_executed.sum", "warp inst (M)", 1e-6),
    ("launch__registers_per_thread", "regs", None),
    ("launch__grid_size", "grid", None),
]


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True,
                         check=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    for row in r[2:]:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        yield d, u


def main():
    print("| kernel | " + " | ".join(c[1] for c in COLS) + " | top stalls (% of samples) |")
    print("|---|" + "---:|" * len(COLS) + "---|")
    for rep in sys.argv[1:]:
        for d, u in rows(rep):
            name = short(d["Kernel Name"])
            vals = []
            for key, label, scale in COLS:
                v = d.get(key, "")
                try:
                    x = float(v.replace(",", ""))
                except ValueError:
                    vals.append("–")
                    continue
                if scale == 1e-6 and label == "us":
                    x = x * UNIT_SCALE.get(u.get(key, "ns"), 1e-9) / 1e-6
                elif scale == 1e9:
                    x = x * UNIT_SCALE.get(u.get(key, "byte"), 1) / 1e9
                elif scale == 1e-6:
                    x = x * 1e-6
                vals.append(f"{x:.3g}" if abs(x) < 1000 else f"{x:.0f}")
            st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v) for k, v in d.items()
                  if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
                  and v not in ("", "n/a")}
            tot = sum(st.values()) or 1.0
            top = ", ".join(f"{k} {100 * v / tot:.0f}" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:5])
            print(f"| `{name}` | " + " | ".join(vals) + f" | {top} |")


if __name__ == "__main__":
    main()
