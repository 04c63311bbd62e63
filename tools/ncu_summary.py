"""Summarise ncu captures for profiles/ (run here, on the CPU host).

    python tools/ncu_summary.py launches gpurun_out/launches_c2.csv > profiles/r01_launches_c2.md
    python tools/ncu_summary.py full gpurun_out/prof_c2.ncu-rep --workload c2 \
        --traffic profiles/traffic.json > profiles/r01_ncu_full_c2.md
    python tools/ncu_summary.py bytes gpurun_out/ncu_bytes_c2.csv gpurun_out/ncu_bytes_c4.csv \
        > profiles/r01_ncu_bytes.md
"""
import argparse
import csv
import io
import json
import os
import re
import subprocess
from collections import defaultdict

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_%peak"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_%"),
    ("smsp__inst_executed.sum", "warp_inst"),
    ("sm__sass_thread_inst_executed_op_ffma_pred_on.sum", "ffma_thread_inst"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem_wavefronts"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__occupancy_limit_shared_mem", "occ_limit_smem"),
]

UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
              "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}


SETS = {256: "s0", 896: "f1", 1984: "f2", 4064: "f3", 8176: "f4", 1344: "l2", 2336: "l3", 4368: "l4", 131071: "f8"}


def short(name):
    """ncu kernel name -> the library's kernel name (paraprox_last_kernel())."""
    m = re.match(r"void (?:ppx::)?k_tiles<(\d+), (\d+), (\d+)u?, (\d+)u?, (\d|true|false)(?:, (\d|true|false))?>", name)
    if m:
        sep = m.group(5) in ("1", "true")
        return f"{'sep' if sep else 'dense'}_{SETS.get(int(m.group(3)), m.group(3))}_{SETS.get(int(m.group(4)), m.group(4))}"
    m = re.match(r"void (?:ppx::)?k_pointwise_(flat|rows)<(\d|true|false)>", name)
    if m:
        kind = "sep" if m.group(2) in ("1", "true") else "dense"
        return f"{kind}_map" + ("_rows" if m.group(1) == "rows" else "")
    m = re.match(r"void (?:ppx::)?k_lattice<(\d+), (\d+), (\d|true|false)>", name)
    if m:
        kind = "sep" if m.group(3) in ("1", "true") else "dense"
        return f"lattice_{kind}_s{m.group(1)}_r{m.group(2)}"
    m = re.match(r"void (?:ppx::)?(\w+)(<[^>]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else name[:70]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = defaultdict(lambda: [0, 0.0])
    order = []
    for r in rows[hdr + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", "")) * UNIT_SCALE.get(r[ui], 1e-9)
        k = short(r[ki])
        agg[k][0] += 1
        agg[k][1] += v
        order.append((k, v))
    tot = sum(t for _, t in agg.values())
    print(f"# ncu launch list: {os.path.basename(path)}\n")
    print("`ncu --metrics gpu__time_duration.sum --clock-control none` over the bench command (cold-cache, serialised:"
          " compare shares, not absolutes).\n")
    print(f"{len(order)} launches, {tot * 1e3:.3f} ms total\n")
    print("| kernel | launches | total us | mean us | share |")
    print("|---|---:|---:|---:|---:|")
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"| `{k}` | {n} | {t * 1e6:.1f} | {t * 1e6 / n:.1f} | {100 * t / tot:.1f}% |")


def full(path, workload, traffic_json):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    idx = {m: h.index(m) for m, _ in METRICS if m in h}
    ki = h.index("Kernel Name")
    print(f"# ncu --set full summary: {os.path.basename(path)} (workload {workload})\n")
    print("| kernel | " + " | ".join(lbl for m, lbl in METRICS if m in idx) + " |")
    print("|---|" + "---:|" * len(idx))
    traffic = {}
    for r in rows[2:]:
        vals = []
        for m, lbl in METRICS:
            if m not in idx:
                continue
            vals.append(r[idx[m]])
        print(f"| `{short(r[ki])}` | " + " | ".join(vals) + " |")
        if "dram__bytes_read.sum" in idx:
            scale = UNIT_SCALE.get(units[idx["dram__bytes_read.sum"]], 1)
            b = (float(r[idx["dram__bytes_read.sum"]].replace(",", "")) +
                 float(r[idx["dram__bytes_write.sum"]].replace(",", ""))) * scale
            traffic.setdefault(short(r[ki]), []).append(b)
    print("\nunits: " + ", ".join(f"{lbl}={units[idx[m]]}" for m, lbl in METRICS if m in idx))
    if traffic_json:
        d = json.load(open(traffic_json)) if os.path.exists(traffic_json) else {}
        d.setdefault(workload, {})
        for k, v in traffic.items():
            d[workload][k] = sum(v) / len(v)
        json.dump(d, open(traffic_json, "w"), indent=1, sort_keys=True)


PIXELS = {"c2": 4096 * 4096, "c4": 32768 * 32768}


def bytes_table(paths):
    """DRAM bytes per launch (ncu --metrics dram__bytes_*) against the
    algorithmic bytes: 8 B/px for the stencils, 4/s + 4 B/px for the row
    lattice of stride s (only every s-th row is read)."""
    print("# DRAM bytes: exact vs per-window approximation vs row lattice (NEXT-1)\n")
    print("`tools/ncu_bytes.sh`: `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum "
          "--clock-control none` (L2 flushed before every kernel), one launch each on the bench's input. "
          "`alg` = algorithmic bytes per pixel; `measured` = (read + write) / pixels.\n")
    print("| workload | kernel | read MB | write MB | measured B/px | alg B/px | measured / alg | vs exact | us (cold) |")
    print("|---|---|---:|---:|---:|---:|---:|---:|---:|")
    for path in paths:
        wl = re.search(r"(c\d)", os.path.basename(path)).group(1)
        rows = list(csv.reader(open(path)))
        hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[hdr]
        ii, ki, mi, ui, vi = (h.index("ID"), h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Unit"),
                              h.index("Metric Value"))
        launches = {}
        for r in rows[hdr + 1:]:
            if len(r) <= vi:
                continue
            d = launches.setdefault(r[ii], {"kernel": short(r[ki])})
            d[r[mi]] = float(r[vi].replace(",", "")) * UNIT_SCALE.get(r[ui], 1)
        exact_b = None
        for _, d in sorted(launches.items(), key=lambda x: int(x[0])):
            b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
            px = PIXELS[wl]
            m = re.match(r"lattice_\w+_s(\d+)_r\d+", d["kernel"])
            alg = 4.0 / int(m.group(1)) + 4.0 if m else 8.0
            if exact_b is None:
                exact_b = b
            t = d.get("gpu__time_duration.sum", 0.0)
            t_us = t * 1e6 if t < 1 else t / 1e3
            print(f"| {wl} | `{d['kernel']}` | {d.get('dram__bytes_read.sum', 0) / 1e6:.1f} | "
                  f"{d.get('dram__bytes_write.sum', 0) / 1e6:.1f} | {b / px:.3f} | {alg:.3f} | {b / px / alg:.3f} | "
                  f"{b / exact_b:.3f} | {t_us:.1f} |")


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("kind", choices=["launches", "full", "bytes"])
    ap.add_argument("path", nargs="+")
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--traffic", default=None)
    a = ap.parse_args()
    if a.kind == "launches":
        launches(a.path[0])
    elif a.kind == "bytes":
        bytes_table(a.path)
    else:
        full(a.path[0], a.workload, a.traffic)
