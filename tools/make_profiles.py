"""Copy the round's GPU measurements from gpurun_out/ to profiles/ and
regenerate their Markdown summaries (run here, on the CPU host).

    python tools/make_profiles.py [--round r01]
"""
import argparse
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")


def load(name):
    p = os.path.join(OUT, name)
    return json.load(open(p)) if os.path.exists(p) else None


def toq_md(rows, tag):
    out = [f"# c5: TOQ sweep (BASELINE.json configs[4]) — {tag}", "",
           "`python tools/toq_sweep.py` on one B200. Train on 10 seeded frames (PAPER.md L1620-1628), measure held-out "
           "frames. `q_*` = 1 − error (MRE for Gaussian/mean, L2 for the convolutions). `fig13` = share of output "
           "pixels with relative error < 10 % (Fig. 13 analogue, P:L2086-2090). Speedup = exact / chosen kernel, CUDA "
           "events on the held-out batch (> L2). `oracle` = the oracle tuner's decision on the same training subset "
           "as the GPU tuner (`gpu`).", "",
           "| case | TOQ | chosen | q_train | q_heldout (min/frame) | fig13 | exact µs | approx µs | speedup | gpu "
           "subset | oracle subset | same |", "|---|---:|---|---:|---:|---:|---:|---:|---:|---|---|---|"]
    for r in rows:
        out.append("| %s | %.2f | %s:%d | %.4f | %.4f (%.4f) | %.3f | %.1f | %.1f | %.2f | %s:%d | %s:%d | %s |" % (
            r["case"], r["toq"], r["scheme"], r["reach"], r["q_train"], r["q_heldout"], r.get("q_heldout_min", 1.0),
            r["fig13_lt10"], r["exact_us"], r["approx_us"], r["speedup"], r["gpu_subset"][0], r["gpu_subset"][1],
            r["oracle_subset"][0], r["oracle_subset"][1], "yes" if r["decision_identical"] else "NO"))
    n_same = sum(r["decision_identical"] for r in rows)
    out += ["", f"{n_same}/{len(rows)} decisions identical to the oracle tuner."]
    return "\n".join(out) + "\n"


def convsep_md(rows, tag):
    out = [f"# NEXT-3: Convolution Separable (2048², two 1×17 loops, L2) — stencil vs reduction approximation — {tag}",
           "", "`python tools/convsep.py` on one B200. The paper's workload (PAPER.md Table 1 L1650; results "
           "L1920-1996: stencil optimisation 1.7× and reduction optimisation 1.6× on a GTX 560 at ~90 % quality). "
           "Train on 10 seeded frames, time on 16 held-out 2048² frames (CUDA events, 512 MiB in + out > L2) against "
           "the fused exact separable kernel (`sep8_f8_f8`). `family` = the extended tuner's candidate set (flags 1 "
           "stencil, 2 reduction, 3 both). `oracle = gpu`: the oracle tuner on a 2-frame subset agrees with the GPU "
           "tuner on the same subset.", "",
           "| TOQ | family | chosen | kernel | q_train | q_heldout | exact µs | approx µs | speedup | GB/s | oracle = gpu |",
           "|---:|---|---|---|---:|---:|---:|---:|---:|---:|---|"]
    for r in rows:
        out.append("| %.2f | %s | %s:%d | `%s` | %.4f | %.4f | %.1f | %.1f | %.2f | %s | %s |" % (
            r["toq"], r["family"], r["scheme"], r["rate_or_reach"], r["kernel"], r["q_train"], r["q_heldout"],
            r["exact_us"], r["approx_us"], r["speedup"], "%.0f" % r["gbs"] if "gbs" in r else "-",
            "yes" if r["decision_identical"] else "NO"))
    return "\n".join(out) + "\n"


def hotspot_md(rows, tag):
    out = [f"# NEXT-4: HotSpot (Table 1 L1648: 1024², Stencil-Partition, MRE) — {tag}", "",
           "`python tools/hotspot.py` on one B200: `iterations` steps in one `paraprox_hotspot` call, captured in a "
           "CUDA graph and replayed (CUDA events). Exact, row and column schemes run the temporally blocked kernel "
           "(`hotspot_tb_*`: up to 8 steps per HBM pass, bit-identical to single steps); the centre scheme at full "
           "reach reads no neighbour and fuses all steps into one pass (`dense_map`). quality = 1 − MRE of the final "
           "temperature against the exact iteration. `alg. GB/s` = 12 B/px × HBM passes / time (the blocked kernels "
           "are FMA/issue-bound, not HBM-bound). *unblocked* = one `paraprox_hotspot` call (one tile-kernel pass) per "
           "step, the same scheme; *blocked ×* = unblocked ÷ blocked time.", "",
           "| grid | steps | scheme | kernel | µs / step | quality | HBM passes | alg. GB/s | speedup vs exact | "
           "unblocked kernel | unblocked µs / step | blocked × |",
           "|---|---:|---|---|---:|---:|---:|---:|---:|---|---:|---:|"]
    for r in rows:
        out.append("| %s | %d | %s | `%s` | %.2f | %.5f | %d | %.0f | %.2f | `%s` | %.1f | %.2f |" % (
            r["grid"], r["iterations"], r["scheme"], r["kernel"], r["us_per_step"], r["quality_mre"], r["hbm_passes"],
            r["algorithmic_gbs"], r["speedup_vs_exact"], r.get("unblocked_kernel", "-"),
            r.get("unblocked_us_per_step", float("nan")), r.get("blocked_speedup", float("nan"))))
    return "\n".join(out) + "\n"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", default="r02")
    a = ap.parse_args()
    tag = a.round
    for c in ("c1", "c2", "c3", "c4"):
        src = os.path.join(OUT, f"bench_{c}.json")
        if os.path.exists(src):
            shutil.copy(src, os.path.join(PROF, f"{tag}_bench_{c}.json"))
    for name, fn in (("toq_sweep", toq_md), ("convsep", convsep_md), ("hotspot", hotspot_md)):
        rows = load(f"{name}.json")
        if rows:
            json.dump(rows, open(os.path.join(PROF, f"{tag}_{name}.json"), "w"), indent=1)
            open(os.path.join(PROF, f"{tag}_{name}.md"), "w").write(fn(rows, tag))
    if os.path.exists(os.path.join(OUT, "kbench.jsonl")):
        shutil.copy(os.path.join(OUT, "kbench.jsonl"), os.path.join(PROF, f"{tag}_kbench.jsonl"))
    summ = os.path.join(ROOT, "tools", "ncu_summary.py")
    # summaries made on the GPU box (the captures themselves stay there)
    for wl in ("c1", "c2", "c3", "c4"):
        md = os.path.join(OUT, f"ncu_full_{wl}.md")
        if os.path.exists(md):
            shutil.copy(md, os.path.join(PROF, f"{tag}_ncu_full_{wl}.md"))
    for wl in ("c2", "c3"):
        if os.path.exists(os.path.join(OUT, f"launches_{wl}.md")):
            shutil.copy(os.path.join(OUT, f"launches_{wl}.md"), os.path.join(PROF, f"{tag}_launches_{wl}.md"))
    for name in ("ncu_kernels_c3.md", "ncu_bytes.md", "bench_ref.json"):
        if os.path.exists(os.path.join(OUT, name)):
            shutil.copy(os.path.join(OUT, name), os.path.join(PROF, f"{tag}_{name}"))
    sani = [os.path.join(OUT, f"sanitize_{t}.log") for t in ("memcheck", "racecheck", "synccheck", "initcheck")]
    if all(os.path.exists(x) for x in sani):
        lines = [f"# compute-sanitizer over tools/sanitize_run.py — {tag}", ""]
        for x in sani:
            txt = open(x).read().splitlines()
            keep = [ln for ln in txt if "SUMMARY" in ln or "sanitize run ok" in ln]
            lines.append(f"* `{os.path.basename(x)[9:-4]}`: " + "; ".join(keep))
        open(os.path.join(PROF, f"{tag}_sanitizers.md"), "w").write("\n".join(lines) + "\n")
    box = os.path.join(OUT, "traffic_box.json")
    if os.path.exists(box):
        tj = os.path.join(PROF, "traffic.json")
        d = json.load(open(tj)) if os.path.exists(tj) else {}
        for wl, kv in json.load(open(box)).items():
            d.setdefault(wl, {}).update(kv)
        json.dump(d, open(tj, "w"), indent=1, sort_keys=True)
    if os.path.exists(os.path.join(OUT, "launches_c2.csv")) and not os.path.exists(os.path.join(OUT, "launches_c2.md")):
        with open(os.path.join(PROF, f"{tag}_launches_c2.md"), "w") as fh:
            subprocess.run([sys.executable, summ, "launches", os.path.join(OUT, "launches_c2.csv")], stdout=fh, check=True)
    for wl in ("c1", "c2", "c3", "c4"):
        rep = os.path.join(OUT, f"prof_{wl}.ncu-rep")
        if os.path.exists(rep):
            with open(os.path.join(PROF, f"{tag}_ncu_full_{wl}.md"), "w") as fh:
                subprocess.run([sys.executable, summ, "full", rep, "--workload", wl, "--traffic",
                                os.path.join(PROF, "traffic.json")], stdout=fh, check=True)


if __name__ == "__main__":
    main()
