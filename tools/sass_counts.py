"""Per-kernel SASS instruction counts of libparaprox.so (cuobjdump -sass):
the evidence that the tile kernels are Blackwell-native (TMA tensor loads
UTMALDG and stores UTMASTG, mbarrier SYNCS ops, packed FFMA2), for
profiles/sass_r02.md.

    python tools/sass_counts.py [paper_conf_asplos_samadijlm14_b200/libparaprox.so] > profiles/sass_r02.md
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

COLS = ["UTMALDG", "UTMASTG", "UTMAPF", "SYNCS", "FFMA2", "FFMA", "FADD", "LDS", "STS", "LDG", "STG", "SHFL",
        "DFMA", "BAR", "MOV"]


def demangle(names):
    try:
        out = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.splitlines()
        return out if len(out) == len(names) else names
    except OSError:
        return names


def main():
    so = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "paper_conf_asplos_samadijlm14_b200",
                                                             "libparaprox.so")
    sass = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True, check=True).stdout
    counts = collections.OrderedDict()
    arch = set()
    cur = None
    for line in sass.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            counts[cur] = collections.Counter()
            continue
        m = re.search(r"arch = (sm_\w+)", line)
        if m:
            arch.add(m.group(1))
        m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]*)?", line)
        if m and cur:
            op = m.group(1)
            counts[cur][op] += 1
            counts[cur]["_total"] += 1
    names = list(counts)
    pretty = dict(zip(names, demangle(names)))
    from ncu_summary import short  # the library's kernel names for k_tiles instances
    print("# SASS instruction counts per kernel (r02)\n")
    print(f"`cuobjdump -sass {os.path.relpath(so, ROOT)}` ({', '.join(sorted(arch)) or 'arch ?'}), "
          "`tools/sass_counts.py`. Static counts (instructions in the code, not executed). "
          "UTMALDG/UTMASTG = TMA tensor load/store (`cp.async.bulk.tensor`), UTMAPF = tensor-map prefetch, "
          "SYNCS = mbarrier operations, FFMA2 = packed `fma.rn.f32x2` (sm_100).\n")
    print("| kernel | " + " | ".join(COLS) + " | total |")
    print("|---|" + "---:|" * (len(COLS) + 1))
    tot = collections.Counter()
    for n in names:
        c = counts[n]
        p = pretty[n]
        if "k_tiles<" in p:
            label = short(p) + ("_quality" if re.search(r"k_tiles<[^>]*, (true|1)>", p) else "")
        else:
            label = re.sub(r"^void ", "", p.split("(")[0]).replace("ppx::", "")
        row = [c.get(k, 0) if k != "SYNCS" else sum(v for o, v in c.items() if o.startswith("SYNCS")) for k in COLS]
        tot.update(dict(zip(COLS, row)))
        tot["_total"] += c["_total"]
        print(f"| `{label}` | " + " | ".join(str(v) for v in row) + f" | {c['_total']} |")
    print("| **all** | " + " | ".join(str(tot[k]) for k in COLS) + f" | {tot['_total']} |")


if __name__ == "__main__":
    main()
