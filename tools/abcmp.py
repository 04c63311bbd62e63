"""Compare kbench JSON lines of A/B variants: python tools/abcmp.py base.jsonl other.jsonl ..."""
import json
import sys

files = sys.argv[1:]
rows = {}
for i, fn in enumerate(files):
    for line in open(fn):
        if not line.startswith("{"):
            continue
        d = json.loads(line)
        key = (d["wl"], d.get("dy", d.get("lattice_dy")), d.get("dx", "L"), d["kernel"])
        rows.setdefault(key, {})[i] = d["gbs"]
print("key", *[f.split("/")[-1] for f in files])
for k, v in rows.items():
    base = v.get(0)
    cells = [f"{v[i]:.0f}" + (f" ({v[i] / base:.3f})" if base and i else "") if i in v else "-" for i in range(len(files))]
    print(*k, *cells)
