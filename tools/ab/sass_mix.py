"""Instruction mix and stall hotspots of an ncu source-page export
(`ncu -i rep --page source --csv --print-source sass > x.csv`):
    python tools/ab/sass_mix.py x.csv"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
iS, iE = hdr.index("Source"), hdr.index("Instructions Executed")
iA, iN = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Warp Stall Sampling (Not-issued Samples)")
ce, ca, cn = Counter(), Counter(), Counter()
for r in data:
    s = r[iS].strip().split()
    if not s:
        continue
    op = (s[1] if s[0].startswith("@") else s[0]).split(".")[0]
    ce[op] += int(r[iE] or 0)
    ca[op] += int(r[iA] or 0)
    cn[op] += int(r[iN] or 0)
E, A = sum(ce.values()), sum(ca.values())
fma = sum(ce[o] for o in ("FFMA2", "FFMA", "IMAD", "HFMA2", "FMUL", "FADD"))
print(f"{rows[0][1][:90]}\nwarp instructions {E / 1e6:.2f} M; FMA-pipe ops {fma / E:.1%} of them; samples {A}")
for op, v in ce.most_common(14):
    print(f"  {op:10s} {v / 1e6:8.2f} M {v / E:6.1%}   stall samples {ca[op] / A:6.1%} (not issued {cn[op] / A:5.1%})")
