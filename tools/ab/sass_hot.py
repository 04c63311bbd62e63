"""Non-FMA instructions of an ncu source-page export ranked by execution
count x (a rough) issue cost, with their neighbourhood:
    python tools/ab/sass_hot.py x.csv [n]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
iS, iE = hdr.index("Source"), hdr.index("Instructions Executed")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 12
skip = ("FFMA2", "FFMA ", "LDS", "FFMA")
cands = [(int(r[iE] or 0), i) for i, r in enumerate(data)
         if r[iS].strip() and not r[iS].strip().split()[-1].startswith("FFMA")
         and not any(r[iS].strip().lstrip("@!P0123456789T ").startswith(s) for s in skip)]
cands.sort(reverse=True)
tot = sum(int(r[iE] or 0) for r in data)
print("total", tot / 1e6, "M warp instructions")
# group consecutive blocks with the same exec count
seen = set()
for e, i in cands[:400]:
    if e in seen:
        continue
    seen.add(e)
    block = [r for r in data if int(r[iE] or 0) == e]
    ops = {}
    for r in block:
        s = r[iS].strip().split()
        op = (s[1] if s[0].startswith("@") else s[0]).split(".")[0]
        ops[op] = ops.get(op, 0) + 1
    print(f"exec {e:>10d} x {len(block):4d} instrs = {e * len(block) / tot:6.1%}: " +
          ", ".join(f"{k} {v}" for k, v in sorted(ops.items(), key=lambda x: -x[1])[:10]))
    if len(seen) >= n:
        break
