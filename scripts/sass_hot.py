"""Summarise an ncu --page source (SASS) CSV: top instructions by stall samples and per-opcode totals.
usage: ncu -i X.ncu-rep --page source --csv --print-source sass > X.csv; python scripts/sass_hot.py X.csv"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
i_src = hdr.index("Source")
i_ex = hdr.index("Instructions Executed")
tot = sum(float(r[i_s] or 0) for r in data) or 1.0
print("total samples", tot)
for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{float(r[i_s]) / tot * 100:5.1f}% {r[0][-5:]} {r[i_src][:80]:80s} ex={r[i_ex]}")
c, e = Counter(), Counter()
for r in data:
    toks = r[i_src].split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
    op = op.split(".")[0]
    c[op] += float(r[i_s] or 0)
    e[op] += float(r[i_ex] or 0)
for op, v in c.most_common(15):
    print(f"{op:10s} {v / tot * 100:5.1f}%  executed {e[op]:.0f}")
