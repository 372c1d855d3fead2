"""Summarise an ncu --page source --csv --print-source sass dump: top stall PCs and per-class totals."""
import csv
import re
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = [r for r in rows[2:] if len(r) == len(hdr)]
i_s, i_src, i_ex = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source"), hdr.index("Instructions Executed")
tot = sum(float(r[i_s] or 0) for r in data)
print("total stall samples", tot, "instructions", sum(float(r[i_ex] or 0) for r in data))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
for k, r in enumerate(sorted(data, key=lambda r: -float(r[i_s] or 0))[:n]):
    print(f"{float(r[i_s]) / tot * 100:5.1f}%  {r[0][-5:]}  {r[i_src].strip()[:80]:80s} exec={r[i_ex]}")
cls = defaultdict(float)
ex = defaultdict(float)
for r in data:
    op = r[i_src].strip().split()[0] if r[i_src].strip() else "?"
    if op.startswith("@"):
        op = r[i_src].strip().split()[1]
    op = op.split(".")[0]
    cls[op] += float(r[i_s] or 0)
    ex[op] += float(r[i_ex] or 0)
print("\nby opcode (stall %, executed warp-instr):")
for op, v in sorted(cls.items(), key=lambda kv: -kv[1])[:25]:
    print(f"  {op:10s} {v / tot * 100:5.1f}%  {ex[op]:.3g}")
