#!/usr/bin/env python
"""Summarise an `ncu --page source --csv --print-source sass` export: hottest instructions by
stall samples, and instruction-executed totals by opcode.  python tools/sass_hot.py f.csv [N]"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
body = [r for r in rows[2:] if len(r) == len(hdr)]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
tot_s = sum(int(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in body)
tot_i = sum(int(r[ix["Instructions Executed"]] or 0) for r in body)
print(f"samples {tot_s}  warp-instructions {tot_i}")
ops = Counter()
for r in body:
    op = r[ix["Source"]].split()[0] if r[ix["Source"]].split() else "?"
    if op.startswith("@"):
        op = r[ix["Source"]].split()[1]
    ops[op.split(".")[0]] += int(r[ix["Instructions Executed"]] or 0)
print("by opcode:", ", ".join(f"{k} {v/tot_i*100:.1f}%" for k, v in ops.most_common(25)))
hot = sorted(body, key=lambda r: -int(r[ix["Warp Stall Sampling (All Samples)"]] or 0))[:N]
for r in hot:
    print(f'{r[ix["Address"]][-5:]} {int(r[ix["Warp Stall Sampling (All Samples)"]]):7d} {int(r[ix["Instructions Executed"]]):10d}  {r[ix["Source"]].strip()[:90]}')
