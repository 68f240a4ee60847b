"""Opcode mix of one kernel from an `ncu --page source --csv` (SASS) export: executed warp
instructions and stall samples per opcode class (dev aid).   python tools/sass_mix.py FILE.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h, data = rows[hi], rows[hi + 1:]
ie, st = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
cnt, stall = collections.Counter(), collections.Counter()
for r in data:
    if len(r) <= ie or not r[ie] or not r[ie].replace(",", "").isdigit():
        continue                       # blank rows, repeated headers of further launches
    op = r[1].split()
    if not op:
        continue
    o = op[1] if op[0].startswith("@") else op[0]
    key = o.split(".")[0]
    if key == "DADD" and ", RZ," in r[1]:
        key = "DADD(move)"
    if key == "IMAD" and "MOV" in o:
        key = "IMAD.MOV"
    cnt[key] += int(r[ie].replace(",", ""))
    stall[key] += float(r[st] or 0)
tot, ts = sum(cnt.values()), sum(stall.values())
for k, v in cnt.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 30):
    print(f"{k:14s} {v / tot * 100:5.1f}% instr  {stall[k] / ts * 100:5.1f}% stall")
print("total warp instructions", tot)
