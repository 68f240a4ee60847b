"""Summarise an ncu --page source --csv --print-source sass dump: executed instructions and stall
samples by opcode, the top instructions, shared-memory excess wavefronts (development aid)."""
import csv, collections, sys
rows = list(csv.reader(open(sys.argv[1])))
ends = [i for i, r in enumerate(rows) if i > 0 and r and r[0] == "Kernel Name"]
rows = rows[:ends[0]] if ends else rows   # first kernel section only
h = rows[1]
ix = {k: h.index(k) for k in ("Address", "Source", "Warp Stall Sampling (All Samples)", "Instructions Executed",
                              "L1 Wavefronts Shared Excessive")}
ops, st, exc = collections.Counter(), collections.Counter(), collections.Counter()
tot = totst = 0
top = []
for r in rows[2:]:
    if len(r) < len(h) - 2:
        continue
    src = r[ix["Source"]].strip()
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    op = op.split(".")[0]
    n = int(r[ix["Instructions Executed"]] or 0)
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    e = int(r[ix["L1 Wavefronts Shared Excessive"]] or 0)
    ops[op] += n; st[op] += s; exc[op] += e; tot += n; totst += s
    top.append((s, n, e, r[ix["Address"]][-5:], src[:70]))
print("instructions", tot, "stall samples", totst)
for op, n in ops.most_common(28):
    print(f"{op:10s} {n:12d} {100*n/tot:5.1f}%  stall {100*st[op]/max(totst,1):5.1f}%  excess_wf {exc[op]}")
print("top stall instructions:")
for t in sorted(top, reverse=True)[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(t)
