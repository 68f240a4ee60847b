"""Per-opcode executed-instruction totals and the hottest SASS lines from an ncu source-page CSV
(ncu -i REP --page source --csv --print-source sass -k regex:K > file.csv)."""
import csv, sys, collections, re
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ai, si, ii, wi = h.index("Address"), h.index("Source"), h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
tot = collections.Counter(); stall = collections.Counter()
lines = []
for r in rows[2:]:
    if len(r) <= ii:
        continue
    try:
        n = float(r[ii]); w = float(r[wi] or 0)
    except ValueError:
        continue
    op = re.sub(r"^@!?U?P[0-9T]+\s+", "", r[si].strip()).split(" ")[0]
    tot[op] += n; stall[op] += w
    lines.append((w, n, r[si].strip()))
T = sum(tot.values()); S = sum(stall.values())
elems = float(sys.argv[2]) if len(sys.argv) > 2 else None
print(f"total warp-instructions {T:.4g}" + (f"  = {32*T/elems:.1f} thread-instr per element" if elems else ""))
for op, n in tot.most_common(25):
    print(f"{op:28s} {n:12.4g} {100*n/T:5.1f}%  stall-samples {100*stall[op]/max(S,1):5.1f}%" + (f"  {32*n/elems:6.2f}/elem" if elems else ""))
print("--- hottest lines by stall samples")
for w, n, s in sorted(lines, reverse=True)[:15]:
    print(f"{w:8.0f} {n:10.4g}  {s}")
