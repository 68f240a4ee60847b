"""Basic-block view of an ncu source-page CSV: consecutive SASS lines with the same executed
count are grouped; prints each group's address range, count, size and thread-instr/elem share.
usage: python tools/sass_blocks.py SRC.csv ELEMS [MIN_SHARE]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ai, si, ii = h.index("Address"), h.index("Source"), h.index("Instructions Executed")
elems = float(sys.argv[2]); mn = float(sys.argv[3]) if len(sys.argv) > 3 else 0.5
seen = {}
for r in rows[2:]:
    if len(r) <= ii:
        continue
    try:
        a = int(r[ai], 16); n = float(r[ii])
    except ValueError:
        continue
    seen[a] = (n, r[si].strip())
base = min(seen)
groups = []
for a in sorted(seen):
    n, s = seen[a]
    if groups and groups[-1][1] == n:
        groups[-1][2].append(s)
    else:
        groups.append([a - base, n, [s]])
for off, n, ins in groups:
    share = n * len(ins) * 32 / elems
    if share >= mn:
        ops = collections.Counter((x.split()[1] if x.startswith("@") else x.split()[0]) for x in ins)
        print(f"0x{off:05x} n={n:9.0f} len={len(ins):4d} {share:6.2f}/elem  " + ", ".join(f"{o}:{c}" for o, c in ops.most_common(7)))
