"""Executed warp-instructions of one kernel split into address regions.
usage: python tools/sass_regions.py SRC.csv ELEMS [ADDR1 ADDR2 ...]   (hex addresses relative to
the function start; regions are [start, ADDR1), [ADDR1, ADDR2), ...).  SRC.csv from
ncu -i REP --page source --csv --print-source sass -k regex:K"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ai, si, ii = h.index("Address"), h.index("Source"), h.index("Instructions Executed")
elems = float(sys.argv[2])
cuts = [int(a, 16) for a in sys.argv[3:]]
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
reg = collections.defaultdict(float)
ops = collections.defaultdict(collections.Counter)
for a, (n, s) in seen.items():
    off = a - base
    k = sum(1 for c in cuts if off >= c)
    reg[k] += n
    op = s.split()[0] if not s.startswith("@") else s.split()[1]
    ops[k][op] += n
tot = sum(reg.values())
print(f"total {tot:.4g} warp-instr = {tot*32/elems:.1f} thread-instr/elem")
for k in sorted(reg):
    lo = 0 if k == 0 else cuts[k - 1]
    print(f"region {k} [0x{lo:x}..): {reg[k]*32/elems:7.2f}/elem  top: " +
          ", ".join(f"{o} {c*32/elems:.1f}" for o, c in ops[k].most_common(6)))
