"""Instruction histogram of one kernel's SASS (optionally only between two addresses / the
largest backward-branch loop).  Usage: python tools/sass_loop.py LIB.so KERNEL_SUBSTRING [--loop]"""
import re, subprocess, sys, collections
lib, name = sys.argv[1], sys.argv[2]
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", out)
body = next(f for f in funcs if f.split("\n")[0].strip() == name or name in f.split("\n")[0])
ins = []
for ln in body.split("\n"):
    m = re.match(r"\s+/\*([0-9a-f]+)\*/\s+(.*?);", ln)
    if m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
if "--loop" in sys.argv:
    # largest backward branch = main loop
    best = None
    for a, t in ins:
        m = re.search(r"BRA (?:`\(\.L_x_\d+\)|0x([0-9a-f]+))", t)
        mm = re.search(r"BRA\s+(?:.*?)0x([0-9a-f]+)", t)
        if mm:
            tgt = int(mm.group(1), 16)
            if tgt < a and (best is None or a - tgt > best[1] - best[0]):
                best = (tgt, a)
    if best:
        ins = [(a, t) for a, t in ins if best[0] <= a <= best[1]]
        print(f"loop 0x{best[0]:x}..0x{best[1]:x}: {len(ins)} instructions")
c = collections.Counter()
for a, t in ins:
    op = re.sub(r"^@!?U?P[0-9T]+\s+", "", t).split()[0]
    c[op] += 1
print(len(ins), "instructions")
for op, n in c.most_common(40):
    print(f"{n:6d} {op}")
