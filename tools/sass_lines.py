"""Map an ncu source-page SASS dump (--page source --csv --print-source sass) of one kernel to
source lines via the line table of the same build (development aid).

    python tools/sass_lines.py LIB.so KERNEL_MANGLED_PREFIX DUMP.csv [N]"""
import collections, csv, os, re, subprocess, sys, tempfile

lib, kname, dump = sys.argv[1:4]
ntop = int(sys.argv[4]) if len(sys.argv) > 4 else 40
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=tmp, capture_output=True)
off2src = None
for cub in sorted(os.listdir(tmp)):
    out = subprocess.run(["nvdisasm", "--print-line-info", os.path.join(tmp, cub)], capture_output=True, text=True).stdout
    lines = out.splitlines()
    idx = [i for i, l in enumerate(lines) if l.startswith(".text." + kname)]
    if not idx:
        continue
    s = idx[0]; e = s + 1
    while e < len(lines) and not lines[e].startswith(".text."):
        e += 1
    off2src, cur = {}, None
    for l in lines[s:e]:
        if "//##" in l:
            m = re.search(r'File "([^"]+)", line (\d+)', l)
            if m:
                cur = (m.group(1).split("/")[-1], int(m.group(2)))
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*)", l)
        if m:
            off2src[int(m.group(1), 16)] = cur
    break
rows = list(csv.reader(open(dump)))
ends = [i for i, r in enumerate(rows) if i > 0 and r and r[0] == "Kernel Name"]
rows = rows[:ends[0]] if ends else rows   # first kernel section only
h = rows[1]
a, n, st = h.index("Address"), h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
base = int(rows[2][a], 16)
bl, bs = collections.Counter(), collections.Counter()
for r in rows[2:]:
    if len(r) <= n:
        continue
    src = off2src.get(int(r[a], 16) - base)
    bl[src] += int(r[n] or 0); bs[src] += int(r[st] or 0)
tot = sum(bl.values())
for k, v in sorted(bl.items(), key=lambda x: -x[1])[:ntop]:
    print(k, v, f"{100 * v / tot:.1f}%", "stall", bs[k])
