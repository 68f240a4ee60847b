"""A/B device timing of library builds (development aid; bench.py is the contract).

    python tools/ab_time.py CONFIG LIB_A LIB_B ...

Each library runs in its own process (CZC_LIB), rounds interleaved A, B, A, B, ...; per pattern
(P1, DERIV, AC, SSIM, ALL) the best library event time over the rounds is printed."""
import json, os, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, os, json
sys.path.insert(0, ROOT)
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
spec = synth.CONFIGS[CFG]
x, y = synth.make_pair(spec)
xd, yd = x.cuda(), y.cuda()
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
clean = torch.zeros(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
out = {}
with czc.Assessor(ndim=x.dim(), ssim_window=8, timing=True) as a:
    for name, mask, k in (("P1", czc.M_P1, 0), ("DERIV", czc.M_DERIV, 1), ("AC", czc.M_AUTOCORR, 2),
                          ("SSIM", czc.M_SSIM, 3), ("ALL", czc.M_ALL, 4)):
        for _ in range(2):
            a.assess(xd, yd, mask)
        ts = []
        for _ in range(7):
            flush.zero_(); clean.sum()
            r = a.assess(xd, yd, mask)
            ts.append(r["kernel_ms"][k] if name != "ALL" else sum(r["kernel_ms"][:4]))
        ts.sort()
        out[name] = ts[len(ts) // 2]
print("AB " + json.dumps(out))
'''

def main():
    cfg, libs = sys.argv[1], sys.argv[2:]
    best = {l: {} for l in libs}
    for rnd in range(2):
        for l in libs:
            env = dict(os.environ, CZC_LIB=os.path.abspath(l))
            code = CHILD.replace("ROOT", repr(ROOT)).replace("CFG", repr(cfg))
            r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
            line = [s for s in r.stdout.splitlines() if s.startswith("AB ")]
            if not line:
                print(l, "FAILED", r.stderr[-2000:]); continue
            d = json.loads(line[0][3:])
            for k, v in d.items():
                best[l][k] = min(best[l].get(k, 1e9), v)
    for l in libs:
        b = best[l]
        print(f"{cfg} {os.path.basename(l):24s} " + " ".join(f"{k}={v:.4f}" for k, v in b.items()))

if __name__ == "__main__":
    main()
