"""Per-window SSIM of two library builds on one small field; where they differ (debug aid)."""
import os, sys, subprocess, json
sys.path.insert(0, os.getcwd())
import numpy as np
code = r'''
import os, sys
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
x, y = synth.make_pair(synth.config("C2", dims=(20, 60, 40)))
nw = [n - 7 for n in x.shape]
dbg = torch.full(nw, float("nan"), dtype=torch.float64, device="cuda")
with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
    r = a.assess(x.cuda(), y.cuda(), czc.M_SSIM | czc.M_P1)
np.save(sys.argv[1], dbg.cpu().numpy())
print(r["ssim"], r["n_ssim_exact"])
'''
for lib in sys.argv[1:3]:
    out = subprocess.run([sys.executable, "-c", code, "/tmp/" + os.path.basename(lib) + ".npy"],
                         env=dict(os.environ, CZC_LIB=os.path.abspath(lib)), capture_output=True, text=True)
    print(lib, out.stdout.strip(), out.stderr[-300:])
a = np.load("/tmp/" + os.path.basename(sys.argv[1]) + ".npy")
b = np.load("/tmp/" + os.path.basename(sys.argv[2]) + ".npy")
d = np.abs(a - b) > 1e-9
print("differ", int(d.sum()), "of", d.size)
z, yy, xx = np.nonzero(d)
print("z", np.bincount(z)[:20])
print("y mod 24", np.bincount(yy % 24, minlength=24))
print("x", np.bincount(xx, minlength=33))
idx = list(zip(*np.nonzero(d)))[:6]
for i in idx:
    print(i, a[i], b[i])
print("plane means", [float(np.nanmean(a[z])) for z in range(4)], [float(np.nanmean(b[z])) for z in range(4)])
