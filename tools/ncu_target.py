"""Small driver for ncu captures: C2 workload, full metric set, N calls (default 3)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
calls = int(sys.argv[2]) if len(sys.argv) > 2 else 3
x, y = synth.make_pair(synth.CONFIGS[cfg])
xd, yd = x.cuda(), y.cuda()
with czc.Assessor(ndim=x.dim(), ssim_window=8) as a:
    for _ in range(calls):
        r = a.assess(xd, yd, czc.M_ALL)
torch.cuda.synchronize()
print("psnr", r["psnr"], "ssim", r["ssim"])
