"""Exact-path count and SSIM time of one config under the library in CZC_LIB (development aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
x, y = synth.make_pair(synth.CONFIGS[cfg])
xd, yd = x.cuda(), y.cuda()
with czc.Assessor(ndim=x.dim(), ssim_window=8, timing=True) as a:
    for _ in range(3):
        r = a.assess(xd, yd, czc.M_SSIM | czc.M_P1)
print(cfg, os.path.basename(os.environ.get("CZC_LIB", "default")), "exact", r["n_ssim_exact"], "of", r["n_windows"],
      "ssim_ms", round(r["kernel_ms"][3], 4))
