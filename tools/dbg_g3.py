"""SSIM + P1 on a small C2-shaped field with and without per-kernel timing under the library in
CZC_LIB: mean SSIM, window count, exact recomputes, kernel times (development aid)."""
import os, sys
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
x, y = synth.make_pair(synth.config("C2", dims=(40, 70, 90)))
xd, yd = x.cuda(), y.cuda()
for timing in (False, True):
    try:
        with czc.Assessor(ssim_window=8, timing=timing) as a:
            r = a.assess(xd, yd, czc.M_SSIM | czc.M_P1)
        torch.cuda.synchronize()
        print("timing", timing, "ssim", r["ssim"], "n", r["n_windows"], "exact", r["n_ssim_exact"], r.get("kernel_ms"))
    except Exception as e:
        print("ERR", repr(e))
