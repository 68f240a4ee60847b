"""SSIM + P1 on a small and the full C2 shape under the library in CZC_LIB; prints the mean SSIM
and exact recomputes or the error (development aid: tensor-copy bring-up)."""
import os, sys
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
for dims in [(40, 72, 92), (100, 500, 500)]:
    x, y = synth.make_pair(synth.config("C2", dims=dims))
    try:
        with czc.Assessor(ssim_window=8) as a:
            r = a.assess(x.cuda(), y.cuda(), czc.M_SSIM | czc.M_P1)
        print(dims, r["ssim"], r["n_ssim_exact"])
    except Exception as e:
        print(dims, "ERR", e)
