"""Small assessments covering every kernel of libczc.so, for compute-sanitizer runs
(memcheck / racecheck / synccheck / initcheck): 3-D float32 and float64 (odd shapes, all window
extents class), 2-D, 1-D, 4-D, PDFs, loopback slabs, the pipelined host path, an adversarial
step field (exact SSIM fallback) and misaligned views.  Prints one line per case."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_cluster_yudgtc21_b200 as czc
import synth


def run(tag, x, y, mask=czc.M_FULL, **cfg):
    with czc.Assessor(ndim=x.dim(), **cfg) as a:
        r = a.assess(x.cuda(), y.cuda(), mask)
    print(f"{tag}: mask {r['computed_mask']} ssim {r['ssim']:.6f} exact {r['n_ssim_exact']} psnr {r['psnr']:.3f}", flush=True)


x, y = synth.make_pair(synth.config("C2", dims=(21, 37, 45)))
run("3d f32 w8", x, y, ssim_window=8, pdf_bins=32)
run("3d f32 w5 step", x, y, ssim_window=5, ssim_step=(1, 2, 3), ac_max_lag=16)
run("3d f32 w12", x, y, ssim_window=12, ac_max_lag=3)
run("3d f64 w8", x.double(), y.double(), ssim_window=8)
run("3d loopback", x, y, ssim_window=6, ac_max_lag=5, loopback_slabs=3)
x2, y2 = synth.make_pair(synth.config("C4", dims=(60, 130)))
run("2d w8", x2, y2, ssim_window=8)
run("1d w9", x2[7].contiguous(), y2[7].contiguous(), ssim_window=9)
x4 = x[:, :36, :].reshape(3, 7, 36, 45)
run("4d w3", x4, y[:, :36, :].reshape(3, 7, 36, 45), ssim_window=3, ac_max_lag=4)
rng = np.random.default_rng(3)
xs = np.where(np.indices((18, 20, 40))[2] < 20, 1.0, 1000.0) + 1e-3 * rng.standard_normal((18, 20, 40))
xs = xs.astype(np.float32)
ys = (0.2 * np.rint(xs.astype(np.float64) / 0.2)).astype(np.float32)
run("step exact fallback", torch.from_numpy(xs), torch.from_numpy(ys), ssim_window=8)
xf, yf = x.reshape(-1), y.reshape(-1)
with czc.Assessor(ndim=1, pdf_bins=16) as a:
    r = a.assess(xf.cuda()[1:], yf.cuda()[1:], czc.M_P1 | czc.M_PDF)
    print("misaligned p1/pdf", r["mse"], flush=True)
with czc.Assessor(ndim=3, ssim_window=6) as a:
    r = a.assess_host(x.pin_memory(), y.pin_memory(), czc.M_ALL)
    print("host pipeline", r["ssim"], flush=True)
torch.cuda.synchronize()
print("sanitize target done")
