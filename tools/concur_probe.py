"""Probe: do two pattern kernels overlap usefully when run on separate streams? (dev aid)"""
import sys, os, threading, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth
x, y = synth.make_pair(synth.CONFIGS["C2"])
xd, yd = x.cuda(), y.cuda()
s1, s2, s3 = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
a1 = czc.Assessor(ndim=3, ssim_window=8, stream=s1)
a2 = czc.Assessor(ndim=3, ssim_window=8, stream=s2)
a3 = czc.Assessor(ndim=3, ssim_window=8, stream=s3)
a0 = czc.Assessor(ndim=3, ssim_window=8)
flush = torch.empty(256 * 1024 * 1024 // 4, device="cuda")
def seq(masks):
    flush.zero_(); torch.cuda.synchronize()
    t = time.perf_counter()
    for m in masks: a0.assess(xd, yd, m)
    torch.cuda.synchronize()
    return (time.perf_counter() - t) * 1e3
def par(groups):
    flush.zero_(); torch.cuda.synchronize()
    t = time.perf_counter()
    ths = [threading.Thread(target=lambda a=a, ms=ms: [a.assess(xd, yd, m) for m in ms]) for a, ms in zip((a1, a2, a3), groups)]
    [h.start() for h in ths]; [h.join() for h in ths]
    torch.cuda.synchronize()
    return (time.perf_counter() - t) * 1e3
for name, fn in (("all-in-one", lambda: seq([czc.M_ALL])),
                 ("seq 4 calls", lambda: seq([czc.M_P1, czc.M_DERIV, czc.M_P1 | czc.M_AUTOCORR, czc.M_SSIM])),
                 ("par deriv|ssim|p1ac", lambda: par([[czc.M_DERIV], [czc.M_SSIM], [czc.M_P1 | czc.M_AUTOCORR]])),
                 ("par deriv|ssim", lambda: par([[czc.M_DERIV], [czc.M_SSIM], []])),
                 ("seq deriv,ssim", lambda: seq([czc.M_DERIV, czc.M_SSIM]))):
    for _ in range(3): fn()
    ts = sorted(fn() for _ in range(7))
    print(f"{name:22s} wall {ts[len(ts)//2]:.3f} ms (min {ts[0]:.3f})")
