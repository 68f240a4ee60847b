"""Quick per-pattern device timing on a config (development aid; bench.py is the contract)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cluster_yudgtc21_b200 as czc
import synth

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
spec = synth.CONFIGS[cfg]
x, y = synth.make_pair(spec)
xd, yd = x.cuda(), y.cuda()
nbytes = 2 * x.numel() * 4
flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
w = 8
with czc.Assessor(ndim=x.dim(), ssim_window=w, timing=True) as a:
    for name, mask in (("P1", czc.M_P1), ("DERIV", czc.M_DERIV), ("AC", czc.M_AUTOCORR),
                       ("SSIM", czc.M_SSIM), ("ALL", czc.M_ALL)):
        for _ in range(2):
            a.assess(xd, yd, mask)
        ts = []
        for _ in range(5):
            flush.zero_(); flush.sum()
            r = a.assess(xd, yd, mask)
            ts.append(r["kernel_ms"])
        best = [min(t[i] for t in ts) for i in range(5)]
        tot = sum(best[:4])
        print(f"{cfg} {name:6s} p1={best[0]:.4f} deriv={best[1]:.4f} ac={best[2]:.4f} ssim={best[3]:.4f} "
              f"call={best[4]:.4f} ms -> {nbytes/ (tot*1e-3) / 1e9:.1f} GB/s (kernels)")
