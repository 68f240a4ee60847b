"""A/B of the single-GPU launch sequence: two concurrent branches vs one stream (CZC_SEQUENTIAL),
timed as the bench times a step (graph replay, events around the call, L2 flushed between).
Development aid.    python tools/ab_concurrent.py C2 [C3 ...]"""
import os, subprocess, sys, json
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, json
sys.path.insert(0, ROOT)
import torch, bench, synth
import paper_conf_cluster_yudgtc21_b200 as czc
spec = synth.CONFIGS[CFG]
x, y = bench.make_slab_device(spec, 0, spec.dims[0], torch.device("cuda", 0), 1)
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
clean = torch.zeros(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
st = torch.cuda.current_stream()
with czc.Assessor(ndim=x.dim(), ssim_window=8, stream=st) as a:
    for _ in range(3):
        r = a.assess(x, y, czc.M_ALL)
    ts = []
    for _ in range(15):
        flush.zero_(); clean.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); r = a.assess(x, y, czc.M_ALL); e1.record(st); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
ts.sort()
print("AB " + json.dumps({"ms": ts[len(ts) // 2], "ssim": r["ssim"], "mse": r["mse"], "ac1": float(r["ac"][1]), "der1": r["der1_mae"]}))
'''
for cfg in sys.argv[1:]:
    for mode in ("1", "b0", "b1", "b2", "1", "b0", "b1", "b2"):
        env = dict(os.environ, CZC_SEQUENTIAL="1" if mode == "1" else "0")
        if mode.startswith("b"):
            env["CZC_BRANCHES"] = mode[1:]
        r = subprocess.run([sys.executable, "-c", CHILD.replace("ROOT", repr(ROOT)).replace("CFG", repr(cfg))],
                           env=env, capture_output=True, text=True)
        line = [l for l in r.stdout.splitlines() if l.startswith("AB ")]
        print(cfg, "sequential" if mode == "1" else "branches " + mode[1:], line[0][3:] if line else r.stderr[-1500:], flush=True)
