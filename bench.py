#!/usr/bin/env python
"""Benchmark of the B200 cuZ-Checker assessment hot path (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C2]

One STEP = one czc_assess call with the full metric set (P1 fused reduction, P2 derivatives +
autocorrelation lags 1..10, P3 8^3 SSIM step 1) over one (orig, recon) float32 pair resident in
HBM.  Workload at N=1: BASELINE.json configs[1], the Hurricane-shaped 100x500x500 field (abs
error bound 1e-4).  N>1 (torchrun, one rank per GPU): weak scaling, rank r owns planes
[100 r, 100 r + 100) of a (100 N) x 500 x 500 field, with NCCL halo exchange and two small
allgathers inside czc_assess.  Metric: GB/s of orig+recon bytes, whole job.

`--impl reference` times the CPU oracle (the paper's method written out plainly, test
infrastructure) on a bounded slab of the same workload; under torchrun only rank 0 runs it.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "assessment GB/s (orig+recon bytes) and % HBM roofline per pattern at 1/2/4/8 B200"
UNIT = "GB/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="C2")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-f64", action="store_true", help="skip the float64-input measurement")
    return p.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    return rank, world, local


# ------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [v.strip() for v in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic():
    """Per-launch DRAM bytes of the dominant kernel from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_dominant.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f)
    return None


# ------------------------------------------------------------------------------------ oracle leg
def oracle_sample(spec, planes: int = 100):
    """The CPU oracle on a bounded slab (first `planes` planes; default the whole Hurricane-shaped
    field, ~25 core-seconds) of the workload, full metric set.
    Returns (GB/s, seconds, cores, description)."""
    import oracle
    import synth
    x, y = synth.make_pair(spec, 0, planes)
    xn, yn = x.numpy(), y.numpy()
    t0 = time.perf_counter()
    oracle.p1(xn, yn)
    oracle.deriv(xn, yn)
    oracle.autocorr(xn, yn, 10)
    oracle.ssim(xn, yn, [8, 8, 8])
    dt = time.perf_counter() - t0
    nbytes = 2 * xn.size * 4
    desc = (f"planes [0,{planes}) of {spec.name} ({planes}x{spec.dims[1]}x{spec.dims[2]} pair, "
            f"{nbytes / 1e6:.1f} MB), full metric set (P1, derivatives, AC lags 1..10, 8^3 SSIM step 1)")
    return nbytes / dt / 1e9, dt, oracle.threads(), desc


def run_reference(args, rank, world):
    if rank != 0:
        return
    import synth
    spec = synth.CONFIGS[args.config]
    vals, secs = [], []
    cores, desc = None, None
    for i in range(args.warmup + args.steps):
        v, dt, cores, desc = oracle_sample(spec, planes=min(spec.dims[0], 25))
        if i >= args.warmup:
            vals.append(v)
            secs.append(dt)
    value = len(vals) / sum(1.0 / v for v in vals)    # harmonic mean = total bytes / total time
    line = {"impl": "reference", "metric": METRIC, "value": round(value, 6), "unit": UNIT,
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1e3 * sum(secs) / len(secs), 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{spec.name} (bounded slab sample)", "sample": desc},
            "cpu_baseline": {"value": round(value, 6), "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": round(value, 6), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------ our leg
def run_ours(args, rank, world, local):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_cluster_yudgtc21_b200 as czc
    import synth

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    spec = synth.CONFIGS[args.config]
    nz_local = spec.dims[0]
    gdims = (nz_local * world,) + tuple(spec.dims[1:])
    gspec = synth.config(args.config, dims=gdims)
    z0 = rank * nz_local
    # generate this rank's slab on the host (bit-identical recipe), copy once to HBM
    xh, yh = synth.make_pair(gspec, z0, z0 + nz_local, device="cpu",
                             range_hint=None)
    xd, yd = xh.to(dev), yh.to(dev)
    nbytes_rank = 2 * xh.numel() * 4

    uid = None
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        obj = [czc_nccl_uid() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    stream = torch.cuda.current_stream(dev)
    cfg = dict(ssim_window=8, ssim_step=1, ac_max_lag=10)
    if world > 1:
        cfg.update(rank=rank, nranks=world, nccl_uid=uid)
    # the timed steps run as users run them (single GPU: the launch sequence replays as one CUDA
    # graph); per-kernel times come from a second context with per-kernel events (timing=True,
    # direct launches) over as many untimed-for-value steps afterwards
    a = czc.Assessor(ndim=3, device=local, stream=stream, **cfg)
    kw = dict(dims=gdims, z0=z0) if world > 1 else {}

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # 256 MB > L2
    clean = torch.zeros(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # read-only after this
    for _ in range(args.warmup):
        a.assess(xd, yd, czc.M_ALL, **kw)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    kms = []
    sampler = ClockSampler(local)
    barrier()
    sampler.start()
    time.sleep(0.3)
    t_wall = time.perf_counter()
    for i in range(args.steps):
        flush.zero_()                                   # L2 flush between timed steps (not timed):
        clean.sum()                                     # write 256 MB, then read ANOTHER 256 MB so
                                                        # the dirty lines are written back before the
                                                        # step starts and L2 holds only clean lines
        ev[i][0].record(stream)
        a.assess(xd, yd, czc.M_ALL, **kw)
        ev[i][1].record(stream)
    barrier()
    t_wall = time.perf_counter() - t_wall
    clocks = sampler.stop()
    cfg_t = dict(cfg)
    if world > 1:                       # a second communicator needs its own ncclUniqueId
        obj = [czc_nccl_uid() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        cfg_t["nccl_uid"] = obj[0]
    with czc.Assessor(ndim=3, device=local, stream=stream, timing=True, **cfg_t) as at:
        for i in range(args.warmup + args.steps):
            flush.zero_()
            clean.sum()
            r = at.assess(xd, yd, czc.M_ALL, **kw)
            if i >= args.warmup:
                kms.append(r["kernel_ms"])
    step_ms = [s.elapsed_time(e) for s, e in ev]
    tot_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
    value = world * nbytes_rank * args.steps / (tot_ms * 1e-3) / 1e9

    # per-kernel device time (library events on the launching stream), averaged over timed steps:
    # P1, P2 derivatives, P2 autocorrelation (3 walk launches), P3 SSIM
    shares = {name: statistics.mean(k[i] for k in kms)
              for i, name in enumerate(("P1", "P2_deriv", "P2_autocorr", "P3_ssim"))}
    dom = max(shares, key=shares.get)
    # secondary ceiling: every pattern is FP64-arithmetic / issue bound, so the
    # algorithmic FP64 operations of the method (per element / interior point /
    # window) are also set against the FP64 pipe rate measured on this GPU model
    # (profiles/r01_pipes2.txt: DFMA 61.6 lanes/clk/SM; 148 SMs at 1.965 GHz)
    fp64_peak = 61.6 * 148 * 1.965                     # G FP64 instructions / s
    units = {"P1": (12, int(r["n"]), "element: e, 6 moment sums, |e| sum, 2 extrema, pwr quotient + sum"),
             "P2_deriv": (74, int(r["n_interior"]), "interior point: 2 x 22 stencil ops, 2 sqrt, 5 x 6 statistics"),
             "P2_autocorr": (31, int(r["n"]), "element: eps, 10 lags x 3 axes FMAs"),
             "P3_ssim": (42, int(r["n_windows"]), "window: 24 running-sum adds, 2 products, 16 mix ops")}
    fp64 = {}
    for k, (ops, n_units, what) in units.items():
        if shares.get(k, 0) > 0:
            a_g = ops * n_units / world / (shares[k] * 1e-3) / 1e9    # per GPU (units are global)
            fp64[k] = {"achieved": round(a_g, 1), "frac": round(a_g / fp64_peak, 4), "ops_per_unit": ops,
                       "units_per_launch": n_units, "unit": what}
    peak, peak_src = measured_peak()
    alg_bytes = nbytes_rank                              # each pattern reads the pair once (+ halos)
    achieved = alg_bytes / (shares[dom] * 1e-3) / 1e9
    tr = ncu_traffic()
    traffic = tr.get("dram_bytes_per_launch") if tr and tr.get("kernel_pattern") == dom else None
    traffic_src = tr.get("source") if tr and traffic else None
    # kernels of ours per step: P1, derivatives, AC z-walk + in-plane tile kernel, SSIM
    # (slab mode adds the on-device P1 state merge); the record memset is not counted
    launches_per_step = (1 + 1 + 2 + 1) if world == 1 else (2 + 1 + 2 + 1)

    # end-to-end through the public host-buffer entry point (H2D + kernels + D2H inside)
    e2e = None
    if not args.no_e2e:
        # czc_assess_host pipelines K = min(8, nz / 4) z-chunks and copies back one record
        # prefix per chunk (czc_sizeof(4) bytes each)
        K = min(8, nz_local // 4) if world == 1 else world
        d2h_host = int(czc.get_lib().czc_sizeof(4)) * (K if K >= 2 else 1)
        xp = xh.pin_memory()
        yp = yh.pin_memory()
        for _ in range(max(3, args.warmup)):            # the H2D path keeps speeding up over the
            a.assess_host(xp, yp, czc.M_ALL, **kw)      # first calls (4.39 -> 4.23 ms); warm it like the kernels
        barrier()
        t0 = time.perf_counter()
        e_tot = 0.0
        for _ in range(max(3, args.steps // 2)):
            s_ev, e_ev = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s_ev.record(stream)
            a.assess_host(xp, yp, czc.M_ALL, **kw)
            e_ev.record(stream)
            e_ev.synchronize()
            e_tot += s_ev.elapsed_time(e_ev)
        nsteps_e2e = max(3, args.steps // 2)
        if world > 1:
            t = torch.tensor([e_tot], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_tot = float(t.item())
        e2e = {"value": round(world * nbytes_rank * nsteps_e2e / (e_tot * 1e-3) / 1e9, 3), "unit": UNIT,
               "h2d_bytes_per_step": nbytes_rank, "d2h_bytes_per_step": d2h_host,
               "ms_per_step": round(e_tot / nsteps_e2e, 4)}

    # float64 inputs (NEXT row f3): the same field widened to double, 16 B per element pair
    f64 = None
    if world == 1 and not args.no_f64:
        xd64, yd64 = xd.double(), yd.double()
        n64 = 2 * xd64.numel() * 8
        with czc.Assessor(ndim=3, device=local, stream=stream, **cfg) as a64, \
                czc.Assessor(ndim=3, device=local, stream=stream, timing=True, **cfg) as t64:
            for _ in range(args.warmup):
                a64.assess(xd64, yd64, czc.M_ALL)
            tot64, k64 = 0.0, []
            for i in range(args.steps):
                flush.zero_()
                clean.sum()
                s_ev, e_ev = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s_ev.record(stream)
                a64.assess(xd64, yd64, czc.M_ALL)
                e_ev.record(stream)
                e_ev.synchronize()
                tot64 += s_ev.elapsed_time(e_ev)
                flush.zero_()
                clean.sum()
                k64.append(t64.assess(xd64, yd64, czc.M_ALL)["kernel_ms"])
        sh64 = {name: statistics.mean(k[i] for k in k64)
                for i, name in enumerate(("P1", "P2_deriv", "P2_autocorr", "P3_ssim"))}
        f64 = {"value": round(n64 * args.steps / (tot64 * 1e-3) / 1e9, 3), "unit": UNIT,
               "ms_per_step": round(tot64 / args.steps, 4), "dtype": "f64",
               "workload": f"the same field widened to float64 ({n64 / 1e6:.0f} MB pair)",
               "per_pattern_ms": {k: round(v, 4) for k, v in sh64.items()},
               "per_pattern_gbs": {k: round(n64 / (v * 1e-3) / 1e9, 2) for k, v in sh64.items() if v > 0}}
        del xd64, yd64

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, dt, cores, desc = oracle_sample(spec, planes=spec.dims[0])
        cpu = {"value": round(v, 6), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": desc,
               "seconds": round(dt, 3)}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(tot_ms / args.steps, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{gspec.name.split('-')[0]} Hurricane-shaped {'x'.join(map(str, gdims))} "
                                   f"float32 pair, abs eb {spec.eb:g}, full metric set (P1, derivatives, "
                                   f"AC lags 1..10, SSIM 8^3 step 1)",
                       "per_rank_planes": nz_local, "parallelism": f"slab{world}",
                       "l2": "flushed between timed steps (256 MB write + 256 MB read of another buffer, "
                                 "outside the step events); the pair (200 MB) is also larger than L2"},
            "per_pattern_ms": {k: round(v, 4) for k, v in shares.items()},
            "per_pattern_gbs": {k: round(alg_bytes / (v * 1e-3) / 1e9, 2) for k, v in shares.items() if v > 0},
            "per_pattern_hbm_frac": {k: round(alg_bytes / (v * 1e-3) / 1e9 / peak, 4)
                                     for k, v in shares.items() if v > 0},
            "roofline": {"bound": "hbm", "kernel": dom, "achieved": round(achieved, 2), "peak": peak,
                         "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                         "peak_source": peak_src, "traffic_source": traffic_src,
                         "algorithmic_bytes_per_launch": alg_bytes},
            "roofline_fp64": {"bound": "alu", "kernel": dom, "achieved": fp64[dom]["achieved"],
                              "peak": round(fp64_peak, 1), "unit": "G FP64 ops/s", "frac": fp64[dom]["frac"],
                              "peak_source": "measured DFMA issue rate (profiles/r01_pipes2.txt) x 148 SMs x 1.965 GHz",
                              "per_pattern": fp64},
            "cpu_baseline": cpu, "e2e": e2e, "float64_inputs": f64,
            "gpu_launches": launches_per_step * args.steps,
            "clocks": clocks, "wall_s_timed_region": round(t_wall, 4),
        }
        print(json.dumps(line), flush=True)
    a.close()
    if world > 1:
        dist.destroy_process_group()


def czc_nccl_uid() -> bytes:
    """ncclGetUniqueId via the NCCL library torch already loaded (128 bytes)."""
    import ctypes
    import glob

    import torch
    cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "nccl", "lib", "libnccl.so*"))
    cands += ["libnccl.so.2"]
    for c in cands:
        try:
            lib = ctypes.CDLL(c)
            buf = ctypes.create_string_buffer(128)
            if lib.ncclGetUniqueId(buf) == 0:
                return buf.raw
        except OSError:
            continue
    raise RuntimeError("cannot load libnccl for ncclGetUniqueId")


def main():
    args = parse()
    rank, world, local = dist_env()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_ours(args, rank, world, local)


if __name__ == "__main__":
    main()
