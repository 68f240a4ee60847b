"""Host-only checks of czc_combine (the rank-ordered combine + finish of slab mode) without a GPU,
including a world_size-2 gloo run: each rank builds the partial record of its slab from numpy
(ownership rules of DESIGN.md §7), the records are all-gathered over gloo, every rank combines
them and must reproduce the whole-field oracle."""
import math
import os
import struct

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from parity_util import check_ac, check_deriv, check_p1, check_ssim, report

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _czc():
    from paper_conf_cluster_yudgtc21_b200 import build
    build.build()
    import paper_conf_cluster_yudgtc21_b200 as m
    return m


# Record layout (mirrors czc_internal.cuh `Record`): P1State {n, mx, my, me, m2x, m2y, cxy, m2e, sae,
# emin, emax, pmin, pmax, spwr, npwr, xmin, xmax : double}, deriv[25], ac[3][16], ssim[3],
# pdf[2][256] (uint64 counts of the error / pwr-error PDFs, binned over the GLOBAL ranges).
PDF_MAX = 256


def pdf_counts(x, y, xg, yg, nb):
    """Counts of this slab's values in the bins of the whole field (reading R24's bin rule)."""
    def bins(v, lo, hi):
        w = (hi - lo) / nb
        if not (w > 0):
            return np.zeros(v.shape, dtype=np.int64)
        b = np.floor((v - lo) / w).astype(np.int64)
        return np.clip(b, 0, nb - 1)
    e = y.astype(np.float64).ravel() - x.astype(np.float64).ravel()
    eg = yg.astype(np.float64).ravel() - xg.astype(np.float64).ravel()
    nzg = xg.ravel() != 0
    qg = np.abs(eg[nzg]) / np.abs(xg.astype(np.float64).ravel()[nzg])
    nz = x.ravel() != 0
    q = np.abs(e[nz]) / np.abs(x.astype(np.float64).ravel()[nz])
    ce = np.bincount(bins(e, eg.min(), eg.max()), minlength=PDF_MAX)
    cp = np.bincount(bins(q, qg.min(), qg.max()), minlength=PDF_MAX) if q.size else np.zeros(PDF_MAX, np.int64)
    return struct.pack(f"<{2 * PDF_MAX}Q", *[int(v) for v in ce], *[int(v) for v in cp])
def p1_state(x, y):
    xd, yd = x.astype(np.float64).ravel(), y.astype(np.float64).ravel()
    e = yd - xd
    nz = x.ravel() != 0
    q = np.abs(e[nz]) / np.abs(xd[nz])
    vals = [float(xd.size), xd.mean(), yd.mean(), e.mean(), ((xd - xd.mean()) ** 2).sum(),
            ((yd - yd.mean()) ** 2).sum(), ((xd - xd.mean()) * (yd - yd.mean())).sum(),
            ((e - e.mean()) ** 2).sum(), np.abs(e).sum(), e.min(), e.max(),
            q.min() if q.size else math.inf, q.max() if q.size else -math.inf, q.sum(), float(q.size)]
    return struct.pack("<17d", *vals, float(x.min()), float(x.max()))


def deriv_fields(f):
    f = f.astype(np.float64)
    c = f[1:-1, 1:-1, 1:-1]
    out = {k: 0.0 for k in ("der1", "der2", "g2", "div", "lap")}
    for a in range(3):
        sl_p = [slice(1, -1)] * 3
        sl_m = [slice(1, -1)] * 3
        sl_p[a] = slice(2, None)
        sl_m[a] = slice(0, -2)
        fp, fm = f[tuple(sl_p)], f[tuple(sl_m)]
        d = fp - fm
        l = fp - 2 * c + fm
        out["der1"] = out["der1"] + np.abs(d)
        out["der2"] = out["der2"] + np.abs(l)
        out["g2"] = out["g2"] + (d / 2) ** 2
        out["div"] = out["div"] + d / 2
        out["lap"] = out["lap"] + l
    return [out["der1"], out["der2"], np.sqrt(out["g2"]), out["div"], out["lap"]]


def record(x, y, z0, z1, w, T=10, nb=0):
    """The record of slab [z0, z1) computed with numpy from the whole field (ownership rules)."""
    nz = x.shape[0]
    rec = p1_state(x[z0:z1], y[z0:z1])
    Fx, Fy = deriv_fields(x), deriv_fields(y)      # interior points, z index = 1..nz-2
    zi = np.arange(1, nz - 1)
    own = (zi >= z0) & (zi < z1)
    dslots = []
    for fx, fy in zip(Fx, Fy):
        fx, fy = fx[own], fy[own]
        d = fy - fx
        if d.size:
            dslots += [np.abs(d).max(), np.abs(d).sum(), (d * d).sum(), fx.min(), fx.max()]
        else:
            dslots += [-math.inf, 0.0, 0.0, math.inf, -math.inf]
    rec += struct.pack("<25d", *dslots)
    e = y.astype(np.float64) - x.astype(np.float64)
    eps = e - e.mean()
    ac = np.zeros((3, 16))
    for t in range(1, min(T, min(e.shape) - 1) + 1):
        R = tuple(slice(0, n - t) for n in e.shape)
        zz = np.arange(nz - t)
        ownz = (zz >= z0) & (zz < z1)
        c = eps[R][ownz]
        for a in range(3):
            sh = [slice(0, n - t) for n in e.shape]
            sh[a] = slice(t, sh[a].stop + t)
            ac[a, t - 1] = np.sum(c * eps[tuple(sh)][ownz])
    rec += struct.pack("<48d", *ac.ravel())
    import oracle
    s, cnt = 0.0, 0
    for oz in range(max(z0, 0), min(z1, nz - w + 1)):
        for oy in range(x.shape[1] - w + 1):
            for ox in range(x.shape[2] - w + 1):
                s += oracle.ssim_window(x, y, [oz, oy, ox], [w, w, w])
                cnt += 1
    rec += struct.pack("<3d", s, float(cnt), 0.0)
    rec += pdf_counts(x[z0:z1], y[z0:z1], x, y, nb) if nb else bytes(16 * PDF_MAX)
    return rec


def compare(g, o):
    errors = []
    check_p1(g, o, errors)
    check_deriv(g, o, errors)
    check_ac(g["ac"], g["ac_count"], o["ac"], o["ac_count"], errors)
    check_ssim(g["ssim"], g["n_windows"], o["ssim"], o["n_windows"], errors)
    report(errors)


def oracle_all(x, y, w):
    import oracle
    o = {}
    o.update(oracle.p1(x, y))
    o.update(oracle.deriv(x, y))
    o["ac"], o["ac_count"] = oracle.autocorr(x, y, 10)
    o["ssim"], o["n_windows"] = oracle.ssim(x, y, [w] * 3)
    return o


def test_record_size_matches(orc):
    czc = _czc()
    x, y = synth.make_pair(synth.config("C1", dims=(8, 9, 10)))
    assert len(record(x.numpy(), y.numpy(), 0, 8, 3)) == czc.lib.czc_sizeof(3)


@pytest.mark.parametrize("cuts", [(0, 12), (0, 5, 12), (0, 3, 7, 12)])
def test_combine_matches_oracle(orc, cuts):
    czc = _czc()
    x, y = synth.make_pair(synth.config("C1", dims=(12, 11, 13)))
    xn, yn = x.numpy(), y.numpy()
    w = 4
    recs = b"".join(record(xn, yn, a, b, w) for a, b in zip(cuts[:-1], cuts[1:]))
    cfg = czc.make_config(ndim=3, ssim_window=w, ac_max_lag=10)
    g = czc.czc_combine(recs, len(cuts) - 1, xn.shape, cfg)
    compare(g, oracle_all(xn, yn, w))


def test_combine_pdf_counts(orc):
    """Per-slab PDF counts over the global ranges, summed in slab order, equal the oracle's."""
    czc = _czc()
    import oracle
    x, y = synth.make_pair(synth.config("C2q", dims=(10, 9, 12)))
    xn, yn = x.numpy(), y.numpy()
    w, nb = 3, 37
    cuts = (0, 4, 10)
    recs = b"".join(record(xn, yn, a, b, w, nb=nb) for a, b in zip(cuts[:-1], cuts[1:]))
    cfg = czc.make_config(ndim=3, ssim_window=w, ac_max_lag=10, pdf_bins=nb)
    g = czc.czc_combine(recs, len(cuts) - 1, xn.shape, cfg, czc.M_FULL)
    o = oracle.pdf(xn, yn, nb)
    assert g["computed_mask"] == czc.M_FULL and g["pdf_bins"] == nb
    assert np.array_equal(g["err_pdf"], o["err_pdf"]) and np.array_equal(g["pwr_pdf"], o["pwr_pdf"])
    for k in ("err_pdf_lo", "err_pdf_width", "pwr_pdf_lo", "pwr_pdf_width"):
        assert g[k] == o[k], k


def _worker(rank, world, port, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    czc = _czc()
    x, y = synth.make_pair(synth.config("C2q", dims=(14, 12, 11)))
    xn, yn = x.numpy(), y.numpy()
    w = 5
    nz = xn.shape[0]
    z0, z1 = nz * rank // world, nz * (rank + 1) // world
    mine = torch.frombuffer(bytearray(record(xn, yn, z0, z1, w)), dtype=torch.uint8)
    gathered = [torch.empty_like(mine) for _ in range(world)]
    dist.all_gather(gathered, mine)
    recs = b"".join(bytes(t.numpy()) for t in gathered)
    cfg = czc.make_config(ndim=3, ssim_window=w, ac_max_lag=10)
    g = czc.czc_combine(recs, world, xn.shape, cfg)
    ok = True
    try:
        compare(g, oracle_all(xn, yn, w))
    except AssertionError as e:
        ok = str(e)
    out_q.put((rank, ok, g["ssim"], g["mse"]))
    dist.destroy_process_group()


def test_gloo_world2_combine(orc):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + os.getpid() % 1000
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    res.sort()
    assert all(r[1] is True for r in res), res
    assert res[0][2] == res[1][2] and res[0][3] == res[1][3]   # identical results on every rank
