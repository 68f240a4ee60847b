"""CUDA path vs CPU oracle, element by element on the same seeded inputs, through the C ABI.

Sizes span several tiles with ragged tails; edge cases cover 1-D/2-D, inactive axes, misaligned
pointers, steps, global-range SSIM, zero error, sparse fields and an adversarial step field.
Full-size (BASELINE configs[1]) checks compare all of P1/P2 and sampled SSIM windows."""
import math

import numpy as np
import pytest
import torch

import synth
from parity_util import check_ac, check_deriv, check_p1, check_ssim, report

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def czc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_cluster_yudgtc21_b200 as m
    m.get_lib()
    return m


def run_both(czc, orc, x, y, window=8, step=1, lag=10, range_mode=0, mask=None):
    """GPU (through czc_assess) and oracle on the same host arrays."""
    xn, yn = np.ascontiguousarray(x), np.ascontiguousarray(y)
    xd, yd = torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda()
    nd = xn.ndim
    with czc.Assessor(ndim=nd, ssim_window=window, ssim_step=step, ac_max_lag=lag,
                      ssim_range_mode=range_mode) as a:
        g = a.assess(xd, yd, czc.M_ALL if mask is None else mask)
    o = {}
    o.update(orc.p1(xn, yn))
    o.update(orc.deriv(xn, yn))
    o["ac"], o["ac_count"] = orc.autocorr(xn, yn, lag)
    w = [window] * nd if isinstance(window, int) else list(window)
    s = [step] * nd if isinstance(step, int) else list(step)
    o["ssim"], o["n_windows"] = orc.ssim(xn, yn, w, s, range_mode)
    return g, o


def full_check(g, o, ssim_tol=1e-6):
    errors = []
    check_p1(g, o, errors)
    check_deriv(g, o, errors)
    check_ac(g["ac"], g["ac_count"], o["ac"], o["ac_count"], errors)
    check_ssim(g["ssim"], g["n_windows"], o["ssim"], o["n_windows"], errors, ssim_tol)
    report(errors)


CASES = [
    ("C1", (64, 64, 64), 7),
    ("C1", (13, 17, 35), 5),
    ("C2", (40, 70, 90), 8),
    ("C2q", (36, 66, 75), 8),
    ("C3", (33, 45, 61), 8),
    ("C4", (180, 360), 8),
    ("C4", (77, 1000), 16),
    ("C1", (20, 33, 40), 2),
    ("C2", (9, 300, 41), 3),
]


@pytest.mark.parametrize("cfg,dims,w", CASES)
def test_parity_configs(czc, orc, cfg, dims, w):
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=w)
    assert g["computed_mask"] == czc.M_ALL
    full_check(g, o)


@pytest.mark.parametrize("lag", [1, 4, 16])
def test_lags(czc, orc, lag):
    x, y = synth.make_pair(synth.config("C1", dims=(24, 28, 40)))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=4, lag=lag)
    errors = []
    check_ac(g["ac"], g["ac_count"], o["ac"], o["ac_count"], errors)
    report(errors)


@pytest.mark.parametrize("step", [2, 3, (1, 2, 3)])
def test_steps(czc, orc, step):
    x, y = synth.make_pair(synth.config("C1", dims=(21, 34, 47)))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=5, step=step)
    full_check(g, o)


def test_global_range_mode(czc, orc):
    x, y = synth.make_pair(synth.config("C1", dims=(22, 40, 50)))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=7, range_mode=1)
    full_check(g, o)


def test_one_dimensional_and_inactive_axes(czc, orc):
    x, y = synth.make_pair(synth.config("C4", dims=(7, 1000)))
    xn, yn = x.numpy()[3].copy(), y.numpy()[3].copy()            # 1-D
    g, o = run_both(czc, orc, xn, yn, window=9)
    full_check(g, o)
    x3, y3 = x.numpy()[:, None, :].copy(), y.numpy()[:, None, :].copy()   # (7, 1, 1000)
    g, o = run_both(czc, orc, x3, y3, window=(5, 1, 5))
    full_check(g, o)


def test_zero_error(czc, orc):
    x, _ = synth.make_pair(synth.config("C2q", dims=(20, 30, 40)))
    xn = x.numpy()
    g, o = run_both(czc, orc, xn, xn.copy(), window=6)
    full_check(g, o)
    assert g["psnr"] == math.inf and g["mse"] == 0 and g["ssim"] == 1.0
    assert all(math.isnan(v) for v in g["ac"][1:])


def test_adversarial_step_field(czc, orc):
    x, y = synth.make_pair(synth.config("C1", dims=(18, 20, 64), kind="step", recon="quant", eb=0.1))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=8)
    full_check(g, o)


def test_misaligned_pointers(czc, orc):
    """Same 4-byte offset on both arrays (vector path with prologue) and different offsets
    (scalar path): P1 is flat, so views of a larger buffer exercise both."""
    base_x, base_y = synth.make_pair(synth.config("C1", dims=(5, 77, 131)))
    bx, by = base_x.numpy().ravel(), base_y.numpy().ravel()
    n = 50000
    for ox, oy in ((1, 1), (3, 3), (1, 2), (0, 3)):
        xs = torch.from_numpy(bx).cuda()[ox:ox + n]
        ys = torch.from_numpy(by).cuda()[oy:oy + n]
        with czc.Assessor(ndim=1) as a:
            g = a.assess(xs, ys, czc.M_P1)
        o = orc.p1(bx[ox:ox + n], by[oy:oy + n])
        errors = []
        check_p1(g, o, errors)
        report(errors)


def test_determinism(czc):
    x, y = synth.make_pair(synth.config("C3", dims=(40, 64, 96)))
    xd, yd = x.cuda(), y.cuda()
    outs = []
    with czc.Assessor(ssim_window=8) as a:
        for _ in range(5):
            r = a.assess(xd, yd)
            outs.append({k: (v.tobytes() if isinstance(v, np.ndarray) else v) for k, v in r.items() if k != "kernel_ms"})
    for r in outs[1:]:
        for k in r:
            a_, b_ = r[k], outs[0][k]
            assert a_ == b_ or (isinstance(a_, float) and math.isnan(a_) and math.isnan(b_)), k


def test_errors(czc):
    x = torch.zeros((5, 6, 7), device="cuda")
    with czc.Assessor(ssim_window=8) as a:
        with pytest.raises(czc.CzcError) as ei:
            a.assess(x, x, czc.M_SSIM)               # window larger than the field
        assert ei.value.status == 2
        r = a.assess(x, x, czc.M_P1)                   # the context stays usable
        assert r["computed_mask"] == czc.M_P1
    with czc.Assessor(ssim_window=(8, 4, 8)) as a:
        with pytest.raises(czc.CzcError) as ei:
            a.assess(torch.zeros((20, 20, 20), device="cuda"), torch.zeros((20, 20, 20), device="cuda"), czc.M_SSIM)
        assert ei.value.status == 7


def test_debug_windows_match_oracle(czc, orc):
    x, y = synth.make_pair(synth.config("C2q", dims=(30, 50, 70)))
    xn, yn = x.numpy(), y.numpy()
    w = 8
    nw = [n - w + 1 for n in xn.shape]
    dbg = torch.full(nw, float("nan"), dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=w, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(x.cuda(), y.cuda(), czc.M_SSIM)
    d = dbg.cpu().numpy()
    assert not np.isnan(d).any()
    assert abs(d.mean() - g["ssim"]) < 1e-12
    rng = np.random.default_rng(7)
    for _ in range(300):
        o = [int(rng.integers(0, k)) for k in nw]
        ref = orc.ssim_window(xn, yn, o, [w] * 3)
        assert abs(d[tuple(o)] - ref) < 1e-6, (o, d[tuple(o)], ref)


@pytest.mark.slow
def test_full_size_hurricane(czc, orc):
    """BASELINE configs[1]: 100 x 500 x 500 pair, full metric set, bench launch configuration."""
    spec = synth.CONFIGS["C2"]
    x, y = synth.make_pair(spec)
    xn, yn = x.numpy(), y.numpy()
    nw = [n - 8 + 1 for n in xn.shape]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(x.cuda(), y.cuda())
    errors = []
    check_p1(g, orc.p1(xn, yn), errors)
    check_deriv(g, orc.deriv(xn, yn), errors)
    ac, cnt = orc.autocorr(xn, yn, 10)
    check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
    report(errors)
    d = dbg.cpu().numpy()
    assert g["n_windows"] == np.prod(nw)
    assert abs(d.mean() - g["ssim"]) < 1e-12
    rng = np.random.default_rng(11)
    for _ in range(400):
        o = [int(rng.integers(0, k)) for k in nw]
        ref = orc.ssim_window(xn, yn, o, [8, 8, 8])
        assert abs(d[tuple(o)] - ref) < 1e-6, (o, d[tuple(o)], ref)


@pytest.mark.parametrize("cfg,dims,K,w", [("C2", (40, 70, 90), 2, 8), ("C1", (37, 13, 17), 3, 5),
                                          ("C3", (44, 33, 40), 4, 6), ("C2q", (30, 50, 64), 3, 8),
                                          ("C5", (100, 40, 48), 8, 8)])
def test_loopback_slabs(czc, orc, cfg, dims, K, w):
    """The multi-GPU algorithm (slab ownership, halo buffers, rank-ordered combine) on one GPU:
    K slabs must agree with the oracle on the whole field, and with the single-slab run.  The
    C5 case is the bench's 8-GPU strong-scaling split in miniature: 8 uneven slabs (12-13 planes,
    bench.slab_bounds), each barely deeper than the 10-plane AC halo."""
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    xn, yn = x.numpy(), y.numpy()
    xd, yd = x.cuda(), y.cuda()
    with czc.Assessor(ssim_window=w, ac_max_lag=10, loopback_slabs=K) as a:
        g = a.assess(xd, yd)
    with czc.Assessor(ssim_window=w, ac_max_lag=10) as a:
        g1 = a.assess(xd, yd)
    o = {}
    o.update(orc.p1(xn, yn))
    o.update(orc.deriv(xn, yn))
    o["ac"], o["ac_count"] = orc.autocorr(xn, yn, 10)
    o["ssim"], o["n_windows"] = orc.ssim(xn, yn, [w] * 3)
    full_check(g, o)
    for k in ("x_min", "x_max", "err_min", "err_max", "pwr_min", "pwr_max", "n_pwr", "n_windows",
              "der1_maxabs", "lap_f_min", "grad_f_max"):
        assert g[k] == g1[k], k
    assert abs(g["ssim"] - g1["ssim"]) < 1e-12 and abs(g["mse"] - g1["mse"]) <= 1e-12 * g1["mse"]


def test_nccl_slab_path_single_rank(czc):
    """The NCCL slab path (slab table allgather, halo group, P1 allgather + device merge, record
    allgather + host combine) on a 1-rank communicator must reproduce single-GPU mode."""
    import bench
    if not czc.lib.czc_has_nccl():
        pytest.skip("built without NCCL")
    x, y = synth.make_pair(synth.config("C2", dims=(30, 40, 52)))
    xd, yd = x.cuda(), y.cuda()
    with czc.Assessor(ssim_window=8) as a:
        g1 = a.assess(xd, yd)
    uid = bench.czc_nccl_uid()
    with czc.Assessor(ssim_window=8, rank=0, nranks=1, nccl_uid=uid) as a:
        # repeated calls (cached slab signature), a mask change (new signature: re-validated and
        # re-allocated before any collective), then the first mask again
        for mask in (czc.M_ALL, czc.M_ALL, czc.M_SSIM | czc.M_DERIV, czc.M_ALL):
            g = a.assess(xd, yd, mask, dims=xd.shape, z0=0)
            assert g["computed_mask"] == mask
            for k in ("n_windows", "der1_maxabs", "grad_f_max"):
                assert g[k] == g1[k], k
            assert abs(g["ssim"] - g1["ssim"]) <= 1e-12
    for k in ("x_min", "x_max", "err_min", "err_max", "pwr_max", "n_pwr", "n_windows", "der1_maxabs"):
        assert g[k] == g1[k], k
    for k in ("mse", "psnr", "pearson", "ssim", "der1_mae", "lap_mse"):
        assert abs(g[k] - g1[k]) <= 1e-12 * max(1.0, abs(g1[k])), k
    assert np.allclose(g["ac"], g1["ac"], rtol=0, atol=1e-13)
    with czc.Assessor(ssim_window=8, rank=0, nranks=1, nccl_uid=bench.czc_nccl_uid(), timing=True) as a:
        gt = a.assess(xd, yd, dims=xd.shape, z0=0)                  # per-kernel timing: one stream
    assert gt["ssim"] == g["ssim"] and gt["mse"] == g["mse"] and all(v > 0 for v in gt["kernel_ms"][:5])


@pytest.mark.parametrize("dims,w", [((100, 120, 96), 8), ((23, 31, 40), 5), ((9, 300, 41), 3)])
def test_assess_host_pipelined(czc, orc, dims, w):
    """czc_assess_host (chunked H2D overlapped with per-chunk kernels) vs the oracle and vs
    czc_assess on the same data."""
    x, y = synth.make_pair(synth.config("C2", dims=dims))
    xn, yn = x.numpy(), y.numpy()
    with czc.Assessor(ssim_window=w) as a:
        g = a.assess_host(x.pin_memory(), y.pin_memory())
        gd = a.assess(x.cuda(), y.cuda())
    o = {}
    o.update(orc.p1(xn, yn))
    o.update(orc.deriv(xn, yn))
    o["ac"], o["ac_count"] = orc.autocorr(xn, yn, 10)
    o["ssim"], o["n_windows"] = orc.ssim(xn, yn, [w] * 3)
    full_check(g, o)
    for k in ("x_min", "x_max", "err_maxabs", "pwr_min", "pwr_max", "n_pwr", "n_windows", "n_interior"):
        assert g[k] == gd[k], k


@pytest.mark.parametrize("dims,w", [((20, 24, 40), 2), ((22, 20, 40), 16), ((19, 40, 44), 11), ((24, 33, 50), 12)])
def test_window_extents(czc, orc, dims, w):
    """Small and large window extents (W >= 10 uses the register-heavier 1-block/SM variant)."""
    x, y = synth.make_pair(synth.config("C1", dims=dims))
    xn, yn = x.numpy(), y.numpy()
    with czc.Assessor(ssim_window=w) as a:
        g = a.assess(x.cuda(), y.cuda(), czc.M_SSIM | czc.M_P1)
    s, nw = orc.ssim(xn, yn, [w] * 3)
    errors = []
    check_ssim(g["ssim"], g["n_windows"], s, nw, errors)
    report(errors)


def test_context_reuse_across_shapes(czc, orc):
    """One context, shapes growing and shrinking (scratch reallocation), masks varying."""
    with czc.Assessor(ssim_window=5, ac_max_lag=6) as a:
        for dims, mask in (((10, 12, 14), czc.M_ALL), ((40, 50, 60), czc.M_ALL), ((8, 9, 10), czc.M_P1),
                           ((30, 31, 32), czc.M_DERIV | czc.M_AUTOCORR), ((12, 13, 14), czc.M_SSIM)):
            x, y = synth.make_pair(synth.config("C1", dims=dims))
            xn, yn = x.numpy(), y.numpy()
            g = a.assess(x.cuda(), y.cuda(), mask)
            errors = []
            if mask & czc.M_P1:
                check_p1(g, orc.p1(xn, yn), errors)
            if mask & czc.M_DERIV:
                check_deriv(g, orc.deriv(xn, yn), errors)
            if mask & czc.M_AUTOCORR:
                ac, cnt = orc.autocorr(xn, yn, 6)
                check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
            if mask & czc.M_SSIM:
                s, nw = orc.ssim(xn, yn, [5, 5, 5])
                check_ssim(g["ssim"], g["n_windows"], s, nw, errors)
            report(errors)
            assert g["computed_mask"] == mask


def test_status_codes(czc):
    import ctypes
    lib = czc.get_lib()
    x = torch.zeros((6, 7, 8), device="cuda")
    with czc.Assessor() as a:
        r = czc.Result()
        shape = czc.make_shape([6, 7, 8])
        assert lib.czc_assess(a.ctx, x.data_ptr(), x.data_ptr(), ctypes.byref(shape), 2, czc.M_P1, ctypes.byref(r)) == 3
        bad = czc.make_shape([6, 0, 8])
        assert lib.czc_assess(a.ctx, x.data_ptr(), x.data_ptr(), ctypes.byref(bad), 0, czc.M_P1, ctypes.byref(r)) == 2
        slab = czc.make_shape([6, 7, 8], z0=2, nz_local=3)            # slab shape without ranks
        assert lib.czc_assess(a.ctx, x.data_ptr(), x.data_ptr(), ctypes.byref(slab), 0, czc.M_P1, ctypes.byref(r)) == 2
        assert r.computed_mask == 0
        assert lib.czc_last_error(a.ctx)


def test_timing_fields(czc):
    x, y = synth.make_pair(synth.config("C1", dims=(40, 40, 40)))
    with czc.Assessor(timing=True) as a:
        g = a.assess(x.cuda(), y.cuda())
    ms = g["kernel_ms"]
    assert all(v > 0 for v in ms[:5]) and ms[4] >= sum(ms[:4]) * 0.99


@pytest.mark.slow
@pytest.mark.parametrize("cfg,dims", [("C3", (96, 128, 160)), ("C2q", (100, 160, 200))])
def test_sampled_windows_large(czc, orc, cfg, dims):
    """Per-window SSIM on log-normal (>= 4 decades) and 70 %-zero fields, sampled against the
    oracle's brute-force window; prints the worst error seen (tolerance 1e-6)."""
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    xn, yn = x.numpy(), y.numpy()
    nw = [n - 8 + 1 for n in dims]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        a.assess(x.cuda(), y.cuda(), czc.M_SSIM)
    d = dbg.cpu().numpy()
    rng = np.random.default_rng(5)
    worst = 0.0
    for _ in range(600):
        o = [int(rng.integers(0, k)) for k in nw]
        worst = max(worst, abs(d[tuple(o)] - orc.ssim_window(xn, yn, o, [8, 8, 8])))
    print(f"{cfg} worst sampled window error {worst:.3e}")
    assert worst < 1e-6


def test_misaligned_3d_views(czc, orc):
    """3-D fields whose base pointers are 4-byte (not 16-byte) aligned: the in-plane AC tile
    kernel and the z-walk take their scalar staging paths, everything else must not care."""
    x, y = synth.make_pair(synth.config("C2", dims=(21, 36, 64)))
    n = x.numel()
    for off in (1, 2):
        bx = torch.zeros(n + 8); by = torch.zeros(n + 8)
        bx[off:off + n] = x.ravel(); by[off:off + n] = y.ravel()
        xd = bx.cuda()[off:off + n].view(21, 36, 64)
        yd = by.cuda()[off:off + n].view(21, 36, 64)
        with czc.Assessor(ndim=3, ssim_window=6, ac_max_lag=10) as a:
            g = a.assess(xd, yd, czc.M_ALL)
        xn, yn = x.numpy(), y.numpy()
        o = {}
        o.update(orc.p1(xn, yn)); o.update(orc.deriv(xn, yn))
        o["ac"], o["ac_count"] = orc.autocorr(xn, yn, 10)
        o["ssim"], o["n_windows"] = orc.ssim(xn, yn, [6, 6, 6], [1, 1, 1], 0)
        full_check(g, o)


@pytest.mark.parametrize("kind", ["negated", "scaled"])
def test_sign_flip_and_scaled_recon(czc, orc, kind):
    """Reconstructions far from the original (opposite sign, 2.5x): every float difference is
    inexact in fp32 and many error magnitudes exceed the values."""
    x, y = synth.make_pair(synth.config("C1", dims=(19, 37, 72)))
    xn = x.numpy()
    yn = (-xn + 1e-3 * y.numpy()).astype(np.float32) if kind == "negated" else (2.5 * xn).astype(np.float32)
    g, o = run_both(czc, orc, xn, yn, window=5)
    full_check(g, o)


@pytest.mark.parametrize("dims,lag", [((12, 74, 138), 10), ((11, 32, 64), 10), ((13, 42, 74), 10),
                                      ((20, 50, 90), 16), ((15, 33, 65), 3)])
def test_plane_tile_edges(czc, orc, dims, lag):
    """In-plane AC tiles (64 x 32 + lag halo): fields that end exactly at a tile, at a tile plus
    its halo, one past it, and the 16-lag template."""
    x, y = synth.make_pair(synth.config("C2", dims=dims))
    g, o = run_both(czc, orc, x.numpy(), y.numpy(), window=4, lag=lag)
    errors = []
    check_ac(g["ac"], g["ac_count"], o["ac"], o["ac_count"], errors)
    report(errors)


# ---------------------------------------------------------------- error PDF / pwr-error PDF (f1)
def pdf_check(g, o, nb):
    """Counts are bit-exact (the bin rule is the same IEEE arithmetic on both sides, R24)."""
    assert g["pdf_bins"] == nb
    assert np.array_equal(g["err_pdf"], o["err_pdf"]), (g["err_pdf"] - o["err_pdf"].astype(np.int64))
    assert np.array_equal(g["pwr_pdf"], o["pwr_pdf"]), (g["pwr_pdf"] - o["pwr_pdf"].astype(np.int64))
    for k in ("err_pdf_lo", "err_pdf_width", "pwr_pdf_lo", "pwr_pdf_width"):
        assert g[k] == o[k] or (math.isnan(g[k]) and math.isnan(o[k])), (k, g[k], o[k])


@pytest.mark.parametrize("cfg,dims,nb", [("C1", (30, 41, 53), 100), ("C2", (20, 90, 130), 256),
                                         ("C2q", (17, 60, 77), 64), ("C3", (25, 33, 47), 7),
                                         ("C4", (180, 360), 1), ("C1", (1001,), 13)])
def test_pdf_counts(czc, orc, cfg, dims, nb):
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    xn, yn = x.numpy(), y.numpy()
    with czc.Assessor(ndim=xn.ndim, pdf_bins=nb) as a:
        g = a.assess(torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda(), czc.M_PDF | czc.M_P1)
    assert g["computed_mask"] == czc.M_PDF | czc.M_P1
    pdf_check(g, orc.pdf(xn, yn, nb), nb)


def test_pdf_edge_values_and_degenerate(czc, orc):
    """Errors exactly on bin edges (dyadic construction), a constant error and misaligned views."""
    k = np.repeat(np.arange(17), np.arange(1, 18))
    x = np.ones(k.size, np.float32)
    y = (1.0 + k / 16.0).astype(np.float32)
    for xs, ys in ((x, y), (x, x + np.float32(2.0 ** -10))):
        with czc.Assessor(ndim=1, pdf_bins=4) as a:
            g = a.assess(torch.from_numpy(xs).cuda(), torch.from_numpy(ys).cuda(), czc.M_PDF)
        pdf_check(g, orc.pdf(xs, ys, 4), 4)
    xa, ya = synth.make_pair(synth.config("C2q", dims=(9, 40, 51)))
    xd, yd = xa.cuda().reshape(-1), ya.cuda().reshape(-1)
    for off in (1, 3):
        xv, yv = xd[off:].contiguous(), yd[off:].clone()
        xv = xd[off:]                                        # misaligned view (scalar prologue)
        yv = yd[off:]
        with czc.Assessor(ndim=1, pdf_bins=50) as a:
            g = a.assess(xv, yv, czc.M_PDF)
        pdf_check(g, orc.pdf(xv.cpu().numpy(), yv.cpu().numpy(), 50), 50)


def test_pdf_slab_and_host_paths(czc, orc):
    """Loopback slab mode and the pipelined host path give the single-GPU counts."""
    x, y = synth.make_pair(synth.config("C2", dims=(40, 50, 60)))
    xn, yn = x.numpy(), y.numpy()
    o = orc.pdf(xn, yn, 100)
    for kw in ({"loopback_slabs": 3}, {}):
        with czc.Assessor(ndim=3, pdf_bins=100, **kw) as a:
            g = a.assess(torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda(), czc.M_FULL)
            h = a.assess_host(xn, yn, czc.M_FULL)
        pdf_check(g, o, 100)
        pdf_check(h, o, 100)
        assert g["computed_mask"] == czc.M_FULL


# ------------------------------------------------------------ BASELINE full sizes, maximum size
def _sampled_ssim(orc, xn, yn, d, win, count, seed):
    rng = np.random.default_rng(seed)
    nw = d.shape
    worst = 0.0
    for _ in range(count):
        o = [int(rng.integers(0, k)) for k in nw]
        worst = max(worst, abs(d[tuple(o)] - orc.ssim_window(xn, yn, o, win)))
    return worst


def test_full_size_cesm_2d(czc, orc):
    """BASELINE configs[3]: 1800 x 3600 2-D field, 8 x 8 windows, lags 1..10: P1 / derivatives /
    AC against the oracle over the whole field, SSIM on 400 sampled windows + the exact mean."""
    spec = synth.CONFIGS["C4"]
    x, y = synth.make_pair(spec)
    xn, yn = x.numpy(), y.numpy()
    nw = [n - 8 + 1 for n in xn.shape]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ndim=2, ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(x.cuda(), y.cuda())
    errors = []
    check_p1(g, orc.p1(xn, yn), errors)
    check_deriv(g, orc.deriv(xn, yn), errors)
    ac, cnt = orc.autocorr(xn, yn, 10)
    check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
    report(errors)
    d = dbg.cpu().numpy()
    assert g["n_windows"] == np.prod(nw) and abs(d.mean() - g["ssim"]) < 1e-12
    assert _sampled_ssim(orc, xn, yn, d, [8, 8], 400, 21) < 1e-6


def test_full_size_nyx(czc, orc):
    """BASELINE configs[2]: 512^3 log-normal pair (1.07 GB), full metric set in the bench launch
    configuration: P1, derivatives and AC against the oracle over all 134M elements, SSIM on 300
    sampled windows + the exact mean of the per-window values."""
    spec = synth.CONFIGS["C3"]
    x, y = synth.make_pair(spec)
    xn, yn = x.numpy(), y.numpy()
    nw = [n - 8 + 1 for n in xn.shape]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(x.cuda(), y.cuda())
    errors = []
    check_p1(g, orc.p1(xn, yn), errors)
    check_deriv(g, orc.deriv(xn, yn), errors)
    ac, cnt = orc.autocorr(xn, yn, 10)
    check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
    report(errors)
    d = dbg.cpu().numpy()
    assert g["n_windows"] == np.prod(nw) and abs(d.mean() - g["ssim"]) < 1e-11
    del dbg
    assert _sampled_ssim(orc, xn, yn, d, [8, 8, 8], 300, 31) < 1e-6


def test_ordered_after_default_stream_work(czc):
    """A context made on torch's default stream (handle 0 -> the library's own stream) must see
    the fields that default-stream kernels are still writing: the library stream is blocking, so
    it waits for them (regression: a non-blocking stream read half-written inputs and raced the
    ticket reset)."""
    n = 640
    for _ in range(2):
        x = torch.full((n, n, n), 3.0, dtype=torch.float32, device="cuda")
        y = torch.full((n, n, n), 3.5, dtype=torch.float32, device="cuda")
        with czc.Assessor() as a:
            g = a.assess(x, y, czc.M_P1)
        assert g["n"] == n ** 3 and g["x_min"] == 3.0 and g["err_min"] == 0.5 and g["mse"] == 0.25


def test_maximum_size_closed_forms(czc):
    """BASELINE configs[4] size on ONE GPU: a 2048^3 pair (68.7 GB, 8.6e9 elements) with
    x = v constant and y = v + c (c = 2^-10 exact): every metric has a closed form — e = c,
    MSE = c^2, R = 0 (PSNR = -inf, reading R4), dF = 0, sigma_e^2 = 0 (AC NaN, R12), and every
    window has L = 0 -> 1 (R15): SSIM = A / (A + c^2) with A = 2 v (v + c) + 1e-4.  Exercises
    64-bit element counts, 2^31+ element offsets, the largest grids and the PDF pass."""
    n = 2048
    free, _ = torch.cuda.mem_get_info()
    if free < 2 * n ** 3 * 4 + (4 << 30):
        pytest.skip(f"needs ~70 GB free device memory, have {free / 2**30:.0f} GiB")
    v, c = 280.0, 2.0 ** -10
    x = torch.full((n, n, n), v, dtype=torch.float32, device="cuda")
    y = torch.full((n, n, n), v + c, dtype=torch.float32, device="cuda")
    with czc.Assessor(ssim_window=8, pdf_bins=16) as a:
        g = a.assess(x, y, czc.M_FULL)
    del x, y
    torch.cuda.empty_cache()
    N = n ** 3
    assert g["computed_mask"] == czc.M_FULL and g["n"] == N
    assert g["x_min"] == v and g["x_max"] == v and g["value_range"] == 0.0
    assert g["err_min"] == c and g["err_max"] == c and g["err_maxabs"] == c
    assert g["mse"] == c * c and g["rmse"] == c and g["psnr"] == -math.inf
    assert abs(g["err_mean"] - c) <= 1e-15 and g["err_var"] <= 1e-20
    assert g["n_pwr"] == N and g["pwr_min"] == c / v and g["pwr_max"] == c / v
    assert math.isnan(g["pearson"])
    assert g["n_interior"] == (n - 2) ** 3
    for f in ("der1", "der2", "grad", "div", "lap"):
        assert g[f + "_maxabs"] == 0 and g[f + "_mse"] == 0 and g[f + "_psnr"] == math.inf, f
    assert g["ac_count"][10] == (n - 10) ** 3 and all(math.isnan(t) for t in g["ac"][1:])
    A = 2 * v * (v + c) + 1e-4
    assert g["n_windows"] == (n - 7) ** 3
    assert abs(g["ssim"] - A / (A + c * c)) < 1e-12
    assert g["err_pdf"][0] == N and g["err_pdf_width"] == 0.0 and g["pwr_pdf"][0] == N


# ---------------------------------------------------------------- float64 inputs (NEXT row f3)
def f64_pair(cfg, dims, seed=7):
    """A float64 pair with full 53-bit mantissas: the float32 recipe of `cfg`, the original
    perturbed by 1e-9 relative and the reconstruction error by 1e-6 relative (values no float32
    can hold, so every kernel really reads doubles)."""
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    r = np.random.default_rng(seed)
    xd = x.numpy().astype(np.float64)
    e = y.numpy().astype(np.float64) - xd
    xd = xd * (1.0 + 1e-9 * r.standard_normal(xd.shape))
    yd = xd + e * (1.0 + 1e-6 * r.standard_normal(xd.shape))
    assert np.any(xd.astype(np.float32).astype(np.float64) != xd)
    return xd, yd


@pytest.mark.parametrize("cfg,dims,w", [("C1", (64, 64, 64), 7), ("C2", (40, 70, 90), 8),
                                        ("C2q", (21, 66, 75), 8), ("C3", (33, 45, 61), 6),
                                        ("C4", (180, 360), 8), ("C4", (3, 2001), 5)])
def test_f64_parity_configs(czc, orc, cfg, dims, w):
    xd, yd = f64_pair(cfg, dims)
    if dims[0] == 3:
        xd, yd = xd[1].copy(), yd[1].copy()                      # 1-D
    g, o = run_both(czc, orc, xd, yd, window=w)
    assert g["computed_mask"] == czc.M_ALL
    full_check(g, o)


def test_f64_float_representable_matches_f32_path(czc, orc):
    """Float data widened to double: the float64 kernels must give the float32 kernels' exact
    fields bit for bit and agree with them (and the oracle) within the tolerances elsewhere."""
    x, y = synth.make_pair(synth.config("C2", dims=(30, 50, 70)))
    with czc.Assessor(ssim_window=8) as a:
        g32 = a.assess(x.cuda(), y.cuda(), czc.M_FULL)
        g64 = a.assess(x.double().cuda(), y.double().cuda(), czc.M_FULL)
    for k in ("x_min", "x_max", "err_min", "err_max", "err_maxabs", "pwr_min", "pwr_max", "n_pwr",
              "n_windows", "n_interior", "der1_maxabs", "lap_f_min", "grad_f_max"):
        assert g32[k] == g64[k], k
    assert np.array_equal(g32["err_pdf"], g64["err_pdf"]) and np.array_equal(g32["pwr_pdf"], g64["pwr_pdf"])
    for k in ("mse", "psnr", "pearson", "ssim", "der2_mae", "div_mse"):
        assert abs(g32[k] - g64[k]) <= 1e-12 * max(1.0, abs(g32[k])), k


def test_f64_slab_host_pdf_and_misaligned(czc, orc):
    """float64 through the loopback slab path, the pipelined host path, the PDF pass, and views
    that are 8- but not 16-byte aligned (scalar prologue of the vector path)."""
    xd, yd = f64_pair("C2", (36, 48, 58))
    o = {}
    o.update(orc.p1(xd, yd))
    o.update(orc.deriv(xd, yd))
    o["ac"], o["ac_count"] = orc.autocorr(xd, yd, 10)
    o["ssim"], o["n_windows"] = orc.ssim(xd, yd, [8] * 3)
    tx, ty = torch.from_numpy(xd), torch.from_numpy(yd)
    with czc.Assessor(ssim_window=8, loopback_slabs=3) as a:
        full_check(a.assess(tx.cuda(), ty.cuda()), o)
    with czc.Assessor(ssim_window=8) as a:
        full_check(a.assess_host(tx.pin_memory().numpy(), ty.pin_memory().numpy()), o)
    with czc.Assessor(ndim=1, pdf_bins=64) as a:
        g = a.assess(tx.cuda().reshape(-1), ty.cuda().reshape(-1), czc.M_PDF | czc.M_P1)
        pdf_check(g, orc.pdf(xd.ravel(), yd.ravel(), 64), 64)
        xf, yf = tx.cuda().reshape(-1), ty.cuda().reshape(-1)
        for ox, oy in ((1, 1), (1, 2)):
            n = xf.numel() - 2
            g = a.assess(xf[ox:ox + n], yf[oy:oy + n], czc.M_P1 | czc.M_PDF)
            errors = []
            check_p1(g, orc.p1(xd.ravel()[ox:ox + n], yd.ravel()[oy:oy + n]), errors)
            report(errors)
            pdf_check(g, orc.pdf(xd.ravel()[ox:ox + n], yd.ravel()[oy:oy + n], 64), 64)


def test_f64_dtype_errors(czc):
    x = torch.zeros(4, 5, 6, device="cuda", dtype=torch.float64)
    with czc.Assessor() as a:
        with pytest.raises(TypeError):
            a.assess(x, x.float())
        import ctypes
        r = czc.Result()
        assert czc.lib.czc_assess(a.ctx, x.data_ptr(), x.data_ptr(), ctypes.byref(czc.make_shape([4, 5, 6])),
                                  2, czc.M_P1, ctypes.byref(r)) == 3


# ----------------------------------------------------------------- 4-D fields (NEXT row f3, L92)
def pair4(cfg, shape4, dtype=np.float32):
    """A 4-D pair: the `cfg` recipe generated as a 3-D field (n0 n1, n2, n3) and viewed in 4-D."""
    x, y = synth.make_pair(synth.config(cfg, dims=(shape4[0] * shape4[1],) + tuple(shape4[2:])))
    return (x.numpy().reshape(shape4).astype(dtype), y.numpy().reshape(shape4).astype(dtype))


@pytest.mark.parametrize("cfg,shape,w,step,lag", [("C1", (7, 9, 10, 12), 3, 1, 4), ("C2", (6, 8, 20, 24), 4, (1, 2, 1, 3), 6),
                                                  ("C2q", (5, 6, 17, 19), 5, 1, 10), ("C3", (8, 5, 9, 33), 2, 2, 3)])
def test_4d_parity(czc, orc, cfg, shape, w, step, lag):
    x, y = pair4(cfg, shape)
    g, o = run_both(czc, orc, x, y, window=w, step=step, lag=lag)
    assert g["computed_mask"] == czc.M_ALL and g["n_interior"] == np.prod([n - 2 for n in shape])
    full_check(g, o)


def test_4d_float64_pdf_debug_and_modes(czc, orc):
    x, y = pair4("C2", (6, 7, 11, 13), np.float64)
    y = y + 1e-7 * np.random.default_rng(3).standard_normal(y.shape)
    g, o = run_both(czc, orc, x, y, window=3, lag=5)
    full_check(g, o)
    nw = [n - 3 + 1 for n in x.shape]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ndim=4, ssim_window=3, pdf_bins=40, ssim_range_mode=1, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda(), czc.M_FULL)
    pdf_check(g, orc.pdf(x.ravel(), y.ravel(), 40), 40)
    s, n = orc.ssim(x, y, [3] * 4, None, 1)
    assert g["n_windows"] == n and abs(g["ssim"] - s) < 1e-6
    d = dbg.cpu().numpy()
    R = float(x.max() - x.min())
    for o4 in ((0, 0, 0, 0), (3, 4, 8, 10), (1, 2, 5, 7)):
        assert abs(d[o4] - orc.ssim_window(x, y, o4, [3] * 4, 1, R)) < 1e-9


def test_4d_squeezed_and_unsupported(czc, orc):
    """A 4-D shape with an extent-1 axis is a 3-D field (streamed engines, identical results);
    four active axes refuse slab mode."""
    x, y = synth.make_pair(synth.config("C1", dims=(12, 14, 16)))
    with czc.Assessor(ndim=3, ssim_window=4) as a:
        g3 = a.assess(x.cuda(), y.cuda())
    with czc.Assessor(ndim=4, ssim_window=4) as a:
        g4 = a.assess(x.cuda().reshape(12, 1, 14, 16), y.cuda().reshape(12, 1, 14, 16))
    for k in ("x_min", "err_max", "mse", "ssim", "n_windows", "der1_mae", "n_interior"):
        assert g3[k] == g4[k], k
    assert np.array_equal(g3["ac"], g4["ac"])
    x4 = x.cuda().reshape(3, 4, 14, 16)
    with czc.Assessor(ndim=4, ssim_window=3, loopback_slabs=2) as a:
        with pytest.raises(czc.CzcError) as ei:
            a.assess(x4, x4)
        assert ei.value.status == 7


def test_graph_replay_sees_new_contents_and_plans(czc, orc):
    """The single-GPU sequence replays as a CUDA graph while the call signature repeats: new
    contents in the same buffers must be read, and a different mask / window (new signature)
    must re-capture, then returning to the first signature must be right again."""
    x, y = synth.make_pair(synth.config("C2", dims=(20, 40, 48)))
    xd, yd = x.cuda(), y.cuda()
    with czc.Assessor(ssim_window=5) as a:
        for it in range(3):
            if it:
                yd.copy_(xd + (yd - xd) * (1.0 + it))             # same buffers, new contents
            g = a.assess(xd, yd)
            xn, yn = xd.cpu().numpy(), yd.cpu().numpy()
            errors = []
            check_p1(g, orc.p1(xn, yn), errors)
            check_ssim(g["ssim"], g["n_windows"], *orc.ssim(xn, yn, [5] * 3), errors)
            report(errors)
            gp = a.assess(xd, yd, czc.M_P1 | czc.M_PDF)           # another signature in between
            assert gp["computed_mask"] == czc.M_P1 | czc.M_PDF and gp["mse"] == g["mse"]


def test_full_size_hurricane_float64(czc, orc):
    """BASELINE configs[1] shape with float64 inputs (the field widened with a 1e-9 relative
    perturbation, 400 MB pair): P1, derivatives and AC against the float64 oracle over all 25 M
    elements, the exact mean of the per-window SSIM values, 200 sampled windows."""
    spec = synth.CONFIGS["C2"]
    x, y = synth.make_pair(spec)
    r = np.random.default_rng(17)
    xn = x.numpy().astype(np.float64) * (1.0 + 1e-9 * r.standard_normal(spec.dims))
    yn = xn + (y.numpy().astype(np.float64) - x.numpy().astype(np.float64))
    nw = [n - 8 + 1 for n in xn.shape]
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda())
    errors = []
    check_p1(g, orc.p1(xn, yn), errors)
    check_deriv(g, orc.deriv(xn, yn), errors)
    ac, cnt = orc.autocorr(xn, yn, 10)
    check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
    report(errors)
    d = dbg.cpu().numpy()
    assert g["n_windows"] == np.prod(nw) and abs(d.mean() - g["ssim"]) < 1e-12
    for _ in range(200):
        o = [int(r.integers(0, k)) for k in nw]
        assert abs(d[tuple(o)] - orc.ssim_window(xn, yn, o, [8, 8, 8])) < 1e-6, o


@pytest.mark.slow
def test_full_size_2048_cubed_smooth_pair(czc, orc):
    """BASELINE configs[4] (C5) at its full size on ONE GPU, in the bench's launch configuration:
    the smooth 2048^3 pair of the C5 recipe (68.7 GB, 8.6e9 elements; generated on the device,
    bit-identical to the CPU recipe for this kind) against the oracle over the WHOLE field for P1,
    the derivative metrics and AC lags 1..10, and the local SSIM of 1500 sampled windows plus the
    exact mean of all 8.5e9 per-window values (VERDICT r1 missing #3: the only 2048^3 check was a
    constant field, where no window has a non-zero variance)."""
    import bench
    n = 2048
    free, _ = torch.cuda.mem_get_info()
    if free < 2 * n ** 3 * 4 + (n - 7) ** 3 * 8 + (6 << 30):
        pytest.skip(f"needs ~145 GB free device memory, have {free / 2**30:.0f} GiB")
    spec = synth.CONFIGS["C5"]
    xd, yd = bench.make_slab_device(spec, 0, n, torch.device("cuda", torch.cuda.current_device()), 1)
    nw = [n - 7] * 3
    dbg = torch.empty(nw, dtype=torch.float64, device="cuda")
    with czc.Assessor(ssim_window=8, debug_wssim=dbg.data_ptr()) as a:
        g = a.assess(xd, yd, czc.M_ALL)
    assert g["computed_mask"] == czc.M_ALL and g["n_windows"] == (n - 7) ** 3
    mean_dbg = float(dbg.sum(dtype=torch.float64).item()) / dbg.numel()
    assert abs(mean_dbg - g["ssim"]) < 1e-11
    rng = np.random.default_rng(2048)
    org = rng.integers(0, n - 7, size=(1500, 3))
    oi = torch.from_numpy(org).cuda()
    gw = dbg[oi[:, 0], oi[:, 1], oi[:, 2]].cpu().numpy()
    slab_mean = float(dbg[:256].sum(dtype=torch.float64).item()) / dbg[:256].numel()
    del dbg
    xn, yn = xd.cpu().numpy(), yd.cpu().numpy()
    del xd, yd
    torch.cuda.empty_cache()
    worst = max(abs(gw[i] - orc.ssim_window(xn, yn, list(org[i]), [8, 8, 8])) for i in range(len(org)))
    assert worst < 1e-6, worst
    # the mean of the 1.06e9 windows with origin planes 0..255 (an eighth of the field) against the
    # separable oracle (brute force would take ~5e11 element visits)
    sep, nws, nbr = orc.ssim_separable(xn[:263], yn[:263], [8, 8, 8])
    assert nws == 256 * (n - 7) ** 2 and abs(slab_mean - sep) < 1e-9, (slab_mean, sep, nbr)
    import time
    t0 = time.perf_counter()
    errors = []
    check_p1(g, orc.p1(xn, yn), errors)
    check_deriv(g, orc.deriv(xn, yn), errors)
    ac, cnt = orc.autocorr(xn, yn, 10)
    check_ac(g["ac"], g["ac_count"], ac, cnt, errors)
    report(errors)
    print(f"oracle over 2048^3: {time.perf_counter() - t0:.0f} s on {orc.threads()} threads")
    print(f"C5 2048^3: psnr {g['psnr']:.4f} ssim {g['ssim']:.9f} exact windows {g['n_ssim_exact']} "
          f"worst sampled window {worst:.2e}; planes 0..255: gpu mean {slab_mean:.15f} separable "
          f"oracle {sep:.15f} ({nbr} brute-forced)")
