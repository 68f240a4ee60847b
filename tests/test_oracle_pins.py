"""Pins of the CPU oracle to things other than itself (no GPU needed).

Each test fixes an oracle function against a closed form, an invariant, a library routine that
implements the same definition independently (numpy / scipy), or brute force on tiny inputs —
chosen so that a dropped term, a wrong sign or index, or a transposed operand fails one of them.
Citations: PAPER.md line numbers (Lnnn); readings R1..R23 are DESIGN.md §2.
"""
import math

import numpy as np
import pytest
import scipy.ndimage as ndi

import synth

rng = np.random.default_rng(1234)


def dyadic_field(shape, scale=2.0 ** -20, lo=-(2 ** 18), hi=2 ** 18):
    """Values on a 2^-20 grid with |x| < 1/4: float32-exact, and x + 2^-10 stays exact."""
    return (rng.integers(lo, hi, size=shape).astype(np.float64) * scale).astype(np.float32)


# ------------------------------------------------------------------------------------------ P1
class TestP1:
    def test_zero_error(self, orc):
        """y = x: every error statistic is 0, PSNR = SNR = +inf, Pearson = 1 (north_star)."""
        x = dyadic_field((9, 10, 11))
        x[0, 0, :3] = 0.0
        r = orc.p1(x, x)
        for k in ("err_min", "err_max", "err_maxabs", "err_mean", "err_absmean", "mse", "rmse",
                  "nrmse", "max_rel_err", "pwr_min", "pwr_max", "pwr_mean", "err_var"):
            assert r[k] == 0.0, k
        assert r["psnr"] == math.inf and r["snr"] == math.inf
        assert abs(r["pearson"] - 1.0) < 1e-15
        assert r["n_pwr"] == int(np.count_nonzero(x)) and r["n"] == x.size

    def test_dyadic_offset_closed_form(self, orc):
        """e == c exactly (dyadic grid): MSE = c^2 bit-exact, RMSE = c, PSNR = 20 log10(R/c)."""
        x = dyadic_field((7, 13, 17))
        c = 2.0 ** -10
        y = (x.astype(np.float64) + c).astype(np.float32)
        assert np.all(y.astype(np.float64) - x.astype(np.float64) == c)
        r = orc.p1(x, y)
        R = float(x.max()) - float(x.min())
        assert r["mse"] == c * c and r["rmse"] == c and r["err_mean"] == c
        assert r["err_min"] == c == r["err_max"] == r["err_maxabs"] == r["err_absmean"]
        assert r["err_var"] == 0.0
        assert r["value_range"] == R and r["max_rel_err"] == c / R
        assert abs(r["psnr"] - 20 * math.log10(R / c)) < 1e-12
        assert abs(r["nrmse"] - c / R) < 1e-18
        assert abs(r["pearson"] - 1.0) < 1e-15

    def test_uniform_noise_psnr_statistical(self, orc):
        """C1 recipe, e ~ U[-a, a]: E[MSE] = a^2/3 (rel. sd 0.894/sqrt(N)), E[e] = 0 (sd a/sqrt(3N))."""
        spec = synth.CONFIGS["C1"]
        x, y = synth.make_pair(spec)
        r = orc.p1(x, y)
        a, N = spec.eb, x.numel()
        assert abs(r["mse"] / (a * a / 3) - 1) < 4 * 0.894 / math.sqrt(N)
        assert abs(r["err_mean"]) < 4 * a / math.sqrt(3 * N)
        expect_psnr = 20 * math.log10(r["value_range"]) - 10 * math.log10(a * a / 3)
        assert abs(r["psnr"] - expect_psnr) < 4 * 10 / math.log(10) * 0.894 / math.sqrt(N)
        assert r["err_maxabs"] <= a * (1 + 1e-6)

    @pytest.mark.parametrize("cfg", ["C1", "C2q"])
    def test_against_numpy(self, orc, cfg):
        """Independent numpy float64 formulations (pairwise sums) of every P1 definition."""
        spec = synth.config(cfg, dims=(20, 30, 40))
        x, y = synth.make_pair(spec)
        x, y = x.numpy(), y.numpy()
        r = orc.p1(x, y)
        xd, yd = x.astype(np.float64), y.astype(np.float64)
        e = yd - xd
        assert r["x_min"] == float(x.min()) and r["x_max"] == float(x.max())
        assert r["err_min"] == e.min() and r["err_max"] == e.max() and r["err_maxabs"] == np.abs(e).max()
        nz = x != 0
        q = np.abs(e[nz]) / np.abs(xd[nz])
        assert r["n_pwr"] == int(nz.sum())
        assert r["pwr_min"] == q.min() and r["pwr_max"] == q.max()
        assert abs(r["pwr_mean"] - q.mean()) <= 1e-12 * q.mean()
        assert abs(r["mse"] - np.mean(e * e)) <= 1e-12 * r["mse"]
        assert abs(r["err_var"] - np.var(e)) <= 1e-10 * r["err_var"]
        assert abs(r["err_absmean"] - np.mean(np.abs(e))) <= 1e-12 * r["err_absmean"]
        assert abs(r["err_mean"] - np.mean(e)) <= 1e-12 * r["err_absmean"]
        assert abs(r["pearson"] - np.corrcoef(xd.ravel(), yd.ravel())[0, 1]) < 1e-12
        snr = 10 * np.log10(np.sum((xd - xd.mean()) ** 2) / np.sum(e * e))
        assert abs(r["snr"] - snr) < 1e-9

    def test_pearson_large_mean(self, orc):
        """1e5 +- 100 field (condition ~ mean^2/var): two-pass Pearson vs numpy corrcoef (centred)."""
        x = (1e5 + 100 * rng.standard_normal(4096)).astype(np.float32)
        y = (x.astype(np.float64) + rng.uniform(-0.01, 0.01, 4096)).astype(np.float32)
        r = orc.p1(x, y)
        ref = np.corrcoef(x.astype(np.float64), y.astype(np.float64))[0, 1]
        assert abs(r["pearson"] - ref) < 1e-13
        assert 1 - ref > 1e-10            # the quantity really is resolved

    def test_degenerate(self, orc):
        """Constant original: R = 0 -> PSNR -inf when MSE > 0, Pearson NaN; all-zero x: pwr NaN."""
        x = np.full(64, 3.0, np.float32)
        y = x + np.float32(0.5)
        r = orc.p1(x, y)
        assert r["value_range"] == 0 and r["psnr"] == -math.inf and math.isnan(r["pearson"])
        assert r["nrmse"] == math.inf
        z = np.zeros(16, np.float32)
        r = orc.p1(z, z + np.float32(1))
        assert r["n_pwr"] == 0 and math.isnan(r["pwr_max"]) and math.isnan(r["pwr_mean"])


# ------------------------------------------------------------------------------------------ P2
def _interior(a):
    return a[tuple(slice(1, -1) if n > 1 else slice(None) for n in a.shape)]


def _fields_numpy(f):
    """Derived fields via library routines: numpy.gradient (central /2) and scipy laplace."""
    f = f.astype(np.float64)
    axes = [a for a, n in enumerate(f.shape) if n > 1]
    D = [np.gradient(f, axis=a) for a in axes]          # interior: (f(p+1) - f(p-1)) / 2
    der1 = sum(2 * np.abs(d) for d in D)
    grad = np.sqrt(sum(d * d for d in D))
    div = sum(D)
    lap = ndi.laplace(f, mode="nearest")                 # interior: sum_a f(+1) - 2 f + f(-1)
    sec = []
    for a in axes:
        s = np.zeros_like(f)
        sl = [slice(None)] * f.ndim
        sl[a] = slice(1, -1)
        hi = list(sl); hi[a] = slice(2, None)
        lo = list(sl); lo[a] = slice(0, -2)
        s[tuple(sl)] = f[tuple(hi)] - 2 * f[tuple(sl)] + f[tuple(lo)]
        sec.append(s)
    der2 = sum(np.abs(s) for s in sec)
    return {k: _interior(v) for k, v in
            dict(der1=der1, der2=der2, grad=grad, div=div, lap=lap).items()}


class TestDeriv:
    def test_dyadic_ramp(self, orc):
        """f = sum_a c_a p_a: D_a = c_a, Delta_a = 0 -> Der1 = 2 sum|c|, Grad = |c|, Lap = 0 (L122, L129)."""
        shape = (6, 7, 9)
        p = np.indices(shape).astype(np.float64)
        c = np.array([2 ** -3, -(2 ** -4), 2 ** -5])
        cy = np.array([2 ** -3, 2 ** -4, 2 ** -6])
        x = np.tensordot(c, p, 1).astype(np.float32) + np.float32(1)
        y = np.tensordot(cy, p, 1).astype(np.float32) + np.float32(1)
        r = orc.deriv(x, y)
        assert r["n_interior"] == 4 * 5 * 7
        assert r["der1_f_min"] == r["der1_f_max"] == 2 * np.abs(c).sum()
        assert r["grad_f_min"] == pytest.approx(math.sqrt((c ** 2).sum()), abs=1e-15)
        assert r["div_f_max"] == c.sum() and r["lap_f_max"] == 0 and r["der2_f_max"] == 0
        d1 = 2 * (np.abs(cy).sum() - np.abs(c).sum())
        assert r["der1_maxabs"] == abs(d1) and r["der1_mae"] == abs(d1) and r["der1_mse"] == d1 * d1
        dd = cy.sum() - c.sum()
        assert r["div_maxabs"] == abs(dd) and r["div_mse"] == dd * dd
        assert r["lap_maxabs"] == 0 and r["lap_psnr"] == math.inf

    def test_quadratic(self, orc):
        """f = sum_a q_a p_a^2: Delta_a = 2 q_a exactly -> Lap = 2 sum q, Der2 = 2 sum |q|."""
        shape = (5, 6, 7)
        p = np.indices(shape).astype(np.float64)
        q = np.array([2 ** -4, -(2 ** -5), 2 ** -3])
        x = np.tensordot(q, p ** 2, 1).astype(np.float32)
        r = orc.deriv(x, x)
        assert r["lap_f_min"] == r["lap_f_max"] == 2 * q.sum()
        assert r["der2_f_min"] == r["der2_f_max"] == 2 * np.abs(q).sum()
        assert r["lap_mse"] == 0 and r["der1_maxabs"] == 0

    def test_finite_psnr_rmse_closed_form(self, orc):
        """Finite per-field PSNR / RMSE.  x = alpha z^2 + beta p_x, y = x +
        gamma p_y (dyadic, exact in float32): on the interior (z = 1..nz-2)
          Div(x) = 2 alpha z + beta  (range 2 alpha (nz - 3)),
        with D_a = (f(+1) - f(-1)) / 2: D_z x = 2 alpha z, D_x x = beta, D_y y - D_y x = gamma, so
          dDiv = gamma, dDer1 = |2 gamma| (Eq. 1 has no 1/2), dLap = 0, dDer2 = 0,
          Der1(x) = 4 alpha z + 2 beta (range 4 alpha (nz - 3)),
          Grad(x) = sqrt((2 alpha z)^2 + beta^2),  Grad(y) = sqrt((2 alpha z)^2 + beta^2 + gamma^2).
        PSNR_F = 20 log10(max F(x) - min F(x)) - 10 log10(mse_F): the range of the ORIGINAL's field
        and 20 vs 10 are both pinned (a range of F(y), or 10 log10 of the range, fails)."""
        nz, ny, nx = 11, 6, 7
        a, b, g = 2.0 ** -4, 2.0 ** -3, 2.0 ** -5
        z, yy, xx = np.indices((nz, ny, nx)).astype(np.float64)
        x = (a * z * z + b * xx).astype(np.float32)
        y = (a * z * z + b * xx + g * yy).astype(np.float32)
        assert np.all(y.astype(np.float64) - x.astype(np.float64) == g * yy)
        r = orc.deriv(x, y)
        nI = (nz - 2) * (ny - 2) * (nx - 2)
        assert r["n_interior"] == nI
        zi = np.arange(1, nz - 1, dtype=np.float64)
        # Div: constant error gamma, range 2 alpha (nz - 3)
        assert r["div_maxabs"] == g and r["div_mae"] == g and r["div_mse"] == g * g and r["div_rmse"] == g
        assert r["div_f_min"] == 2 * a * 1 + b and r["div_f_max"] == 2 * a * (nz - 2) + b
        assert r["div_psnr"] == pytest.approx(20 * math.log10(2 * a * (nz - 3)) - 10 * math.log10(g * g), abs=1e-12)
        # Der1: constant error 2 gamma, range 4 alpha (nz - 3)
        assert r["der1_mse"] == 4 * g * g and r["der1_rmse"] == 2 * g
        assert r["der1_psnr"] == pytest.approx(20 * math.log10(4 * a * (nz - 3)) - 10 * math.log10(4 * g * g), abs=1e-12)
        # Lap / Der2: zero error -> +inf
        assert r["lap_mse"] == 0 and r["lap_psnr"] == math.inf and r["der2_psnr"] == math.inf
        # Grad: per-plane closed form, mean over the interior
        gx = np.sqrt((2 * a * zi) ** 2 + b * b)
        gy = np.sqrt((2 * a * zi) ** 2 + b * b + g * g)
        mse = float(np.mean((gy - gx) ** 2))
        assert r["grad_mse"] == pytest.approx(mse, rel=1e-13)
        assert r["grad_rmse"] == pytest.approx(math.sqrt(mse), rel=1e-13)
        assert r["grad_maxabs"] == pytest.approx(float(np.max(gy - gx)), rel=1e-13)
        rng = gx.max() - gx.min()
        assert r["grad_psnr"] == pytest.approx(20 * math.log10(rng) - 10 * math.log10(mse), abs=1e-10)

    @pytest.mark.parametrize("shape", [(12, 14, 16), (30, 40), (9, 1, 33)])
    def test_against_numpy_scipy(self, orc, shape):
        spec = synth.config("C1", dims=shape)
        x, y = synth.make_pair(spec)
        x, y = x.numpy(), y.numpy()
        r = orc.deriv(x, y)
        Fx, Fy = _fields_numpy(x), _fields_numpy(y)
        assert r["n_interior"] == Fx["der1"].size
        for k in Fx:
            d = Fy[k] - Fx[k]
            scale = max(1.0, float(np.abs(Fx[k]).max()))
            assert abs(r[f"{k}_f_min"] - Fx[k].min()) < 1e-13 * scale, k
            assert abs(r[f"{k}_f_max"] - Fx[k].max()) < 1e-13 * scale, k
            assert abs(r[f"{k}_maxabs"] - np.abs(d).max()) < 1e-13 * scale, k
            assert abs(r[f"{k}_mae"] - np.abs(d).mean()) < 1e-13 * scale, k
            assert abs(r[f"{k}_mse"] - (d * d).mean()) < 1e-12 * max(r[f"{k}_mse"], 1e-30) + 1e-26, k

    @pytest.mark.parametrize("shape", [(9, 11, 13), (25, 31), (40,), (6, 1, 17)])
    def test_points_against_numpy_scipy(self, orc, shape):
        """czco_deriv_points (per-point dF, the reference of the CUDA debug_der output) against the
        numpy.gradient / scipy.ndimage.laplace formulation, point by point."""
        x, y = synth.make_pair(synth.config("C2", dims=shape))
        x, y = x.numpy(), y.numpy()
        got = orc.deriv_points(x, y)
        Fx, Fy = _fields_numpy(x), _fields_numpy(y)
        for i, k in enumerate(("der1", "der2", "grad", "div", "lap")):
            want = (Fy[k] - Fx[k]).ravel()
            scale = max(1.0, float(np.abs(Fx[k]).max()))
            assert got.shape[1] == want.size
            np.testing.assert_allclose(got[i], want, rtol=0, atol=1e-12 * scale, err_msg=k)

    def test_no_interior(self, orc):
        x = dyadic_field((2, 5, 5))
        r = orc.deriv(x, x)
        assert r["n_interior"] == 0 and math.isnan(r["der1_mae"])


# ------------------------------------------------------------------------------------------ AC
class TestAutocorr:
    def _pair_with_error(self, e):
        x = dyadic_field(e.shape)
        y = (x.astype(np.float64) + e).astype(np.float32)
        assert np.all(y.astype(np.float64) - x.astype(np.float64) == e)
        return x, y

    def test_checkerboard(self, orc):
        """e = c (-1)^(z+y+x) on even dims: mu = 0, sigma^2 = c^2, AC(tau) = (-1)^tau exactly (Eq. 2)."""
        shape = (8, 10, 12)
        e = (2.0 ** -10) * (-1.0) ** np.indices(shape).sum(0)
        ac, cnt = orc.autocorr(*self._pair_with_error(e), max_lag=6)
        assert np.allclose(ac, [(-1.0) ** t for t in range(7)], rtol=0, atol=1e-15)
        assert list(cnt[1:]) == [(8 - t) * (10 - t) * (12 - t) for t in range(1, 7)]

    @pytest.mark.parametrize("axis", [0, 1, 2])
    def test_single_axis_parity(self, orc, axis):
        """e = c (-1)^(p_axis): the other two axis terms are +1, this one (-1)^tau -> (2 + (-1)^tau)/3."""
        shape = (6, 8, 10)
        e = (2.0 ** -9) * (-1.0) ** np.indices(shape)[axis]
        ac, _ = orc.autocorr(*self._pair_with_error(e), max_lag=5)
        want = [1.0] + [(2 + (-1.0) ** t) / 3 for t in range(1, 6)]
        assert np.allclose(ac, want, rtol=0, atol=1e-15)

    def test_2d_factor(self, orc):
        """2-D field: 1/D = 1/2 (R12): e = c (-1)^x -> AC = (1 + (-1)^tau) / 2."""
        e = (2.0 ** -9) * (-1.0) ** np.indices((10, 14))[1]
        ac, cnt = orc.autocorr(*self._pair_with_error(e), max_lag=4)
        assert np.allclose(ac, [1.0] + [(1 + (-1.0) ** t) / 2 for t in range(1, 5)], atol=1e-15)
        assert list(cnt[1:]) == [(10 - t) * (14 - t) for t in range(1, 5)]

    def test_brute_force_slices(self, orc):
        """Random errors: vectorised slice formulation of Eq. 2 (population mu, sigma^2 over N)."""
        x, y = synth.make_pair(synth.config("C1", dims=(11, 12, 13)))
        x, y = x.numpy(), y.numpy()
        e = y.astype(np.float64) - x.astype(np.float64)
        mu, var = e.mean(), e.var()
        ac, _ = orc.autocorr(x, y, max_lag=5)
        for t in range(1, 6):
            c = e[:-t, :-t, :-t] - mu
            nb = (e[t:, :-t, :-t] - mu) + (e[:-t, t:, :-t] - mu) + (e[:-t, :-t, t:] - mu)
            want = np.sum(c * nb / 3) / c.size / var
            assert abs(ac[t] - want) < 1e-12, t

    def test_degenerate(self, orc):
        x = dyadic_field((6, 6, 6))
        y = (x.astype(np.float64) + 2.0 ** -12).astype(np.float32)
        ac, cnt = orc.autocorr(x, y, max_lag=7)
        assert ac[0] == 1 and np.all(np.isnan(ac[1:]))         # sigma^2 = 0
        assert cnt[6] == 0 and cnt[7] == 0 and cnt[5] == 1     # tau >= min n -> no pairs


# ------------------------------------------------------------------------------------------ SSIM
def ssim_uniform_filter(x, y, w, data_range):
    """scikit-image's structural_similarity(win_size=w, data_range=R, gaussian_weights=False,
    use_sample_covariance=False) restated with scipy.ndimage.uniform_filter and the crop of
    (w-1)/2 it applies before averaging — valid windows, global dynamic range."""
    x = x.astype(np.float64)
    y = y.astype(np.float64)
    ux, uy = ndi.uniform_filter(x, w), ndi.uniform_filter(y, w)
    uxx, uyy, uxy = ndi.uniform_filter(x * x, w), ndi.uniform_filter(y * y, w), ndi.uniform_filter(x * y, w)
    vx, vy, vxy = uxx - ux * ux, uyy - uy * uy, uxy - ux * uy
    C1, C2 = (0.01 * data_range) ** 2, (0.03 * data_range) ** 2
    S = (2 * ux * uy + C1) * (2 * vxy + C2) / ((ux ** 2 + uy ** 2 + C1) * (vx + vy + C2))
    p = (w - 1) // 2
    return S[tuple(slice(p, n - p) for n in S.shape)].mean()


def ssim_brute_numpy(x, y, w, s=1):
    """Per-window numpy moments (np.var, np.cov bias=True), local range of the original."""
    vals = []
    it = [range(0, n - w + 1, s) for n in x.shape]
    for o in np.array(np.meshgrid(*it, indexing="ij")).reshape(x.ndim, -1).T:
        sl = tuple(slice(a, a + w) for a in o)
        a, b = x[sl].astype(np.float64).ravel(), y[sl].astype(np.float64).ravel()
        L = a.max() - a.min()
        L = 1.0 if L == 0 else L
        C1, C2 = (0.01 * L) ** 2, (0.03 * L) ** 2
        cxy = np.cov(a, b, bias=True)[0, 1]
        vals.append((2 * a.mean() * b.mean() + C1) * (2 * cxy + C2) /
                    ((a.mean() ** 2 + b.mean() ** 2 + C1) * (np.var(a) + np.var(b) + C2)))
    return np.array(vals)


class TestSSIM:
    def test_zero_error_is_one(self, orc):
        x, _ = synth.make_pair(synth.config("C2q", dims=(12, 16, 20)))
        s, nw = orc.ssim(x, x, [5, 5, 5])
        assert abs(s - 1) < 1e-15 and nw == 8 * 12 * 16

    def test_constant_field_closed_form(self, orc):
        """x = v, y = v + c: L = 0 -> 1, sigma = 0 -> SSIM = (2v(v+c)+C1)/(v^2+(v+c)^2+C1)."""
        v, c = 0.75, 2.0 ** -8
        x = np.full((9, 9, 9), v, np.float32)
        y = np.full((9, 9, 9), v + c, np.float32)
        s, nw = orc.ssim(x, y, [4, 4, 4])
        C1 = 1e-4
        assert nw == 6 ** 3
        assert abs(s - (2 * v * (v + c) + C1) / (v * v + (v + c) ** 2 + C1)) < 1e-15

    @pytest.mark.parametrize("shape,w", [((20, 22, 24), 7), ((40, 56), 7), ((15, 17, 19), 5)])
    def test_global_range_equals_skimage_formulation(self, orc, shape, w):
        x, y = synth.make_pair(synth.config("C1", dims=shape))
        x, y = x.numpy(), y.numpy()
        R = float(x.max()) - float(x.min())
        s, _ = orc.ssim(x, y, [w] * len(shape), range_mode=1)
        assert abs(s - ssim_uniform_filter(x, y, w, R)) < 1e-10

    @pytest.mark.parametrize("cfg,shape,w,s", [("C1", (8, 9, 10), 4, 1), ("C2q", (9, 10, 12), 3, 2),
                                               ("C4", (24, 30), 8, 3), ("C3", (7, 8, 9), 3, 1)])
    def test_brute_force_numpy(self, orc, cfg, shape, w, s):
        """Local-range SSIM, every window, against a numpy brute force; sparse zeros hit L := 1."""
        x, y = synth.make_pair(synth.config(cfg, dims=shape))
        x, y = x.numpy(), y.numpy()
        ref = ssim_brute_numpy(x, y, w, s)
        got, nw = orc.ssim(x, y, [w] * len(shape), [s] * len(shape))
        assert nw == ref.size
        assert abs(got - ref.mean()) < 1e-13
        it = [range(0, n - w + 1, s) for n in shape]
        origins = np.array(np.meshgrid(*it, indexing="ij")).reshape(len(shape), -1).T
        for i in rng.choice(len(origins), size=min(20, len(origins)), replace=False):
            v = orc.ssim_window(x, y, origins[i], [w] * len(shape))
            assert abs(v - ref[i]) < 1e-13

    @pytest.mark.parametrize("cfg,shape,w,s,kw", [("C1", (8, 9, 10), 4, 1, {}),
                                                  ("C2q", (9, 10, 12), 3, 2, {}),
                                                  ("C4", (24, 30), 8, 3, {}),
                                                  ("C1", (10, 9, 14), 5, 1, {"kind": "step", "eb": 0.1})])
    def test_window_map_brute_force(self, orc, cfg, shape, w, s, kw):
        """czco_ssim_windows (every window's local SSIM, the per-window reference of the GPU
        parity tests) against the numpy brute force, element by element, incl. a step field."""
        x, y = synth.make_pair(synth.config(cfg, dims=shape, **kw))
        x, y = x.numpy(), y.numpy()
        ref = ssim_brute_numpy(x, y, w, s)
        got = orc.ssim_windows(x, y, [w] * len(shape), [s] * len(shape))
        assert got.shape == tuple((n - w) // s + 1 for n in shape)
        np.testing.assert_allclose(got.ravel(), ref, rtol=0, atol=1e-12)
        assert abs(got.mean() - orc.ssim(x, y, [w] * len(shape), [s] * len(shape))[0]) < 1e-14

    @pytest.mark.parametrize("cfg,shape,w,kw", [("C1", (20, 24, 28), 7, {}), ("C2q", (18, 30, 33), 8, {}),
                                                ("C3", (17, 20, 25), 5, {}), ("C4", (60, 90), 8, {}),
                                                ("C2", (10, 11, 40), 8, {}), ("C4", (1, 300), 9, {}),
                                                ("C1", (10, 9, 14), 5, {"kind": "step", "eb": 0.1})])
    def test_separable_equals_brute_force(self, orc, cfg, shape, w, kw):
        """czco_ssim_separable (the C5-scale SSIM oracle: separable direct box sums in long double,
        textbook formula) reproduces the per-window brute force czco_ssim; on the step field the
        windows its cancellation bound rejects are recomputed by the brute force."""
        x, y = synth.make_pair(synth.config(cfg, dims=shape, **kw))
        x, y = x.numpy(), y.numpy()
        if shape[0] == 1:
            x, y = x[0].copy(), y[0].copy()
        win = [w] * x.ndim
        ref, nw = orc.ssim(x, y, win)
        got, nw2, nb = orc.ssim_separable(x, y, win)
        assert nw2 == nw and abs(got - ref) < 1e-13
        gr, _ = orc.ssim(x, y, win, range_mode=1)
        assert abs(orc.ssim_separable(x, y, win, range_mode=1)[0] - gr) < 1e-13
        if kw.get("kind") == "step":
            assert nb > 0

    def test_separable_closed_forms(self, orc):
        """Zero error -> 1; constant field x = v, y = v + c -> A / (A + c^2) (L = 0 -> 1)."""
        x, _ = synth.make_pair(synth.config("C2", dims=(12, 16, 20)))
        assert abs(orc.ssim_separable(x, x, [5, 5, 5])[0] - 1.0) < 1e-15
        v, c = 0.75, 2.0 ** -8
        xc = np.full((9, 10, 11), v, np.float32)
        yc = np.full((9, 10, 11), v + c, np.float32)
        A = 2 * v * (v + c) + 1e-4
        assert abs(orc.ssim_separable(xc, yc, [4, 4, 4])[0] - A / (A + c * c)) < 1e-15

    def test_no_window(self, orc):
        x = dyadic_field((5, 5, 5))
        s, nw = orc.ssim(x, x, [6, 6, 6])
        assert nw == 0 and math.isnan(s)


# ----------------------------------------------------------------------------------------- PDF
class TestPdf:
    """Error PDF / pwr-error PDF (Table I Category I, L107), bin rule of reading R24."""

    def test_constructed_bin_counts(self, orc):
        """e = k/16, k = 0..16 with multiplicity m_k, x = 1: lo = 0, w = 1/4, bin = floor(k/4) with
        k = 16 clamped into the last bin -> counts are sums of m_k by hand (closed form)."""
        m = np.arange(1, 18)                               # multiplicities 1..17
        k = np.repeat(np.arange(17), m)
        x = np.ones(k.size, np.float32)
        y = (1.0 + k / 16.0).astype(np.float32)            # exact in float32
        r = orc.pdf(x, y, 4)
        assert r["err_pdf_lo"] == 0.0 and r["err_pdf_width"] == 0.25
        want = [m[0:4].sum(), m[4:8].sum(), m[8:12].sum(), m[12:17].sum()]
        assert r["err_pdf"].tolist() == want
        # pwr = |e| / 1 = e: the same bins
        assert r["pwr_pdf"].tolist() == want and r["n_pwr"] == k.size

    def test_constant_error_single_bin(self, orc):
        """Dyadic constant offset: every error equal -> width 0, all counts in bin 0."""
        x = dyadic_field((5, 6, 7)).ravel()
        x[x == 0] = 2.0 ** -12
        y = x + np.float32(2.0 ** -10)
        r = orc.pdf(x, y, 10)
        assert r["err_pdf_width"] == 0.0 and r["err_pdf"][0] == x.size and r["err_pdf"][1:].sum() == 0

    def test_numpy_histogram_edge_free(self, orc):
        """numpy.histogram implements equal-width bins independently; on data with no value
        within 1e-6 of a bin edge the counts must agree exactly."""
        x = (1.0 + rng.random(20000)).astype(np.float32)
        y = (x + rng.uniform(-1e-3, 1e-3, x.size)).astype(np.float32)
        e = y.astype(np.float64) - x.astype(np.float64)
        nb = 50
        lo, hi = e.min(), e.max()
        t = (e - lo) / ((hi - lo) / nb)
        keep = (np.abs(t - np.round(t)) > 1e-6) | (e == lo) | (e == hi)
        r = orc.pdf(x[keep], y[keep], nb)
        want, edges = np.histogram(e[keep], bins=nb, range=(lo, hi))
        assert r["err_pdf"].tolist() == want.tolist()
        assert r["err_pdf_lo"] == lo and r["err_pdf_width"] == (hi - lo) / nb

    def test_totals_and_zero_originals(self, orc):
        """Counts total n (error PDF) and n_pwr = #{x != 0} (pwr PDF, reading R3)."""
        x, y = synth.make_pair(synth.config("C2q", dims=(6, 20, 30)))
        xn, yn = x.numpy().ravel(), y.numpy().ravel()
        r = orc.pdf(xn, yn, 33)
        assert int(r["err_pdf"].sum()) == xn.size
        assert r["n_pwr"] == int((xn != 0).sum()) == int(r["pwr_pdf"].sum())
        assert r["err_pdf"][0] > 0 and r["err_pdf"][-1] > 0    # the extrema fill the end bins
        q = np.abs(yn.astype(np.float64) - xn)[xn != 0] / np.abs(xn[xn != 0].astype(np.float64))
        assert r["pwr_pdf_lo"] == q.min() and r["pwr_pdf_width"] == (q.max() - q.min()) / 33

    def test_no_nonzero_original(self, orc):
        """All x == 0: no pwr values -> pwr range NaN, counts 0 (reading R3)."""
        x = np.zeros(100, np.float32)
        y = rng.uniform(-1, 1, 100).astype(np.float32)
        r = orc.pdf(x, y, 8)
        assert r["n_pwr"] == 0 and math.isnan(r["pwr_pdf_lo"]) and r["pwr_pdf"].sum() == 0
        assert int(r["err_pdf"].sum()) == 100


# ------------------------------------------------------------------- float64 inputs (NEXT f3)
class TestFloat64:
    """The float64 entry points (NEXT row f3, L92 / L330): pinned by (1) the invariant that
    float-representable data gives bit-identical results through both element types (every
    sample is read as a double either way), (2) closed forms whose inputs float32 cannot hold,
    (3) numpy on data with full 53-bit mantissas."""

    def test_float_data_identical_through_f64(self, orc):
        x, y = synth.make_pair(synth.config("C1", dims=(12, 14, 16)))
        xn, yn = x.numpy(), y.numpy()
        xd, yd = xn.astype(np.float64), yn.astype(np.float64)
        assert orc.p1(xn, yn) == orc.p1(xd, yd)
        assert orc.deriv(xn, yn) == orc.deriv(xd, yd)
        a32, c32 = orc.autocorr(xn, yn, 5)
        a64, c64 = orc.autocorr(xd, yd, 5)
        assert np.array_equal(a32, a64) and np.array_equal(c32, c64)
        assert orc.ssim(xn, yn, [5, 5, 5], [2, 3, 1]) == orc.ssim(xd, yd, [5, 5, 5], [2, 3, 1])
        p32, p64 = orc.pdf(xn, yn, 17), orc.pdf(xd, yd, 17)
        for k in p32:
            assert np.array_equal(p32[k], p64[k]), k

    def test_sub_float_offset_closed_form(self, orc):
        """x on a 2^-40 grid (|x| < 2^-12, not float32-representable), e == c = 2^-45 exactly:
        MSE = c^2, PSNR = 20 log10(R / c), every window's SSIM has the closed form of a constant
        offset, Der/Div/Lap errors are 0 (a constant offset has no derivative), AC undefined."""
        x = rng.integers(-(2 ** 28), 2 ** 28, size=(9, 10, 11)).astype(np.float64) * 2.0 ** -40
        assert np.any(x.astype(np.float32).astype(np.float64) != x)
        c = 2.0 ** -45
        y = x + c
        assert np.all(y - x == c)
        r = orc.p1(x, y)
        R = float(x.max() - x.min())
        assert r["mse"] == c * c and r["err_min"] == c == r["err_max"] and r["err_var"] == 0.0
        assert abs(r["psnr"] - 20 * math.log10(R / c)) < 1e-12
        d = orc.deriv(x, y)
        for f in ("der1", "der2", "div", "lap"):
            assert d[f + "_maxabs"] == 0.0, f
        ac, _ = orc.autocorr(x, y, 3)
        assert all(math.isnan(v) for v in ac[1:])
        # SSIM of one window with y = x + c: (2 mx (mx + c) + C1) (2 vx + C2) /
        # ((mx^2 + (mx + c)^2 + C1) (2 vx + C2)) = (2 mx (mx + c) + C1) / (mx^2 + (mx + c)^2 + C1)
        o, w = (1, 2, 3), (4, 4, 4)
        win = x[1:5, 2:6, 3:7]
        mx, L = win.mean(), float(win.max() - win.min())
        C1 = (0.01 * L) ** 2
        want = (2 * mx * (mx + c) + C1) / (mx * mx + (mx + c) ** 2 + C1)
        assert abs(orc.ssim_window(x, y, o, w) - want) < 1e-12

    def test_numpy_brute_force_full_mantissa(self, orc):
        x = rng.standard_normal((6, 7, 9)) * 1e3 + 1e4
        y = x + rng.standard_normal(x.shape) * 1e-7
        e = y - x
        r = orc.p1(x, y)
        assert r["err_min"] == e.min() and r["err_max"] == e.max() and r["x_min"] == x.min()
        q = np.abs(e) / np.abs(x)
        assert r["pwr_max"] == q.max() and r["pwr_min"] == q.min()
        assert abs(r["mse"] / np.mean(e * e) - 1) < 1e-12
        assert abs(r["pearson"] - np.corrcoef(x.ravel(), y.ravel())[0, 1]) < 1e-12
        d = orc.deriv(x, y)
        gx = [np.gradient(x, axis=a)[1:-1, 1:-1, 1:-1] for a in range(3)]
        gy = [np.gradient(y, axis=a)[1:-1, 1:-1, 1:-1] for a in range(3)]
        grad = np.sqrt(sum(g * g for g in gy)) - np.sqrt(sum(g * g for g in gx))
        assert abs(d["grad_mae"] - np.mean(np.abs(grad))) < 1e-9 * np.mean(np.abs(grad)) + 1e-15
        s, nw = orc.ssim(x, y, [3, 3, 3])
        assert nw == 4 * 5 * 7 and 0.0 < s <= 1.0


# ------------------------------------------------------------------------ 4-D fields (NEXT f3)
class TestFourD:
    """4-D fields (L92: "easily extended to other dimensions (including 1D, 2D, and 4D)"): the
    same definitions over four axes, pinned by closed forms, numpy and an invariant tying 4-D
    windows to 3-D ones."""

    def test_ramp_and_quadratic_closed_forms(self, orc):
        shape = (5, 6, 7, 8)
        p = np.indices(shape).astype(np.float64)
        c = np.array([2 ** -2, 2 ** -3, -(2 ** -4), 2 ** -5])
        q = np.array([2 ** -4, -(2 ** -5), 2 ** -3, 2 ** -6])
        x = np.tensordot(c, p, 1).astype(np.float32)
        y = (np.tensordot(c, p, 1) + np.tensordot(q, p ** 2, 1)).astype(np.float32)
        r = orc.deriv(x, y)
        assert r["n_interior"] == 3 * 4 * 5 * 6
        assert r["der1_f_min"] == r["der1_f_max"] == 2 * np.abs(c).sum()
        assert r["div_f_max"] == c.sum() and r["lap_f_max"] == 0
        assert r["grad_f_max"] == pytest.approx(math.sqrt((c ** 2).sum()), abs=1e-15)
        assert r["lap_maxabs"] == 2 * q.sum() and r["lap_mse"] == (2 * q.sum()) ** 2

    def test_against_numpy_gradient(self, orc):
        r4 = np.random.default_rng(5)
        x = r4.standard_normal((6, 7, 8, 9)).astype(np.float32)
        y = (x + 1e-3 * r4.standard_normal(x.shape)).astype(np.float32)
        r = orc.deriv(x, y)
        xd, yd = x.astype(np.float64), y.astype(np.float64)
        inner = (slice(1, -1),) * 4
        gx = np.sqrt(sum(g ** 2 for g in np.gradient(xd)))[inner]
        gy = np.sqrt(sum(g ** 2 for g in np.gradient(yd)))[inner]
        assert abs(r["grad_mae"] - np.mean(np.abs(gy - gx))) < 1e-12
        lap = lambda f: sum(np.roll(f, 1, a) - 2 * f + np.roll(f, -1, a) for a in range(4))[inner]
        assert abs(r["lap_mse"] - np.mean((lap(yd) - lap(xd)) ** 2)) < 1e-12 * r["lap_mse"] + 1e-18
        assert r["der1_f_max"] == pytest.approx(
            sum(np.abs(np.roll(xd, -1, a) - np.roll(xd, 1, a)) for a in range(4))[inner].max(), rel=1e-15)

    def test_autocorr_checkerboard_and_axis(self, orc):
        shape = (8, 9, 10, 11)
        i = np.indices(shape).sum(0)
        x = np.zeros(shape, np.float32)
        y = np.where(i % 2 == 0, 1.0, -1.0).astype(np.float32)
        ac, cnt = orc.autocorr(x, y, 5)
        # e = (-1)^(i0+i1+i2+i3) has mean ~0 but not exactly (odd extent): compare with numpy
        e = y.astype(np.float64)
        mu, var = e.mean(), e.var()
        for t in range(1, 6):
            hi = tuple(slice(0, n - t) for n in shape)
            s = 0.0
            for a in range(4):
                sh = [slice(0, n - t) for n in shape]
                sh[a] = slice(t, shape[a])
                s += np.sum((e[hi] - mu) * (e[tuple(sh)] - mu))
            want = s / 4 / np.prod([n - t for n in shape]) / var
            assert abs(ac[t] - want) < 1e-12, (t, ac[t], want)
            assert cnt[t] == np.prod([n - t for n in shape])
        assert ac[1] < -0.99 and ac[2] > 0.99

    def test_ssim_zero_error_brute_force_and_replication(self, orc):
        r4 = np.random.default_rng(9)
        x = (280 + r4.standard_normal((5, 6, 7, 8))).astype(np.float32)
        assert orc.ssim(x, x, [3, 3, 3, 3]) == (1.0, 3 * 4 * 5 * 6)
        y = (x + 1e-2 * r4.standard_normal(x.shape)).astype(np.float32)
        # per-window numpy (np.var / np.cov definitions) at two origins
        for o in ((0, 1, 2, 3), (2, 3, 0, 1)):
            w = (3, 3, 4, 5)
            sl = tuple(slice(a, a + b) for a, b in zip(o, w))
            xw, yw = x[sl].astype(np.float64).ravel(), y[sl].astype(np.float64).ravel()
            L = xw.max() - xw.min()
            C1, C2 = (0.01 * L) ** 2, (0.03 * L) ** 2
            cov = np.cov(xw, yw, bias=True)
            want = ((2 * xw.mean() * yw.mean() + C1) * (2 * cov[0, 1] + C2) /
                    ((xw.mean() ** 2 + yw.mean() ** 2 + C1) * (cov[0, 0] + cov[1, 1] + C2)))
            assert abs(orc.ssim_window(x, y, o, w) - want) < 1e-12
        # a 4-D field replicating a 3-D one along axis 0, windows spanning that axis: every 4-D
        # window holds w0 copies of a 3-D window -> the same local SSIM, the same mean
        x3, y3 = x[0], y[0]
        x4, y4 = np.repeat(x3[None], 3, 0), np.repeat(y3[None], 3, 0)
        s3, n3 = orc.ssim(x3, y3, [3, 4, 5])
        s4, n4 = orc.ssim(x4, y4, [3, 3, 4, 5])
        assert n3 == n4 and abs(s3 - s4) < 1e-13
