"""Derivative-family parity POINT BY POINT (VERDICT r1 missing #7): the CUDA path's per-point
errors dF = F(recon) - F(orig) of Der1 / Der2 / Grad / Div / Lap (czc_config.debug_der, Alg. 2
L246 "Der[]") against the oracle's plain stencil of every interior point (czco_deriv_points,
Eq. 1; readings R7, R9, R11), on 3-D / 2-D / 1-D / 4-D fields, float64, slab mode and
the pipelined host path.  Tolerance: north_star's 1e-6 absolute, and 1e-12 of the field scale
(both sides evaluate the same FP64 differences; only the square root of Grad differs in the
last bits)."""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def czc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_cluster_yudgtc21_b200 as m
    m.get_lib()
    return m


def n_interior(shape):
    n = 1
    for d in shape:
        n *= (d - 2 if d > 2 else 0) if d > 1 else 1
    return n


def check_points(czc, orc, x, y, host=False, **cfg):
    xn, yn = np.ascontiguousarray(x), np.ascontiguousarray(y)
    nI = n_interior(xn.shape)
    dbg = torch.full((5, nI), float("nan"), dtype=torch.float64, device="cuda")
    with czc.Assessor(ndim=xn.ndim, debug_der=dbg.data_ptr(), **cfg) as a:
        if host:
            r = a.assess_host(xn, yn, czc.M_DERIV)
        else:
            r = a.assess(torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda(), czc.M_DERIV)
    g = dbg.cpu().numpy()
    o = orc.deriv_points(xn, yn)
    assert r["n_interior"] == nI and o.shape == g.shape and not np.isnan(g).any()
    od = orc.deriv(xn, yn)
    for i, f in enumerate(("der1", "der2", "grad", "div", "lap")):
        scale = max(1.0, abs(od[f + "_f_max"]), abs(od[f + "_f_min"]))
        err = np.abs(g[i] - o[i])
        assert err.max() <= min(1e-6, 1e-12 * scale), (f, float(err.max()), int(np.argmax(err)))
        # the streamed statistics are the reductions of these points
        assert abs(np.abs(g[i]).max() - r[f + "_maxabs"]) <= 1e-15 * scale, f
        assert abs(np.abs(g[i]).mean() - r[f + "_mae"]) <= 1e-12 * scale, f


@pytest.mark.parametrize("cfg,dims", [("C2", (21, 37, 45)), ("C3", (33, 45, 61)), ("C2q", (17, 40, 70)),
                                      ("C1", (64, 64, 64)), ("C4", (60, 130)), ("C4", (3, 300)),
                                      ("C2", (7, 1, 90))])
def test_points(czc, orc, cfg, dims):
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    xn, yn = x.numpy(), y.numpy()
    if dims == (3, 300):                                   # 1-D
        xn, yn = xn[1].copy(), yn[1].copy()
    check_points(czc, orc, xn, yn)


def test_points_4d_f64_slabs_host(czc, orc):
    x, y = synth.make_pair(synth.config("C2", dims=(30, 17, 19)))
    x4, y4 = x.numpy().reshape(5, 6, 17, 19), y.numpy().reshape(5, 6, 17, 19)
    check_points(czc, orc, x4, y4)                                     # 4-D generic kernel
    check_points(czc, orc, x.numpy().astype(np.float64), y.numpy().astype(np.float64) + 1e-9)   # float64
    check_points(czc, orc, x.numpy(), y.numpy(), loopback_slabs=3)     # slab mode (halo planes)
    x2, y2 = synth.make_pair(synth.config("C2", dims=(40, 36, 44)))
    check_points(czc, orc, x2.numpy(), y2.numpy(), host=True)          # pipelined host path
