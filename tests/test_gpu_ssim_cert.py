"""SSIM parity on EVERY window, including the adversarial fields the certified fast path exists for
(VERDICT r1 "What's missing" #1): steps placed mid-tile along x, y and z, fill
values of 1e35, 2-D and 1-D fields and float64 inputs.  The CUDA path's per-window local SSIM
(debug_wssim, Alg. 3 "wssim") is compared with the oracle's brute-force value of every window
(czco_ssim_windows, L139) at the 1e-6 absolute tolerance of north_star, and the windows the
certificate sent to the exact path are counted (czc_result.n_ssim_exact): > 0 on the adversarial
fields, 0 on the BASELINE recipes C1-C4."""
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


def gpu_windows(czc, x, y, w, step=1, range_mode=0, **cfg):
    """(per-window local SSIM array, result dict) through czc_assess with a debug buffer."""
    xn, yn = np.ascontiguousarray(x), np.ascontiguousarray(y)
    nd = xn.ndim
    ws = [w] * nd if isinstance(w, int) else list(w)
    ss = [step] * nd if isinstance(step, int) else list(step)
    nw = [(n - a) // s + 1 for n, a, s in zip(xn.shape, ws, ss)]
    dbg = torch.full(nw, float("nan"), dtype=torch.float64, device="cuda")
    with czc.Assessor(ndim=nd, ssim_window=w, ssim_step=step, ssim_range_mode=range_mode,
                      debug_wssim=dbg.data_ptr(), **cfg) as a:
        r = a.assess(torch.from_numpy(xn).cuda(), torch.from_numpy(yn).cuda(), czc.M_SSIM | czc.M_P1)
    return dbg.cpu().numpy(), r


def check_all_windows(czc, orc, x, y, w, step=1, range_mode=0, **cfg):
    d, r = gpu_windows(czc, x, y, w, step, range_mode, **cfg)
    nd = x.ndim
    ws = [w] * nd if isinstance(w, int) else list(w)
    ss = [step] * nd if isinstance(step, int) else list(step)
    ref = orc.ssim_windows(x, y, ws, ss, range_mode)
    assert d.shape == ref.shape and not np.isnan(d).any()
    err = np.abs(d - ref)
    worst = np.unravel_index(int(np.argmax(err)), err.shape)
    assert err.max() < 1e-6, f"worst window {worst}: gpu {d[worst]!r} oracle {ref[worst]!r}"
    assert r["n_windows"] == ref.size
    assert abs(r["ssim"] - ref.mean()) < 1e-6
    assert abs(r["ssim"] - d.mean()) < 1e-12           # the mean is the mean of the windows
    return r, float(err.max())


def step_pair(shape, axis, pos, lo=1.0, hi=1000.0, eb=0.1, seed=3, dtype=np.float32):
    """Adversarial step field (SURVEY.md probe 12): lo | hi halves split at `pos` along `axis`,
    a 1e-3 texture, recon pre-quantised with eb (locally constant reconstruction)."""
    rng = np.random.default_rng(seed)
    idx = np.indices(shape)[axis]
    x = np.where(idx < pos, lo, hi) + 1e-3 * rng.standard_normal(shape)
    x = x.astype(dtype)
    y = (2 * eb * np.rint(x.astype(np.float64) / (2 * eb))).astype(dtype)
    return x, y


@pytest.mark.parametrize("nx,pos", [(40, 20), (45, 12), (57, 37), (40, 3)])
def test_step_along_x_mid_tile(czc, orc, nx, pos):
    """The step sits inside a 25-origin x tile, so windows on both sides share a tile anchor
    (18x20x40 gave 3.35e-6 on the mean and 1.8e-4 on single windows)."""
    x, y = step_pair((18, 20, nx), 2, pos)
    r, worst = check_all_windows(czc, orc, x, y, 8)
    print(f"x-step nx={nx} at {pos}: worst {worst:.2e}, exact recomputes {r['n_ssim_exact']}")
    if (nx, pos) == (40, 20):                          # the case VERDICT r1 emulated
        assert r["n_ssim_exact"] > 0


@pytest.mark.parametrize("axis,pos", [(0, 9), (0, 21), (1, 11)])
def test_step_along_z_and_y(czc, orc, axis, pos):
    """A z-step passes THROUGH the running z-sums (every later window of the column
    was polluted); a y-step spans the running y-sums of the G origin rows of a warp."""
    x, y = step_pair((40, 22, 36), axis, pos)
    r, worst = check_all_windows(czc, orc, x, y, 8)
    print(f"step axis {axis} at {pos}: worst {worst:.2e}, exact recomputes {r['n_ssim_exact']}")


def test_fill_values_1e35(czc, orc):
    """A block of 1e35 fill values (a common missing-value marker) inside a smooth field."""
    x, y = synth.make_pair(synth.config("C2", dims=(30, 34, 45)))
    x, y = x.numpy().copy(), y.numpy().copy()
    x[10:14, 5:20, 7:30] = np.float32(1e35)
    y[10:14, 5:20, 7:30] = np.float32(1e35)
    y[12, 8, 9] = np.float32(9.9e34)                    # one reconstruction error at the fill scale
    r, _ = check_all_windows(czc, orc, x, y, 8)
    assert r["n_ssim_exact"] > 0


def test_step_2d_and_1d(czc, orc):
    tot = 0
    for shape, axis, pos in (((70, 61), 1, 29), ((70, 61), 0, 33), ((300,), 0, 150)):
        x, y = step_pair(shape, axis, pos)
        r, worst = check_all_windows(czc, orc, x, y, 9 if len(shape) == 1 else 8)
        print(f"{len(shape)}-D step axis {axis} at {pos}: worst {worst:.2e}, exact {r['n_ssim_exact']}")
        tot += r["n_ssim_exact"]
    assert tot > 0


def test_step_float64(czc, orc):
    x, y = step_pair((20, 24, 45), 2, 30, dtype=np.float64)
    x = x + 1e-9 * np.random.default_rng(5).standard_normal(x.shape)   # not float-representable
    r1, _ = check_all_windows(czc, orc, x, y, 8)
    x, y = step_pair((40, 22, 36), 0, 17, dtype=np.float64)
    r2, _ = check_all_windows(czc, orc, x, y, 6)
    print(f"float64 steps: exact recomputes {r1['n_ssim_exact']}, {r2['n_ssim_exact']}")


def test_step_with_steps_ranges_and_extents(czc, orc):
    """Window steps, the global-range mode and other window extents on a step field."""
    x, y = step_pair((26, 30, 50), 2, 23)
    check_all_windows(czc, orc, x, y, 5, step=(1, 2, 3))
    check_all_windows(czc, orc, x, y, 7, range_mode=1)
    check_all_windows(czc, orc, x, y, 12)
    check_all_windows(czc, orc, x, y, 3)


def test_step_loopback_slabs(czc, orc):
    """Slab mode (halo planes in separate buffers) on a z-step that crosses a slab boundary."""
    x, y = step_pair((36, 22, 40), 0, 18)
    r, _ = check_all_windows(czc, orc, x, y, 8, loopback_slabs=3)
    x, y = step_pair((36, 22, 40), 2, 20)
    r, _ = check_all_windows(czc, orc, x, y, 8, loopback_slabs=3)
    assert r["n_ssim_exact"] > 0


@pytest.mark.parametrize("cfg,dims,w", [("C1", (64, 64, 64), 7), ("C2", (40, 70, 90), 8), ("C2q", (36, 66, 75), 8),
                                        ("C3", (33, 45, 61), 8), ("C4", (180, 360), 8), ("C3", (48, 96, 128), 8)])
def test_recipes_every_window_no_fallback(czc, orc, cfg, dims, w):
    """The BASELINE recipes: every window within 1e-6, and no window of C1-C4 needs the exact path.
    C2q (the QCLOUD-like second Hurricane field: 70 % exact zeros next to log-normal clouds) may
    send a handful of near-zero windows whose z-extended sums touched a cloud 100x larger to the
    exact path (the bound is rigorous, not tuned): <= 1e-4 of the windows."""
    x, y = synth.make_pair(synth.config(cfg, dims=dims))
    r, worst = check_all_windows(czc, orc, x.numpy(), y.numpy(), w)
    print(f"{cfg} {dims}: worst window error {worst:.2e}, exact recomputes {r['n_ssim_exact']}")
    if cfg == "C2q":
        assert r["n_ssim_exact"] <= 1e-4 * r["n_windows"]
    else:
        assert r["n_ssim_exact"] == 0


def test_adversarial_result_deterministic(czc):
    """The exact-path recomputation keeps the result bit-identical across runs."""
    x, y = step_pair((30, 40, 57), 2, 37)
    outs = [gpu_windows(czc, x, y, 8)[1] for _ in range(3)]
    assert all(o["ssim"] == outs[0]["ssim"] and o["n_ssim_exact"] == outs[0]["n_ssim_exact"] for o in outs)


@pytest.mark.parametrize("dims,step", [((1100, 160, 160), 1), ((600, 26, 33), 3)])
def test_tall_fields_long_chunks(czc, orc, dims, step):
    """Tall fields: with 70 tiles the launcher's cost model (p3_ssim.cu launch_t) walks the
    1100-plane field in 4 chunks of 274 origin planes (one wave), so one block's z-sums slide and
    resync across hundreds of planes and the chunk boundaries fall mid-field; the small field
    takes many short chunks with a z step of 3.  Every window is compared with the oracle on a
    log-normal recipe field and on a z-step field whose steps repeat every 97 planes (each block
    meets several; the anchor is re-chosen at every resync, so the exact path takes ~14 % of its
    windows instead of ~51 % with one anchor per 274-plane chunk)."""
    x, y = synth.make_pair(synth.config("C3", dims=dims))
    r, worst = check_all_windows(czc, orc, x.numpy(), y.numpy(), 8, step)
    print(f"tall {dims} step {step} recipe: exact recomputes {r['n_ssim_exact']} of {r['n_windows']}")
    # the log-normal recipe spans decades: a few windows whose z-history since the last resync
    # touched values far above their own fail the rigorous bound (they are exact afterwards)
    assert r["n_ssim_exact"] <= 5e-3 * r["n_windows"]
    rng = np.random.default_rng(11)
    z = np.arange(dims[0])[:, None, None]
    xs = (np.where((z // 97) % 2 == 0, 1.0, 1000.0) + 1e-3 * rng.standard_normal(dims)).astype(np.float32)
    ys = (0.2 * np.rint(xs.astype(np.float64) / 0.2)).astype(np.float32)
    r2, worst2 = check_all_windows(czc, orc, xs, ys, 8, step)
    print(f"tall {dims} step {step}: worst {worst:.2e} / {worst2:.2e}, exact recomputes {r2['n_ssim_exact']}")
