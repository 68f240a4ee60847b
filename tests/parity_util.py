"""Tolerance classes of the CUDA-vs-oracle comparison (north_star of BASELINE.json):
bit-exact for min/max/max-error and integer counts; 1e-9 relative for double-accumulated
moments, PSNR and Pearson; 1e-6 absolute for SSIM and derivative metrics (plus a tighter
relative check on derivative sums, which the FP64 kernels meet)."""
import math

import numpy as np

EXACT = ("n", "x_min", "x_max", "value_range", "err_min", "err_max", "err_maxabs", "max_rel_err",
         "pwr_min", "pwr_max", "n_pwr")
REL9 = ("mse", "rmse", "nrmse", "err_absmean", "pwr_mean", "err_var", "snr", "psnr")
DERIV_FIELDS = ("der1", "der2", "grad", "div", "lap")


def _same_special(a, b):
    if math.isnan(a) or math.isnan(b):
        return math.isnan(a) and math.isnan(b)
    if math.isinf(a) or math.isinf(b):
        return a == b
    return None


def close_rel(a, b, rel, scale=None):
    s = _same_special(a, b)
    if s is not None:
        return s
    ref = abs(b) if scale is None else scale
    return abs(a - b) <= rel * ref


def check_p1(g, o, errors):
    for k in EXACT:
        if not (g[k] == o[k] or (_same_special(g[k], o[k]) is True)):
            errors.append(f"{k}: gpu {g[k]!r} != oracle {o[k]!r} (exact)")
    for k in REL9:
        if not close_rel(g[k], o[k], 1e-9):
            errors.append(f"{k}: gpu {g[k]!r} vs oracle {o[k]!r} (rel 1e-9)")
    if not close_rel(g["err_mean"], o["err_mean"], 1e-9, scale=abs(o["err_absmean"])):
        errors.append(f"err_mean: gpu {g['err_mean']!r} vs oracle {o['err_mean']!r}")
    if not close_rel(g["pearson"], o["pearson"], 1e-9, scale=1.0):
        errors.append(f"pearson: gpu {g['pearson']!r} vs oracle {o['pearson']!r} (abs 1e-9)")


def check_deriv(g, o, errors):
    if g["n_interior"] != o["n_interior"]:
        errors.append(f"n_interior {g['n_interior']} != {o['n_interior']}")
    for f in DERIV_FIELDS:
        for s in ("maxabs", "mae", "mse", "rmse", "f_min", "f_max", "psnr"):
            k = f"{f}_{s}"
            a, b = g[k], o[k]
            sp = _same_special(a, b)
            if sp is False:
                errors.append(f"{k}: gpu {a!r} vs oracle {b!r} (special)")
                continue
            if sp:
                continue
            if abs(a - b) > 1e-6:
                errors.append(f"{k}: gpu {a!r} vs oracle {b!r} (abs 1e-6)")
            elif abs(a - b) > 1e-9 * abs(b) + 1e-15 * (1 + abs(o[f'{f}_f_max'])):
                errors.append(f"{k}: gpu {a!r} vs oracle {b!r} (tight rel 1e-9)")


def check_ac(g_ac, g_cnt, o_ac, o_cnt, errors):
    if list(map(int, g_cnt)) != list(map(int, o_cnt)):
        errors.append(f"ac_count {list(g_cnt)} != {list(o_cnt)}")
    for t, (a, b) in enumerate(zip(g_ac, o_ac)):
        if not close_rel(a, b, 1e-9, scale=1.0):
            errors.append(f"ac[{t}]: gpu {a!r} vs oracle {b!r} (abs 1e-9)")


def check_ssim(g_ssim, g_nw, o_ssim, o_nw, errors, tol=1e-6):
    if int(g_nw) != int(o_nw):
        errors.append(f"n_windows {g_nw} != {o_nw}")
    if not close_rel(g_ssim, o_ssim, tol, scale=1.0):
        errors.append(f"ssim: gpu {g_ssim!r} vs oracle {o_ssim!r} (abs {tol})")


def report(errors):
    assert not errors, "\n".join(errors)
