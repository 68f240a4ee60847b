"""CPU ORACLE for the cuZ-Checker assessment hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` legs may
import this package.  The product path (paper_conf_cluster_yudgtc21_b200) never imports it and
fails loudly if its CUDA library is missing.  The oracle shares no code with the CUDA path.

Thin ctypes wrapper over `liboracle.so` (built from czc_oracle.c by `build()` or on first use).
All metric arithmetic lives in czc_oracle.c, each function citing the PAPER.md passage it
implements.  Pinning status of every function:
  p1        pinned  (closed forms: zero error, dyadic offset; statistical uniform-noise PSNR;
                     numpy corrcoef / longdouble two-pass Pearson; brute-force numpy extrema)
  deriv     pinned  (dyadic ramp / quadratic closed forms; numpy.gradient; scipy.ndimage.laplace)
  autocorr  pinned  (checkerboard (-1)^tau; single-axis cosine; constant error -> NaN)
  ssim      pinned  (zero error = 1; constant-field closed form; global-range mode equals the
                     scipy uniform_filter formulation of scikit-image's SSIM; numpy brute force)
  pdf       pinned  (constructed values at bin centres: exact per-bin counts; numpy.histogram on
                     edge-free data; constant error -> one bin; totals = n, n_pwr; top edge clamp)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Dict, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "czc_oracle.c")
_lib = None

DERIV_FIELDS = ("der1", "der2", "grad", "div", "lap")
DERIV_STATS = ("maxabs", "mae", "mse", "rmse", "f_min", "f_max", "psnr")


class _P1(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64)] + [(k, ctypes.c_double) for k in (
        "x_min", "x_max", "value_range", "err_min", "err_max", "err_maxabs", "err_mean",
        "err_absmean", "mse", "rmse", "nrmse", "psnr", "snr", "max_rel_err", "pwr_min",
        "pwr_max", "pwr_mean")] + [("n_pwr", ctypes.c_uint64), ("pearson", ctypes.c_double),
                                   ("err_var", ctypes.c_double)]


class _DF(ctypes.Structure):
    _fields_ = [(k, ctypes.c_double) for k in DERIV_STATS]


class _Deriv(ctypes.Structure):
    _fields_ = [("n_interior", ctypes.c_uint64), ("f", _DF * 5)]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2 -fopenmp -ffp-contract=off)."""
    srcs = (_SRC, os.path.join(_HERE, "czc_oracle_t.inc"), os.path.join(_HERE, "czc_oracle.h"))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(os.path.getmtime(f) for f in srcs):
        cmd = ["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
               "-std=c11", "-Wall", "-o", _SO, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        I64P = ctypes.POINTER(ctypes.c_int64)
        lib.czco_p1.argtypes = [P, P, ctypes.c_uint64, ctypes.POINTER(_P1)]
        lib.czco_deriv.argtypes = [P, P, ctypes.c_int, I64P, ctypes.POINTER(_Deriv)]
        lib.czco_autocorr.argtypes = [P, P, ctypes.c_int, I64P, ctypes.c_int,
                                      ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_uint64)]
        lib.czco_ssim_window.argtypes = [P, P, ctypes.c_int, I64P, I64P, I64P, ctypes.c_int, ctypes.c_double]
        lib.czco_ssim_window.restype = ctypes.c_double
        lib.czco_ssim.argtypes = [P, P, ctypes.c_int, I64P, I64P, I64P, ctypes.c_int,
                                  ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_uint64)]
        DP = ctypes.POINTER(ctypes.c_double)
        UP = ctypes.POINTER(ctypes.c_uint64)
        lib.czco_pdf.argtypes = [P, P, ctypes.c_uint64, ctypes.c_int, DP, DP, UP, DP, DP, UP, UP]
        lib.czco_ssim_windows.argtypes = [P, P, ctypes.c_int, I64P, I64P, I64P, ctypes.c_int, P]
        lib.czco_deriv_points.argtypes = [P, P, ctypes.c_int, I64P, P]
        lib.czco_ssim_separable.argtypes = [P, P, ctypes.c_int, I64P, I64P, ctypes.c_int,
                                            ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_uint64),
                                            ctypes.POINTER(ctypes.c_uint64)]
        lib.czco_threads.restype = ctypes.c_int
        for name in ("czco_p1", "czco_deriv", "czco_autocorr", "czco_ssim_window", "czco_ssim", "czco_pdf",
                     "czco_ssim_windows", "czco_deriv_points", "czco_ssim_separable"):
            f32, f64 = getattr(lib, name), getattr(lib, name + "_f64")
            f64.argtypes = f32.argtypes
            f64.restype = f32.restype
        _lib = lib
    return _lib


def _np(a) -> np.ndarray:
    if hasattr(a, "detach"):
        a = a.detach().cpu().numpy()
    return np.asarray(a)


def _pair(x, y):
    """The pair as C-contiguous arrays of one element type: float64 if either input is float64
    (NEXT row f3), else float32 (the paper's precision)."""
    x, y = _np(x), _np(y)
    dt = np.float64 if np.float64 in (x.dtype, y.dtype) else np.float32
    return np.ascontiguousarray(x, dtype=dt), np.ascontiguousarray(y, dtype=dt)


def _fn(name: str, x: np.ndarray):
    return getattr(_load(), name + ("_f64" if x.dtype == np.float64 else ""))


def _dims(a: np.ndarray, dims=None):
    d = tuple(a.shape) if dims is None else tuple(int(v) for v in dims)
    return len(d), (ctypes.c_int64 * len(d))(*d)


def _i64(v: Sequence[int]):
    return (ctypes.c_int64 * len(v))(*[int(t) for t in v])


def threads() -> int:
    return int(_load().czco_threads())


def p1(x, y) -> Dict[str, float]:
    x, y = _pair(x, y)
    r = _P1()
    rc = _fn("czco_p1", x)(x.ctypes.data, y.ctypes.data, x.size, ctypes.byref(r))
    if rc:
        raise ValueError(f"czco_p1 failed ({rc})")
    return {k: getattr(r, k) for k, _ in _P1._fields_}


def deriv(x, y, dims=None) -> Dict[str, float]:
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    r = _Deriv()
    rc = _fn("czco_deriv", x)(x.ctypes.data, y.ctypes.data, nd, d, ctypes.byref(r))
    if rc:
        raise ValueError(f"czco_deriv failed ({rc})")
    out = {"n_interior": r.n_interior}
    for i, f in enumerate(DERIV_FIELDS):
        for s in DERIV_STATS:
            out[f"{f}_{s}"] = getattr(r.f[i], s)
    return out


def deriv_points(x, y, dims=None) -> np.ndarray:
    """Per-point dF = F(y) - F(x) of the five derived fields (czco_deriv_points): shape
    (5, n_interior), fields DER1, DER2, GRAD, DIV, LAP, points in C order of the interior grid."""
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    shp = tuple(x.shape) if dims is None else tuple(int(v) for v in dims)
    nI = 1
    for n in shp:
        nI *= (n - 2 if n > 2 else 0) if n > 1 else 1
    out = np.empty(5 * max(nI, 1), dtype=np.float64)
    rc = _fn("czco_deriv_points", x)(x.ctypes.data, y.ctypes.data, nd, d, out.ctypes.data)
    if rc == 3:
        return np.empty((5, 0))
    if rc:
        raise ValueError(f"czco_deriv_points failed ({rc})")
    return out.reshape(5, nI)


def autocorr(x, y, max_lag: int = 10, dims=None):
    """Returns (ac[0..max_lag], count[0..max_lag])."""
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    ac = (ctypes.c_double * (max_lag + 1))()
    cnt = (ctypes.c_uint64 * (max_lag + 1))()
    rc = _fn("czco_autocorr", x)(x.ctypes.data, y.ctypes.data, nd, d, max_lag, ac, cnt)
    if rc:
        raise ValueError(f"czco_autocorr failed ({rc})")
    return np.array(ac[:], dtype=np.float64), np.array(cnt[:], dtype=np.uint64)


def ssim_window(x, y, origin, window, range_mode: int = 0, global_range: float = 0.0, dims=None) -> float:
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    return float(_fn("czco_ssim_window", x)(x.ctypes.data, y.ctypes.data, nd, d, _i64(origin),
                                          _i64(window), range_mode, global_range))


def ssim(x, y, window, step=None, range_mode: int = 0, dims=None):
    """Returns (ssim, n_windows).  window/step: one value per axis (slowest-first)."""
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    if step is None:
        step = [1] * nd
    out = ctypes.c_double()
    nw = ctypes.c_uint64()
    rc = _fn("czco_ssim", x)(x.ctypes.data, y.ctypes.data, nd, d, _i64(window), _i64(step), range_mode,
                           ctypes.byref(out), ctypes.byref(nw))
    if rc == 3:
        return float("nan"), 0
    if rc:
        raise ValueError(f"czco_ssim failed ({rc})")
    return out.value, int(nw.value)


def ssim_windows(x, y, window, step=None, range_mode: int = 0, dims=None) -> np.ndarray:
    """Local SSIM of every valid window (czco_ssim_windows), shaped like the window-origin grid
    (one value per origin, slowest axis first); its mean is ssim()."""
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    shp = tuple(x.shape) if dims is None else tuple(int(v) for v in dims)
    if step is None:
        step = [1] * nd
    nw = [((n - w) // s + 1) if (n > 1 and w <= n) else (1 if n == 1 else 0)
          for n, w, s in zip(shp, window, step)]
    out = np.empty(int(np.prod(nw)), dtype=np.float64)
    rc = _fn("czco_ssim_windows", x)(x.ctypes.data, y.ctypes.data, nd, d, _i64(window), _i64(step), range_mode,
                                     out.ctypes.data)
    if rc:
        raise ValueError(f"czco_ssim_windows failed ({rc})")
    return out.reshape(nw)


def ssim_separable(x, y, window, range_mode: int = 0, dims=None):
    """Separable SSIM (step 1, <= 3 active axes) for large fields: returns (ssim, n_windows,
    n_brute), n_brute = windows recomputed by the brute force (czco_ssim_separable)."""
    x, y = _pair(x, y)
    nd, d = _dims(x, dims)
    out = ctypes.c_double()
    nw = ctypes.c_uint64()
    nb = ctypes.c_uint64()
    rc = _fn("czco_ssim_separable", x)(x.ctypes.data, y.ctypes.data, nd, d, _i64(window), range_mode,
                                       ctypes.byref(out), ctypes.byref(nw), ctypes.byref(nb))
    if rc == 3:
        return float("nan"), 0, 0
    if rc:
        raise ValueError(f"czco_ssim_separable failed ({rc})")
    return out.value, int(nw.value), int(nb.value)


def pdf(x, y, nbins: int = 100) -> Dict:
    """Error PDF and pwr-error PDF counts (czco_pdf): keys err_pdf_lo/width, err_pdf (counts),
    pwr_pdf_lo/width, pwr_pdf, n_pwr."""
    x, y = _pair(x, y)
    d = [ctypes.c_double() for _ in range(4)]
    ec = (ctypes.c_uint64 * nbins)()
    pc = (ctypes.c_uint64 * nbins)()
    npw = ctypes.c_uint64()
    rc = _fn("czco_pdf", x)(x.ctypes.data, y.ctypes.data, x.size, nbins, ctypes.byref(d[0]), ctypes.byref(d[1]),
                          ec, ctypes.byref(d[2]), ctypes.byref(d[3]), pc, ctypes.byref(npw))
    if rc:
        raise ValueError(f"czco_pdf failed ({rc})")
    return {"err_pdf_lo": d[0].value, "err_pdf_width": d[1].value, "err_pdf": np.array(ec[:], dtype=np.uint64),
            "pwr_pdf_lo": d[2].value, "pwr_pdf_width": d[3].value, "pwr_pdf": np.array(pc[:], dtype=np.uint64),
            "n_pwr": int(npw.value)}


def assess(x, y, window=None, step=None, max_lag: int = 10, range_mode: int = 0) -> Dict[str, float]:
    """All oracle metrics in one flat dict keyed like the CUDA binding's result."""
    x, y = _pair(x, y)
    nd = x.ndim
    out = dict(p1(x, y))
    out.update(deriv(x, y))
    ac, cnt = autocorr(x, y, max_lag)
    out["ac"] = ac
    out["ac_count"] = cnt
    if window is None:
        window = [8] * nd
    s, nw = ssim(x, y, window, step, range_mode)
    out["ssim"] = s
    out["n_windows"] = nw
    return out
