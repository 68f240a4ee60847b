"""B200-native cuZ-Checker assessment hot path — thin Python binding over libczc.so.

The library (include/czc.h) exports czc_init / czc_assess / czc_assess_host / czc_free; this
module mirrors those names with argument marshalling only.  PyTorch supplies device memory and
the current CUDA stream; every step of the assessment runs in the library's sm_100a kernels.
There is NO CPU fallback: if libczc.so is missing or cannot be loaded, the first use (any call,
or attribute `lib`) raises ImportError.

    import paper_conf_cluster_yudgtc21_b200 as czc
    r = czc.assess(orig, recon)                # orig/recon: CUDA float32 (or float64) tensors
    r["psnr"], r["ssim"], r["ac"], r["der1_mae"] ...
"""
from __future__ import annotations

import ctypes
import os
from typing import Dict, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# CZC_LIB overrides the library path (development A/B timing only: tools/ab_time.py)
LIB_PATH = os.environ.get("CZC_LIB") or os.path.join(_HERE, "libczc.so")

M_P1, M_DERIV, M_AUTOCORR, M_SSIM, M_PDF = 1, 2, 4, 8, 16
F32, F64 = 0, 1      # czc_dtype
M_ALL = 0xF          # the four pattern groups (bench.py's step)
M_FULL = 0x1F        # + the error / pwr-error PDFs (Table I Category I)
MAX_LAG = 16
MAX_DIMS = 4         # ndim 1..4 (4-D fields: NEXT row f3)
PDF_MAX_BINS = 256
DERIV_FIELDS = ("der1", "der2", "grad", "div", "lap")
DERIV_STATS = ("maxabs", "mae", "mse", "rmse", "f_min", "f_max", "psnr")
STATUS = {0: "ok", 1: "invalid argument", 2: "invalid shape", 3: "unsupported dtype", 4: "CUDA error",
          5: "out of memory", 6: "communication (NCCL) error", 7: "unsupported"}


class CzcError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"czc status {status} ({STATUS.get(status, '?')}): {detail}")


class Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("stream", ctypes.c_void_p),
                ("ssim_window", ctypes.c_int * MAX_DIMS), ("ssim_step", ctypes.c_int * MAX_DIMS),
                ("ssim_range_mode", ctypes.c_int), ("ac_max_lag", ctypes.c_int), ("timing", ctypes.c_int),
                ("rank", ctypes.c_int), ("nranks", ctypes.c_int), ("nccl_uid", ctypes.c_void_p),
                ("debug_wssim", ctypes.c_void_p), ("loopback_slabs", ctypes.c_int), ("pdf_bins", ctypes.c_int),
                ("debug_der", ctypes.c_void_p)]


class Shape(ctypes.Structure):
    _fields_ = [("ndim", ctypes.c_int), ("dims", ctypes.c_int64 * MAX_DIMS), ("z0", ctypes.c_int64),
                ("nz_local", ctypes.c_int64)]


class DerivStats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_double) for k in DERIV_STATS]


_P1_DOUBLES = ("x_min", "x_max", "value_range", "err_min", "err_max", "err_maxabs", "err_mean",
               "err_absmean", "mse", "rmse", "nrmse", "psnr", "snr", "max_rel_err", "pwr_min",
               "pwr_max", "pwr_mean")


class Result(ctypes.Structure):
    _fields_ = ([("computed_mask", ctypes.c_uint64), ("n", ctypes.c_uint64)]
                + [(k, ctypes.c_double) for k in _P1_DOUBLES]
                + [("n_pwr", ctypes.c_uint64), ("pearson", ctypes.c_double), ("err_var", ctypes.c_double),
                   ("n_interior", ctypes.c_uint64), ("deriv", DerivStats * 5),
                   ("ac_max_lag", ctypes.c_int32), ("_pad0", ctypes.c_int32),
                   ("ac", ctypes.c_double * (MAX_LAG + 1)), ("ac_count", ctypes.c_uint64 * (MAX_LAG + 1)),
                   ("ssim_window", ctypes.c_int32 * MAX_DIMS), ("ssim_step", ctypes.c_int32 * MAX_DIMS),
                   ("n_windows", ctypes.c_uint64), ("ssim", ctypes.c_double),
                   ("n_ssim_exact", ctypes.c_uint64),
                   ("pdf_bins", ctypes.c_int32), ("_pad1", ctypes.c_int32),
                   ("err_pdf_lo", ctypes.c_double), ("err_pdf_width", ctypes.c_double),
                   ("pwr_pdf_lo", ctypes.c_double), ("pwr_pdf_width", ctypes.c_double),
                   ("err_pdf", ctypes.c_uint64 * PDF_MAX_BINS), ("pwr_pdf", ctypes.c_uint64 * PDF_MAX_BINS),
                   ("kernel_ms", ctypes.c_float * 6)])


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing — build it with `python -m paper_conf_cluster_yudgtc21_b200.build` "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    lib.czc_init.argtypes = [ctypes.POINTER(P), ctypes.POINTER(Config)]
    lib.czc_init.restype = ctypes.c_int
    lib.czc_assess.argtypes = [P, P, P, ctypes.POINTER(Shape), ctypes.c_int, ctypes.c_uint64, ctypes.POINTER(Result)]
    lib.czc_assess.restype = ctypes.c_int
    lib.czc_assess_host.argtypes = lib.czc_assess.argtypes
    lib.czc_assess_host.restype = ctypes.c_int
    lib.czc_free.argtypes = [P]
    lib.czc_free.restype = None
    lib.czc_strerror.argtypes = [ctypes.c_int]
    lib.czc_strerror.restype = ctypes.c_char_p
    lib.czc_last_error.argtypes = [P]
    lib.czc_last_error.restype = ctypes.c_char_p
    lib.czc_abi_version.restype = ctypes.c_int
    lib.czc_has_nccl.restype = ctypes.c_int
    lib.czc_sizeof.argtypes = [ctypes.c_int]
    lib.czc_sizeof.restype = ctypes.c_uint64
    lib.czc_combine.argtypes = [P, ctypes.c_int, ctypes.POINTER(Shape), ctypes.POINTER(Config), ctypes.c_uint64,
                                ctypes.POINTER(Result)]
    lib.czc_combine.restype = ctypes.c_int
    for what, st in ((0, Config), (1, Shape), (2, Result)):
        if lib.czc_sizeof(what) != ctypes.sizeof(st):
            raise ImportError(f"ABI mismatch: {st.__name__} is {ctypes.sizeof(st)} B here, "
                              f"{lib.czc_sizeof(what)} B in libczc.so")
    return lib


_lib = None


def get_lib():
    global _lib
    if _lib is None:
        _lib = _load()
    return _lib


def __getattr__(name):          # PEP 562: `czc.lib` loads the library on first access
    if name == "lib":
        return get_lib()
    raise AttributeError(name)


EXPORTED = ("czc_init", "czc_assess", "czc_assess_host", "czc_combine", "czc_free", "czc_strerror",
            "czc_last_error", "czc_abi_version", "czc_has_nccl", "czc_sizeof")


def _per_axis(v, ndim) -> Sequence[int]:
    if isinstance(v, int):
        return [v] * ndim + [0] * (MAX_DIMS - ndim)
    v = list(v)
    return v + [0] * (MAX_DIMS - len(v))


def make_config(ndim: int = 3, device: int = -1, stream: Optional[int] = None, ssim_window=8, ssim_step=1,
                ssim_range_mode: int = 0, ac_max_lag: int = 10, timing: bool = False, rank: int = 0,
                nranks: int = 1, nccl_uid: Optional[bytes] = None, debug_wssim: Optional[int] = None,
                loopback_slabs: int = 0, pdf_bins: int = 0, debug_der: Optional[int] = None) -> Config:
    c = Config()
    c.device = device
    c.stream = stream
    for i, w in enumerate(_per_axis(ssim_window, ndim)):
        c.ssim_window[i] = int(w)
    for i, s in enumerate(_per_axis(ssim_step, ndim)):
        c.ssim_step[i] = int(s)
    c.ssim_range_mode = ssim_range_mode
    c.ac_max_lag = ac_max_lag
    c.timing = int(bool(timing))
    c.rank, c.nranks = rank, nranks
    c._uid = None
    if nccl_uid is not None:
        c._uid = ctypes.create_string_buffer(bytes(nccl_uid), 128)
        c.nccl_uid = ctypes.cast(c._uid, ctypes.c_void_p)
    c.debug_wssim = debug_wssim
    c.loopback_slabs = loopback_slabs
    c.pdf_bins = pdf_bins
    c.debug_der = debug_der
    return c


def czc_init(cfg: Config) -> int:
    """czc_init(&ctx, cfg) -> ctx handle (int).  Raises CzcError on failure."""
    h = ctypes.c_void_p()
    lib = get_lib()
    rc = lib.czc_init(ctypes.byref(h), ctypes.byref(cfg))
    if rc:
        raise CzcError(rc, lib.czc_strerror(rc).decode())
    return h.value


def czc_free(ctx: int) -> None:
    get_lib().czc_free(ctx)


def make_shape(dims: Sequence[int], z0: int = 0, nz_local: int = 0) -> Shape:
    s = Shape()
    s.ndim = len(dims)
    for i, d in enumerate(dims):
        s.dims[i] = int(d)
    s.z0, s.nz_local = int(z0), int(nz_local)
    return s


def result_dict(r: Result) -> Dict:
    out = {"computed_mask": r.computed_mask, "n": r.n}
    for k in _P1_DOUBLES:
        out[k] = getattr(r, k)
    out.update(n_pwr=r.n_pwr, pearson=r.pearson, err_var=r.err_var, n_interior=r.n_interior)
    for i, f in enumerate(DERIV_FIELDS):
        for s in DERIV_STATS:
            out[f"{f}_{s}"] = getattr(r.deriv[i], s)
    out["ac_max_lag"] = r.ac_max_lag
    T = max(r.ac_max_lag, 0)
    out["ac"] = np.array(r.ac[:T + 1], dtype=np.float64)
    out["ac_count"] = np.array(r.ac_count[:T + 1], dtype=np.uint64)
    out["ssim_window"] = list(r.ssim_window)
    out["ssim_step"] = list(r.ssim_step)
    out["n_windows"] = r.n_windows
    out["ssim"] = r.ssim
    out["n_ssim_exact"] = r.n_ssim_exact
    nb = max(r.pdf_bins, 0)
    out["pdf_bins"] = nb
    for k in ("err_pdf_lo", "err_pdf_width", "pwr_pdf_lo", "pwr_pdf_width"):
        out[k] = getattr(r, k)
    out["err_pdf"] = np.array(r.err_pdf[:nb], dtype=np.uint64)
    out["pwr_pdf"] = np.array(r.pwr_pdf[:nb], dtype=np.uint64)
    out["kernel_ms"] = list(r.kernel_ms)
    return out


def czc_assess(ctx: int, orig_ptr: int, recon_ptr: int, shape: Shape, mask: int = M_ALL, host: bool = False,
               dtype: int = F32) -> Dict:
    """czc_assess / czc_assess_host with raw pointers; returns the result as a dict."""
    r = Result()
    lib = get_lib()
    fn = lib.czc_assess_host if host else lib.czc_assess
    rc = fn(ctx, orig_ptr, recon_ptr, ctypes.byref(shape), dtype, mask, ctypes.byref(r))
    if rc:
        raise CzcError(rc, lib.czc_last_error(ctx).decode(errors="replace"))
    return result_dict(r)


def czc_combine(records: bytes, nrecords: int, dims: Sequence[int], cfg: Config, mask: int = M_ALL) -> Dict:
    """Host-only rank-ordered combine + finish of per-slab records (czc_sizeof(3) bytes each)."""
    lib = get_lib()
    r = Result()
    buf = ctypes.create_string_buffer(bytes(records), len(records))
    rc = lib.czc_combine(buf, nrecords, ctypes.byref(make_shape(dims)), ctypes.byref(cfg), mask, ctypes.byref(r))
    if rc:
        raise CzcError(rc, "czc_combine")
    return result_dict(r)


class Assessor:
    """A czc context bound to one device and stream (default: torch's current stream)."""

    def __init__(self, ndim: int = 3, device: Optional[int] = None, stream=None, **cfg):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("paper_conf_cluster_yudgtc21_b200 needs a CUDA device (no CPU fallback)")
        dev = torch.cuda.current_device() if device is None else int(device)
        if stream is None:
            stream = torch.cuda.current_stream(dev)
        self.device = dev
        self.stream = stream
        self.cfg = make_config(ndim=ndim, device=dev, stream=stream.cuda_stream, **cfg)
        self.ctx = czc_init(self.cfg)

    def assess(self, orig, recon, mask: int = M_ALL, dims=None, z0: int = 0) -> Dict:
        """orig/recon: CUDA C-contiguous tensors, both float32 or both float64 (slab mode: this
        rank's planes, with the GLOBAL dims passed in `dims` and the first plane index in `z0`)."""
        import torch
        dts = {torch.float32: F32, torch.float64: F64}
        for t in (orig, recon):
            if not (t.is_cuda and t.dtype in dts and t.is_contiguous()):
                raise TypeError("orig/recon must be contiguous float32 or float64 CUDA tensors")
        if orig.dtype != recon.dtype:
            raise TypeError("orig and recon must have the same dtype")
        if orig.shape != recon.shape:
            raise ValueError("orig and recon must have the same shape")
        for t in (orig, recon):               # kernels of this context run on self.device only
            if t.device.index != self.device:
                raise ValueError(f"tensor on cuda:{t.device.index}, context bound to cuda:{self.device}")
        gdims = list(orig.shape) if dims is None else list(dims)
        shape = make_shape(gdims, z0, orig.shape[0] if dims is not None else 0)
        return czc_assess(self.ctx, orig.data_ptr(), recon.data_ptr(), shape, mask, dtype=dts[orig.dtype])

    def assess_host(self, orig, recon, mask: int = M_ALL, dims=None, z0: int = 0) -> Dict:
        """Same, from HOST buffers (numpy arrays or CPU tensors, ideally pinned): the library copies
        them to the device on its stream inside the call."""
        o = orig if isinstance(orig, np.ndarray) else orig.numpy()
        r_ = recon if isinstance(recon, np.ndarray) else recon.numpy()
        dts = {np.dtype(np.float32): F32, np.dtype(np.float64): F64}
        if o.dtype not in dts or r_.dtype != o.dtype or not o.flags.c_contiguous or not r_.flags.c_contiguous:
            raise TypeError("orig/recon must be C-contiguous, both float32 or both float64")
        gdims = list(o.shape) if dims is None else list(dims)
        shape = make_shape(gdims, z0, o.shape[0] if dims is not None else 0)
        return czc_assess(self.ctx, o.ctypes.data, r_.ctypes.data, shape, mask, host=True, dtype=dts[o.dtype])

    def close(self):
        if getattr(self, "ctx", None):
            czc_free(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def assess(orig, recon, mask: int = M_ALL, **cfg) -> Dict:
    """One-shot assessment of two CUDA float32 / float64 tensors (creates and frees a context)."""
    cfg.setdefault("device", orig.device.index if orig.is_cuda else None)
    with Assessor(ndim=orig.dim(), **cfg) as a:
        return a.assess(orig, recon, mask)
