"""Seeded synthetic (orig, recon) field pairs — the ONLY module shared by the oracle side and the
CUDA side (tests, bench, smoke).  It holds none of the assessment arithmetic: it only draws inputs.

Why synthetic: the paper's datasets (Hurricane 100x500x500, NYX 512^3, Scale-LETKF, Miranda —
PAPER.md L328-L330, "All data fields are stored in single precision") are not available here, so
each workload is replaced by a shape-matched field with the same structure (smooth multi-scale
signal, sparse/QCLOUD-like zeros, log-normal decades, 2-D zonal bands).  The recon models stand in
for cuSZ (the compressor the paper measures, L328):
  * "uniform": y = fl32(x + u), u ~ U[-a, a]            (BASELINE.json configs[0])
  * "quant":   y = fl32(2eb * rint(x / (2eb)))           (cuSZ-like pre-quantisation, |e| <= eb)
The full recipe is restated in DESIGN.md §3.

Determinism: everything is produced with torch float64/int64 elementwise ops whose results are
IEEE-defined (add, mul, div, round-half-even, float32 rounding) on both CPU and CUDA, from mode
tables computed once in numpy on the host, and counter-based integer hashing for noise.  Hence
`make_pair(cfg, device="cpu")` and `make_pair(cfg, device="cuda")` produce bit-identical arrays
for every kind except "lognormal"/"qcloud" (torch.exp is not correctly rounded, so CPU and CUDA may
differ by an ulp: generate those on the CPU and copy), and any z-slab [z0, z1) can be regenerated
alone (per-rank generation, sampled oracle checks).
"""
from __future__ import annotations

import dataclasses
import math
from typing import Optional, Sequence, Tuple

import numpy as np
import torch

__all__ = ["FieldSpec", "CONFIGS", "make_pair", "make_field", "uniform_noise", "config"]

_M32 = 0xFFFFFFFF


@dataclasses.dataclass(frozen=True)
class FieldSpec:
    """One synthetic workload.  dims are slowest-first (z, y, x), x contiguous (Alg. 1 puts
    lanes on the contiguous axis, L163/L183)."""
    name: str
    dims: Tuple[int, ...]
    kind: str = "smooth"          # smooth | temperature | qcloud | lognormal | zonal | step | ramp
    recon: str = "quant"          # quant | uniform | exact
    eb: float = 1e-4              # absolute error bound ("quant") or noise half-width a ("uniform")
    eb_relative: bool = False     # if True, eb is relative to the field's value range
    seed: int = 0x5EED0000
    modes: int = 8
    noise: float = 0.01           # white-noise fraction of the signal amplitude
    lo: float = 0.0               # value range of the smooth signal (before kind transform)
    hi: float = 1.0


# BASELINE.json "configs" (C1..C5); C2 has two Hurricane-like fields (temperature + QCLOUD).
CONFIGS = {
    "C1": FieldSpec("C1-64^3-uniform", (64, 64, 64), kind="smooth", recon="uniform", eb=1e-3,
                    seed=0x5EED0001),
    "C2": FieldSpec("C2-hurricane-T-100x500x500", (100, 500, 500), kind="temperature",
                    recon="quant", eb=1e-4, seed=0x5EED0002, lo=275.0, hi=285.0),
    "C2q": FieldSpec("C2-hurricane-QCLOUD-100x500x500", (100, 500, 500), kind="qcloud",
                     recon="quant", eb=1e-4, seed=0x5EED0012),
    "C3": FieldSpec("C3-nyx-512^3", (512, 512, 512), kind="lognormal", recon="quant", eb=1e-4,
                    eb_relative=True, seed=0x5EED0003),
    "C4": FieldSpec("C4-cesm-1800x3600", (1800, 3600), kind="zonal", recon="quant", eb=1e-4,
                    eb_relative=True, seed=0x5EED0004),
    "C5": FieldSpec("C5-2048^3", (2048, 2048, 2048), kind="smooth", recon="quant", eb=1e-4,
                    eb_relative=True, seed=0x5EED0005),
}


def config(name: str, dims: Optional[Sequence[int]] = None, **overrides) -> FieldSpec:
    """A named config, optionally re-shaped (parity tests use the same recipe at smaller dims)."""
    spec = CONFIGS[name]
    if dims is not None:
        overrides["dims"] = tuple(int(d) for d in dims)
    return dataclasses.replace(spec, **overrides) if overrides else spec


# ----------------------------------------------------------------------------- counter-based noise
def _hash32(x: torch.Tensor) -> torch.Tensor:
    """32-bit integer avalanche hash on int64 tensors holding values in [0, 2^32).  Multipliers are
    < 2^31 so no int64 product overflows (bit-identical on CPU and CUDA)."""
    x = x & _M32
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & _M32
    x = x ^ (x >> 15)
    x = (x * 0x6B43A9B5) & _M32
    x = x ^ (x >> 16)
    return x


def _uniform01(index: torch.Tensor, seed: int, stream: int) -> torch.Tensor:
    """U(0,1) doubles from a counter: (hash(index, seed, stream) + 0.5) / 2^32 (exact in float64)."""
    s = (seed * 0x9E37 + stream * 0x85EB + 0x1234567) & _M32
    lo = index & _M32
    hi = index >> 32
    h = _hash32(_hash32(lo ^ s) ^ hi ^ (stream * 0x27D4EB2D & _M32))
    return (h.to(torch.float64) + 0.5) * (1.0 / 4294967296.0)


def uniform_noise(shape, z0: int, seed: int, stream: int, device) -> torch.Tensor:
    """U(0,1) float64 tensor for planes [z0, z0+shape[0]) of a C-order array (counter = flat index)."""
    plane = int(np.prod(shape[1:])) if len(shape) > 1 else 1
    n = int(np.prod(shape))
    idx = torch.arange(n, dtype=torch.int64, device=device) + z0 * plane
    return _uniform01(idx, seed, stream).reshape(shape)


# ----------------------------------------------------------------------------- smooth signal
def _mode_tables(dims: Tuple[int, ...], seed: int, modes: int):
    """Per axis: `modes` cosine tables cos(2*pi*k*p/n + phi), k ~ U{1..ceil(n/8)}, amplitude ~ 1/k."""
    rng = np.random.default_rng(seed)
    amps = np.ones(modes)
    tables = []
    for n in dims:
        kmax = max(1, math.ceil(n / 8))
        ks = rng.integers(1, kmax + 1, size=modes)
        ph = rng.uniform(0.0, 2.0 * math.pi, size=modes)
        p = np.arange(n, dtype=np.float64)
        tables.append(np.cos(2.0 * math.pi * np.outer(ks, p) / max(n, 1) + ph[:, None]))
        amps = amps / ks
    # unit-variance normalisation: each separable product of D cosines has variance 2^-D
    amps = amps / math.sqrt(float(np.sum(amps ** 2)) * 2.0 ** (-len(dims)))
    return amps, tables


def _smooth(spec: FieldSpec, seed: int, z0: int, z1: int, device) -> torch.Tensor:
    """Zero-mean, ~unit-variance smooth multi-scale field on planes [z0, z1), float64."""
    dims = spec.dims
    amps, tables = _mode_tables(dims, seed, spec.modes)
    shape = (z1 - z0,) + tuple(dims[1:])
    out = torch.zeros(shape, dtype=torch.float64, device=device)
    for m in range(spec.modes):
        term = None
        for a, tab in enumerate(tables):
            t = torch.from_numpy(np.ascontiguousarray(tab[m] if a else tab[m][z0:z1])).to(device)
            view = [1] * len(dims)
            view[a] = t.numel()
            t = t.reshape(view)
            term = t if term is None else term * t
        out = out + float(amps[m]) * term
    return out


def make_field(spec: FieldSpec, z0: int = 0, z1: Optional[int] = None, device="cpu") -> torch.Tensor:
    """The original field x (float32) on planes [z0, z1)."""
    z1 = spec.dims[0] if z1 is None else z1
    shape = (z1 - z0,) + tuple(spec.dims[1:])
    g = _smooth(spec, spec.seed, z0, z1, device)
    white = uniform_noise(shape, z0, spec.seed, 1, device) * 2.0 - 1.0
    g = g + spec.noise * math.sqrt(3.0) * white          # 1 % white noise (std-matched)
    k = spec.kind
    if k in ("smooth", "temperature"):
        # map ~[-3, 3] sigma onto [lo, hi]
        f = spec.lo + (spec.hi - spec.lo) * (g / 6.0 + 0.5)
    elif k == "lognormal":                               # NYX-like density, >= 4 decades
        f = torch.exp(2.0 * g)
    elif k == "qcloud":                                  # ~70 % exact zeros, log-normal positives
        g2 = _smooth(spec, spec.seed ^ 0xABCDEF, z0, z1, device)
        f = torch.where(g2 > 0.5, 1e-3 * torch.exp(g), torch.zeros_like(g))
    elif k == "zonal":                                   # CESM-like 2-D: cos(lat) bands + waves
        ny = spec.dims[0]
        lat = (np.arange(z0, z1, dtype=np.float64) + 0.5) / ny * math.pi - math.pi / 2
        view = [z1 - z0] + [1] * (len(spec.dims) - 1)
        band = torch.from_numpy(40.0 * np.cos(lat)).to(device).reshape(view)   # host libm only
        f = 250.0 + band + 5.0 * g
    elif k == "step":                                    # adversarial: 1 | 1000 halves, tiny local std
        nx = spec.dims[-1]
        xs = torch.arange(nx, device=device)
        base = torch.where(xs < nx // 2, torch.tensor(1.0, dtype=torch.float64, device=device),
                           torch.tensor(1000.0, dtype=torch.float64, device=device))
        f = base + 1e-3 * g
    elif k == "ramp":                                    # dyadic linear ramp (exact derivatives)
        f = g * 0.0
        for a, n in enumerate(spec.dims):
            idx = torch.arange(n, dtype=torch.float64, device=device)
            if a == 0:
                idx = idx[z0:z1]
            view = [1] * len(spec.dims)
            view[a] = idx.numel()
            f = f + (2.0 ** -(a + 3)) * idx.reshape(view)
    else:
        raise ValueError(f"unknown field kind {k!r}")
    return f.to(torch.float32)


def value_range(x: torch.Tensor) -> float:
    return float(x.max().double() - x.min().double())


def make_recon(spec: FieldSpec, x: torch.Tensor, z0: int = 0, range_hint: Optional[float] = None) -> torch.Tensor:
    """The reconstructed field y (float32) for planes [z0, z0 + x.shape[0]) of `spec`."""
    eb = spec.eb
    if spec.eb_relative:
        r = range_hint if range_hint is not None else value_range(x)
        eb = eb * (r if r > 0 else 1.0)
    xd = x.to(torch.float64)
    if spec.recon == "exact":
        return x.clone()
    if spec.recon == "uniform":
        u = uniform_noise(tuple(x.shape), z0, spec.seed, 2, x.device) * 2.0 - 1.0
        return (xd + eb * u).to(torch.float32)
    if spec.recon == "quant":
        q = 2.0 * eb
        return (q * torch.round(xd / q)).to(torch.float32)
    raise ValueError(f"unknown recon model {spec.recon!r}")


def make_pair(spec: FieldSpec, z0: int = 0, z1: Optional[int] = None, device="cpu",
              range_hint: Optional[float] = None):
    """(orig, recon) float32 C-contiguous tensors of planes [z0, z1) on `device`.

    For relative error bounds on a slab, pass `range_hint` (the whole field's value range) so every
    slab uses the same eb; without it the slab's own range is used."""
    x = make_field(spec, z0, z1, device)
    y = make_recon(spec, x, z0, range_hint)
    return x.contiguous(), y.contiguous()
