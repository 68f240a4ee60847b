"""In-tree build of libczc.so (the C-ABI library) for sm_100a.

    python -m paper_conf_cluster_yudgtc21_b200.build [--force]

Each .cu under csrc/ is compiled with nvcc (-gencode arch=compute_100a,code=sm_100a -lineinfo
-O3) in parallel and linked into paper_conf_cluster_yudgtc21_b200/libczc.so with NCCL (slab
mode).  The .so is git-ignored but travels to the GPU box with the gpurun snapshot.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# development A/B builds (tools/ab_build.py): extra nvcc flags and another output path
EXTRA = os.environ.get("CZC_NVCC_EXTRA", "").split()
OBJ = os.environ.get("CZC_OBJ_DIR") or os.path.join(HERE, "build_obj")
SO = os.environ.get("CZC_SO_OUT") or os.path.join(HERE, "libczc.so")
ROOT = os.path.dirname(HERE)
SOURCES = ["czc_api.cu", "czc_comm.cu", "p1_reduce.cu", "p2_stencil.cu", "p3_ssim.cu", "p4_generic.cu"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found: the CUDA extension cannot be built")


def _torch_nccl():
    """(include dir, lib dir) of the NCCL that PyTorch loads (the `nvidia-nccl` wheel), or None.
    libczc.so links that one, not the system libnccl: both carry the soname libnccl.so.2, and
    whichever a process loads first serves both, so an older system copy loaded through libczc
    before torch would leave torch's newer NCCL symbols unresolved."""
    import importlib.util
    try:
        spec = importlib.util.find_spec("nvidia.nccl")
    except (ImportError, ValueError):
        spec = None
    for loc in (list(spec.submodule_search_locations) if spec else []):
        inc, lib = os.path.join(loc, "include"), os.path.join(loc, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")) and os.path.exists(os.path.join(lib, "libnccl.so.2")):
            return inc, lib
    return None


def _have_nccl() -> bool:
    return _torch_nccl() is not None or os.path.exists("/usr/include/nccl.h")


def _flags():
    f = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "-Xptxas", "-O3",
                "-I" + os.path.join(ROOT, "include")] + EXTRA
    if _have_nccl():
        f.append("-DCZC_WITH_NCCL")
        tn = _torch_nccl()
        if tn:
            f.append("-I" + tn[0])
    return f


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    nvcc = _nvcc()
    os.makedirs(OBJ, exist_ok=True)
    headers = [os.path.join(CSRC, h) for h in os.listdir(CSRC) if h.endswith((".cuh", ".h"))]
    headers.append(os.path.join(ROOT, "include", "czc.h"))
    jobs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(OBJ, src.replace(".cu", ".o"))
        if force or _stale(o, [s] + headers + [__file__]):
            jobs.append((s, o))

    def run(job):
        s, o = job
        cmd = [nvcc] + _flags() + ["-c", s, "-o", o]
        if verbose:
            print(" ".join(cmd), flush=True)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {os.path.basename(s)}:\n{r.stderr}")
        return o

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        list(ex.map(run, jobs))
    objs = [os.path.join(OBJ, s.replace(".cu", ".o")) for s in SOURCES]
    if force or jobs or _stale(SO, objs):
        cmd = [nvcc] + ARCH + ["-shared", "-o", SO + ".tmp"] + objs + ["-lcudart_static", "-ldl"]
        tn = _torch_nccl()
        if tn:
            cmd += ["-L" + tn[1], "-l:libnccl.so.2", "-Xlinker", "-rpath=" + tn[1]]
        elif _have_nccl():
            cmd.append("-lnccl")
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
        os.replace(SO + ".tmp", SO)
    return SO


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
