"""In-tree build of libtemco.so (sm_100a).  `python -m paper_conf_icpp_songljkj0024_b200.build`."""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
# experiment variants: TEMCO_VARIANT=name TEMCO_EXTRA_FLAGS="-DTEMCO_TRACE" builds
# build/exp/libtemco_<name>.so (select it at run time with TEMCO_LIB)
VARIANT = os.environ.get("TEMCO_VARIANT", "")
EXTRA = os.environ.get("TEMCO_EXTRA_FLAGS", "").split()
BUILD = os.path.join(ROOT, "build", "temco" + ("_" + VARIANT if VARIANT else ""))
LIB = os.path.join(ROOT, "build", "exp", f"libtemco_{VARIANT}.so") if VARIANT else os.path.join(PKG, "libtemco.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SOURCES = ["planner.cpp", "capi.cu", "kernels_simt.cu", "kernels_tc.cu", "kernels_tc_wide.cu", "kernels_conv.cu", "kernels_mma.cu", "kernels_stem.cu", "kernels_rank.cu", "kernels_cat.cu", "kernels_pair.cu", "kernels_gemm.cu", "kernels_tile.cu"]
GENCODE = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
          "--expt-relaxed-constexpr", "-I" + os.path.join(ROOT, "include")]


def _headers():
    return [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))] + \
           [os.path.join(ROOT, "include", "temco.h")]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src, verbose):
    s = os.path.join(CSRC, src)
    o = os.path.join(BUILD, src + ".o")
    if not _stale(o, [s] + _headers()):
        return o
    cmd = [NVCC] + GENCODE + COMMON + EXTRA + ["-c", s, "-o", o]
    if src.endswith(".cu"):
        cmd += ["-Xptxas", "-v"] if verbose else []
    if verbose:
        print(" ".join(cmd), flush=True)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile {src} failed:\n{r.stdout}\n{r.stderr}")
    if verbose and r.stderr:
        print(r.stderr, flush=True)
    return o


def build(verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), SOURCES))
    if _stale(LIB, objs):
        cmd = [NVCC] + GENCODE + ["-shared", "-o", LIB] + objs
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    return LIB


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv))
