"""Build libsf.so (CUDA C++ for sm_100a) in-tree with nvcc.

    python -m paper_conf_ipps_zhangdmwbf17_b200.build        # incremental
    python -m paper_conf_ipps_zhangdmwbf17_b200.build --force

nvcc cross-compiles without a GPU, so this runs on the CPU build box too.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
# SF_VARIANT=name (A/B builds only): objects under _build_<name>, library
# libsf_<name>.so, SF_VARIANT_FLAGS added to the fused-pair objects; loaded
# with SF_LIB=<path> (sf.py)
_VARIANT = os.environ.get("SF_VARIANT", "")
BUILD = os.path.join(PKG, "_build" + (f"_{_VARIANT}" if _VARIANT else ""))
LIB = os.path.join(PKG, f"libsf_{_VARIANT}.so" if _VARIANT else "libsf.so")
_VFLAGS = os.environ.get("SF_VARIANT_FLAGS", "").split() if _VARIANT else []
_VAFLAGS = os.environ.get("SF_VARIANT_ALL_FLAGS", "").split() if _VARIANT else []   # every object
# (source, object, extra flags): the fused GSRB source is built for two tile shapes
SOURCES = [("level.cu", "level.o", []), ("kernels.cu", "kernels.o", []),
           ("kernels_pair.cu", "kernels_pair.o", []),
           ("gsrb_fused.cu", "gsrb_fused_t32.o",
            ["-DSF_GSRB_TX=32", "-DSF_GSRB_PF=5", "-DSF_GSRB_SUFFIX=_t32"]),
           ("gsrb_fused.cu", "gsrb_fused_t64.o",
            ["-DSF_GSRB_TX=64", "-DSF_GSRB_PF=4", "-DSF_GSRB_SUFFIX=_t64"]),
           ("gsrb_fused.cu", "gsrb_fused_t32w4.o",
            ["-DSF_GSRB_TX=32", "-DSF_GSRB_PF=2", "-DSF_GSRB_NWARP=4", "-DSF_GSRB_MINB=3",
             "-DSF_GSRB_SUFFIX=_t32w4"]),
           # the fused pair + residual + restriction (delta form; host side + fix-up)
           ("gsrb_rr.cu", "gsrb_rr.o", []),
           ("comm.cu", "comm.o", []), ("mg.cu", "mg.o", []), ("coarse.cu", "coarse.o", []),
           ("gsrb_twopair.cu", "gsrb_twopair.o", []),
           ("stencil.cu", "stencil.o", [])]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
         "--expt-relaxed-constexpr", "-I", INCLUDE, "-I", CSRC]


def _needs(obj, deps):
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(spec, force):
    src, obj, extra = spec
    s = os.path.join(CSRC, src)
    o = os.path.join(BUILD, obj)
    deps = [s, os.path.join(CSRC, "sf_internal.h"), os.path.join(CSRC, "tma_common.cuh"),
            os.path.join(CSRC, "cell_ops.cuh"),
            os.path.join(INCLUDE, "sf.h")]
    if not force and not _needs(o, deps):
        return o, ""
    if src == "gsrb_fused.cu":
        extra = [*extra, *_VFLAGS]
    cmd = [NVCC, *ARCH, *FLAGS, *extra, *_VAFLAGS, "-c", s, "-o", o]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    return o, r.stderr


def build(force=False, verbose=False):
    os.makedirs(BUILD, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        res = list(ex.map(lambda s: _compile(s, force), SOURCES))
    objs = [o for o, _ in res]
    if verbose:
        for _, log in res:
            if log:
                print(log, file=sys.stderr)
    if force or _needs(LIB, objs):
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "shared", "-o", tmp, *objs, "-ldl",
               "-Xlinker", "-rpath=/usr/local/cuda/lib64"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
