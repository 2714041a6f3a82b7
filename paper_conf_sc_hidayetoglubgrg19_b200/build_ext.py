"""Build libmemxct.so (the C-ABI CUDA library) in-tree with nvcc for sm_100a.

    python -m paper_conf_sc_hidayetoglubgrg19_b200.build_ext [--force]

Each csrc/*.cu is compiled separately (-O3 -lineinfo, -gencode arch=compute_100a,code=sm_100a;
trace.cu additionally with --fmad=false so the geometry is exactly the correctly rounded
expressions of reading R4) and linked into one shared object next to this file.  The CUDA runtime
is linked statically, so the .so only needs the driver.
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
OUT = os.path.join(PKG, "libmemxct.so")
BUILD = os.path.join(PKG, "build")

SOURCES = ["api.cu", "hilbert.cu", "trace.cu", "layout.cu", "spmv.cu", "cg.cu", "comm.cu", "exchange.cu",
           "sirt.cu", "peer.cu", "proccomm.cu", "rle.cu"]
EXTRA = {"trace.cu": ["--fmad=false"]}
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_include() -> str:
    """nccl.h for the declarations only: libnccl.so.2 is dlopen'ed at run time (the one torch
    already loaded), so the library has no link-time NCCL dependency."""
    try:
        import importlib.util
        spec = importlib.util.find_spec("nvidia.nccl")
        for loc in (spec.submodule_search_locations or []):
            if os.path.exists(os.path.join(loc, "include", "nccl.h")):
                return os.path.join(loc, "include")
    except Exception:
        pass
    return "/usr/include"


def _deps_mtime() -> float:
    files = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(INCLUDE, "memxct.h")]
    return max(os.path.getmtime(f) for f in files)


def up_to_date() -> bool:
    return os.path.exists(OUT) and os.path.getmtime(OUT) >= _deps_mtime()


# experiment builds only (scripts/build_variant.sh): extra nvcc flags and another output name
VARIANT_FLAGS = os.environ.get("MEMXCT_VARIANT_FLAGS", "").split()
if os.environ.get("MEMXCT_VARIANT"):
    OUT = os.path.join(PKG, f"libmemxct_{os.environ['MEMXCT_VARIANT']}.so")
    BUILD = os.path.join(PKG, "build", os.environ["MEMXCT_VARIANT"])


def _compile(src: str) -> str:
    obj = os.path.join(BUILD, src.replace(".cu", ".o"))
    cmd = [NVCC, "-c", "-O3", "-lineinfo", "-std=c++17", *ARCH, "-Xcompiler", "-fPIC", *VARIANT_FLAGS,
           "-Xptxas", "-v", "-I", INCLUDE, "-I", CSRC, "-I", _nccl_include(), *EXTRA.get(src, []),
           os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    with open(obj + ".ptxas.txt", "w") as f:
        f.write(r.stderr)
    return obj


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and up_to_date():
        return OUT
    os.makedirs(BUILD, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=min(len(SOURCES), os.cpu_count() or 4)) as ex:
        objs = list(ex.map(_compile, SOURCES))
    tmp = OUT + f".{os.getpid()}.tmp"
    cmd = [NVCC, "-shared", *ARCH, "-o", tmp, *objs, "-cudart", "static", "-ldl"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, OUT)
    if verbose:
        print(f"built {OUT}")
    return OUT


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
