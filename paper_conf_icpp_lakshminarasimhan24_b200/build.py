"""Build libbrickdl.so (the C-ABI library) in-tree for sm_100a with nvcc.

    python -m paper_conf_icpp_lakshminarasimhan24_b200.build [--force]
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libbrickdl.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SOURCES = [
    "layout.cpp",
    "plan.cpp",
    "run.cu",
    "kernels/brickify.cu",
    "kernels/brickify_tma.cu",
    "kernels/chain_brick.cu",
    "kernels/chain_tc.cu",
    "kernels/chain_tc_ws.cu",
    "kernels/chain_tc_pair.cu",
    "kernels/chain_tc_gen.cu",
]
FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=default",
    "--expt-relaxed-constexpr",
    "-I", os.path.join(ROOT, "include"),
] + os.environ.get("BDL_EXTRA_NVCC_FLAGS", "").split()   # e.g. -DBDL_DEBUG for the timing knobs (A/B runs only)


def _headers():
    hs = [os.path.join(ROOT, "include", "brickdl.h")]
    for d, _, fs in os.walk(CSRC):
        hs += [os.path.join(d, f) for f in fs if f.endswith((".h", ".cuh"))]
    return hs


def _compile(src: str, verbose: bool) -> str:
    path = os.path.join(CSRC, src)
    obj = os.path.join(BUILD, src.replace("/", "_") + ".o")
    newest = max(os.path.getmtime(h) for h in _headers() + [path])
    if os.path.exists(obj) and os.path.getmtime(obj) >= newest:
        return obj
    cmd = [NVCC, *FLAGS, "-c", "-x", "cu" if src.endswith(".cu") else "c++", path, "-o", obj]
    if src.endswith(".cu") and verbose:
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    if verbose and r.stderr:
        sys.stderr.write(r.stderr)
    return obj


MB_SRC = os.path.join(CSRC, "microbench", "atomics.cu")
MB_LIB = os.path.join(PKG, "libbdl_microbench.so")


def build_microbench(force: bool = False) -> str:
    """Memo-atomics microbenchmark library (measurement infrastructure, tools/microbench.py)."""
    if force or not os.path.exists(MB_LIB) or os.path.getmtime(MB_LIB) < os.path.getmtime(MB_SRC):
        cmd = [NVCC, *FLAGS, "-shared", MB_SRC, "-o", MB_LIB, "-lcudart"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for microbench:\n{r.stderr}")
    return MB_LIB


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    if force:
        for f in os.listdir(BUILD):
            os.remove(os.path.join(BUILD, f))
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), SOURCES))
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", LIB, *objs, "-lcudart"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
    build_microbench(force)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
