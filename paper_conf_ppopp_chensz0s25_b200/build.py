"""Builds libnm.so (the C-ABI library of include/nm.h) in-tree with nvcc for sm_100a.

    python -m paper_conf_ppopp_chensz0s25_b200.build [--force]

Objects go to paper_conf_ppopp_chensz0s25_b200/_build/, the library to
paper_conf_ppopp_chensz0s25_b200/libnm.so (git-ignored, shipped to the GPU box by gpurun).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libnm.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SOURCES = ["capi.cu", "pack.cu", "spmm_sm100.cu", "spmm_full_sm100.cu", "spmm_tm_sm100.cu", "ops.cu", "models.cu", "counts.cu", "gcn.cu", "reorder.cpp",
           "reorder_gpu.cu"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-I" + os.path.join(ROOT, "include"),
          "-Xcompiler", "-fPIC,-fopenmp,-fvisibility=hidden", "--expt-relaxed-constexpr"]
# tuning experiments only (e.g. NM_NVCC_FLAGS="-DNM_LOAD_GROUPS=4"); the product build sets none
COMMON += os.environ.get("NM_NVCC_FLAGS", "").split()


def _deps_mtime() -> float:
    m = os.path.getmtime(os.path.join(ROOT, "include", "nm.h"))
    for f in os.listdir(CSRC):
        m = max(m, os.path.getmtime(os.path.join(CSRC, f)))
    return m


def _compile(src: str, verbose: bool) -> str:
    out = os.path.join(OBJ, src + ".o")
    cmd = [NVCC] + ARCH + COMMON + ["-c", os.path.join(CSRC, src), "-o", out]
    if src.endswith(".cpp"):
        cmd[1:1] = ["-x", "cu"]
    if verbose and src.startswith("spmm"):
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, " ".join(cmd), r.stderr))
    if verbose and r.stderr.strip():
        sys.stderr.write(r.stderr)
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= _deps_mtime():
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), SOURCES))
    tmp = LIB + ".tmp%d" % os.getpid()
    cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-lcublasLt", "-lgomp",
                                                          "-Xcompiler", "-fopenmp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("link failed:\n%s\n%s" % (" ".join(cmd), r.stderr))
    os.replace(tmp, LIB)
    return LIB


BASELINE_SRC = os.path.join(ROOT, "bench_support", "cusparse_shim.cu")
BASELINE_LIB = os.path.join(ROOT, "bench_support", "libcusparse_shim.so")


def build_baseline(force: bool = False) -> str:
    """cuSPARSE comparison shim used by bench.py (baseline, not part of libnm)."""
    if not force and os.path.exists(BASELINE_LIB) and \
            os.path.getmtime(BASELINE_LIB) >= os.path.getmtime(BASELINE_SRC):
        return BASELINE_LIB
    tmp = BASELINE_LIB + ".tmp%d" % os.getpid()
    cmd = [NVCC] + ARCH + ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", BASELINE_SRC,
                           "-o", tmp, "-lcusparse"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("baseline shim build failed:\n%s" % r.stderr)
    os.replace(tmp, BASELINE_LIB)
    return BASELINE_LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
    print(build_baseline(force="--force" in sys.argv))
