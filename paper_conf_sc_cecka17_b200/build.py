"""Build the CUDA library in-tree: nvcc -> paper_conf_sc_cecka17_b200/libfmmfft.so (sm_100a).

Usage: python -m paper_conf_sc_cecka17_b200.build [--force]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libfmmfft.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include() -> str:
    cands = []
    try:
        import nvidia.nccl  # type: ignore
        cands.append(os.path.join(list(nvidia.nccl.__path__)[0], "include"))
    except Exception:
        pass
    cands += ["/usr/include", "/usr/local/cuda/include"]
    for c in cands:
        if os.path.exists(os.path.join(c, "nccl.h")):
            return c
    raise RuntimeError("nccl.h not found")


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if c and os.path.exists(c):
            return c
    return "nvcc"


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh")) +
                  glob.glob(os.path.join(CSRC, "*.hpp")) + [os.path.join(ROOT, "include", "fmmfft.h")])


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


# No --split-compile: with it, nvcc's partition of the translation unit changed the register
# allocation of unrelated kernels from build to build (k_m2l_lvl 160 vs 209 registers, k_m2m_lvl
# 160 vs 195, measured ~3 % of the cfg3 step) — one partition gives reproducible code.
def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           "-Xcompiler", "-fvisibility=hidden", "--expt-relaxed-constexpr",
           "-I", os.path.join(ROOT, "include"), "-I", _nccl_include(),
           os.path.join(CSRC, "fmmfft.cu"), "-o", LIB + ".tmp", "-ldl"]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), flush=True)
    subprocess.run(cmd, check=True)
    os.replace(LIB + ".tmp", LIB)
    return LIB


def build_variant(name: str, defines) -> str:
    """A tuning build with extra -D macros: paper_conf_sc_cecka17_b200/libfmmfft_<name>.so (select it
    with FMMFFT_LIB=<path>; the default library is unaffected)."""
    out = os.path.join(PKG, f"libfmmfft_{name}.so")
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           "-Xcompiler", "-fvisibility=hidden", "--expt-relaxed-constexpr",
           *[f"-D{d}" for d in defines], "-I", os.path.join(ROOT, "include"), "-I", _nccl_include(),
           os.path.join(CSRC, "fmmfft.cu"), "-o", out, "-ldl"]
    subprocess.run(cmd, check=True)
    return out


CMP_SRC = os.path.join(ROOT, "comparators", "cufftxt.cu")
CMP_LIB = os.path.join(ROOT, "comparators", "libcufftxt_cmp.so")


def build_comparator(force: bool = False) -> str:
    """The cuFFTXt comparator (comparators/cufftxt.cu, a library call timed by bench.py at G > 1;
    not part of the product path)."""
    if not force and os.path.exists(CMP_LIB) and os.path.getmtime(CMP_LIB) >= os.path.getmtime(CMP_SRC):
        return CMP_LIB
    subprocess.run([_nvcc(), *ARCH, "-O2", "-shared", "-Xcompiler", "-fPIC", CMP_SRC, "-o", CMP_LIB + ".tmp", "-lcufft"],
                   check=True)
    os.replace(CMP_LIB + ".tmp", CMP_LIB)
    return CMP_LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    build_comparator(force="--force" in sys.argv)
    print(LIB)
