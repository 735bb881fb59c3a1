"""Build libttlg.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libttlg.so")
SOURCES = ["api.cpp", "planner.cpp", "model.cpp", "kernels.cu"]
HEADERS = ["ttlg_internal.h", "model.h", "model_coeffs.h", "model_gbt.h", "model_gbt2.h",
           "model_gbt3.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS]
    deps.append(os.path.join(ROOT, "include", "ttlg.h"))
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    """Build libttlg.so (or, for A/B experiments, `out` with extra -D defines)."""
    if out is None and not force and not _stale():
        return LIB
    cmd = [NVCC, "-O3", "-std=c++17", "-lineinfo", *ARCH, "-shared", "-Xcompiler", "-fPIC",
           "-Xcompiler", "-Wall", "-cudart", "shared", "-Xptxas", "-v" if verbose else "-O3",
           "-I", os.path.join(ROOT, "include"),
           "-Xlinker", "-rpath,/usr/local/cuda/lib64",
           *[f"-D{d}" for d in defines],
           "-o", (out or LIB) + ".tmp"]
    cmd += [os.path.join(CSRC, s) for s in SOURCES]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc build of libttlg.so failed")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace((out or LIB) + ".tmp", out or LIB)
    return out or LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
