"""Build the in-tree C-ABI library ``liblda.so`` for sm_100a with nvcc.

    python -m paper_conf_hpdc_xie0lt19_b200._build

No torch.utils.cpp_extension: the library has a plain C ABI (include/lda.h)
and is loaded with ctypes.  The .so is written next to this file so it ships
to the GPU box with the repo snapshot.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "liblda.so")
SOURCES = ["api.cpp", "comm.cpp", "host_prep.cpp", "kernels.cu", "layout_gpu.cu"]
HEADERS = ["lda_internal.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "lda.h"),
                                                                 __file__]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    """Compile liblda.so (or a variant at `out` with extra -D defines)."""
    lib_path = out or LIB
    if out is None and not force and not _stale():
        return LIB
    objs = []
    build_dir = os.path.join(PKG, "build", os.path.basename(lib_path))
    os.makedirs(build_dir, exist_ok=True)
    common = ["-std=c++17", "-O3", "-lineinfo", "-Xcompiler", "-fPIC,-O3", "-I", os.path.join(ROOT, "include")]
    common += [f"-D{d}" for d in defines]
    for src in SOURCES:
        obj = os.path.join(build_dir, src + ".o")
        cmd = [NVCC, *ARCH, *common, "-c", os.path.join(CSRC, src), "-o", obj]
        if src.endswith(".cu") and verbose:
            cmd += ["-Xptxas", "-v"]
        if verbose:
            print(" ".join(cmd), flush=True)
        subprocess.check_call(cmd)
        objs.append(obj)
    tmp = lib_path + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-ldl", "-lpthread"]
    if verbose:
        print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)
    os.replace(tmp, lib_path)
    return lib_path


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
