"""Build librtlsim.so in-tree for sm_100a (nvcc; no JIT cache, no torch types).

The .so is the product: the C ABI of include/rtlsim.h. It links the CUDA
runtime statically so the same file loads on the GPU box and on this CPU-only
build host (where only host-only compile / stats calls work).
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "librtlsim.so")
SOURCES = ["compile.cpp", "kernels.cu", "runtime.cu", "jit.cpp"]
HEADERS = ["program.h", "kernels.h", "device_ops.cuh", "jit_rt.cu", "jit.h"]
JIT_RT_PTX = os.path.join(HERE, "jit_rt.ptx")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _newest_input() -> float:
    files = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    files.append(os.path.join(ROOT, "include", "rtlsim.h"))
    return max(os.path.getmtime(f) for f in files)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= _newest_input():
        return LIB
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    cmd = [nvcc, "-O3", "-std=c++17", *ARCH, "-lineinfo",
           "-Xcompiler", "-fPIC,-O2", "-shared", "-cudart", "static",
           "-I", os.path.join(ROOT, "include"),
           "-o", LIB + ".tmp"] + [os.path.join(CSRC, f) for f in SOURCES] + [
           "-L/usr/local/cuda/lib64", "-lnvptxcompiler_static", "-ldl", "-lpthread"]
    if verbose:
        cmd[1:1] = ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building librtlsim.so")
    # PTX of the device functions JIT modules call (prepended to each module)
    r2 = subprocess.run([nvcc, "-ptx", "-rdc=true", "-O3", "-std=c++17", "-arch=compute_100a",
                         "-I", os.path.join(ROOT, "include"), "-o", JIT_RT_PTX, os.path.join(CSRC, "jit_rt.cu")],
                        capture_output=True, text=True)
    if r2.returncode != 0:
        sys.stderr.write(r2.stdout + r2.stderr)
        raise RuntimeError("nvcc failed building jit_rt.ptx")
    os.replace(LIB + ".tmp", LIB)
    if verbose:
        sys.stderr.write(r.stderr)
    return LIB


if __name__ == "__main__":
    build(force=True, verbose="-v" in sys.argv)
    print(LIB)
