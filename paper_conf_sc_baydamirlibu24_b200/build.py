"""Build libjacobi_b200.so in-tree with nvcc for sm_100a (called by __graft_entry__.build())."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libjacobi_b200.so")
SOURCES = ["kernels.cu", "runtime.cu", "plan.cpp"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-std=c++17", "-lineinfo",
    "-fmad=false",                    # oracle operation order: no FMA contraction (R4)
    "-Xcompiler", "-fPIC,-O2,-ffp-contract=off",
    "-I", os.path.join(ROOT, "include"),
    "-shared", "-ldl",
]


LIB_NVSHMEM = os.path.join(HERE, "libjacobi_b200_nvshmem.so")


def nvshmem_home():
    """NVSHMEM 3.x from the nvidia-nvshmem wheel (headers + device .a + host .so), or None."""
    try:
        import nvidia
        for base in nvidia.__path__:
            d = os.path.join(base, "nvshmem")
            if os.path.exists(os.path.join(d, "lib", "libnvshmem_device.a")):
                return d
    except ImportError:
        pass
    return None


def needs_build(lib: str = LIB) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "jacobi.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(cmd, out, verbose):
    tmp = out + f".tmp{os.getpid()}"
    cmd = [*cmd, "-o", tmp]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, out)


def build(force: bool = False, verbose: bool = False) -> str:
    srcs = [os.path.join(CSRC, s) for s in SOURCES]
    if force or needs_build(LIB):
        _compile([NVCC, *FLAGS, *srcs], LIB, verbose)
    nv = nvshmem_home()
    if nv and (force or needs_build(LIB_NVSHMEM)):
        # N3 variant: same sources with -DJB_NVSHMEM, relocatable device code + NVSHMEM device lib
        _compile([NVCC, *FLAGS, "-rdc=true", "-DJB_NVSHMEM", "-I", os.path.join(nv, "include"), *srcs,
                  os.path.join(nv, "lib", "libnvshmem_device.a"), "-L", os.path.join(nv, "lib"),
                  "-l:libnvshmem_host.so.3", "-L", "/usr/local/cuda/lib64/stubs", "-lcuda",
                  "-Xlinker", "-rpath," + os.path.join(nv, "lib")], LIB_NVSHMEM, verbose)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
