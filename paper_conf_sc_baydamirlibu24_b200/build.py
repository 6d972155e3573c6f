"""Build libjacobi_b200.so in-tree with nvcc for sm_100a (called by __graft_entry__.build())."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libjacobi_b200.so")
SOURCES = ["sweep.cu", "resident.cu", "tblock.cu", "cluster.cu", "util.cu", "runtime.cu", "baselines.cu", "multiproc.cu", "plan.cpp"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMPILE_FLAGS = [
    *ARCH,
    "-O3", "-std=c++17", "-lineinfo",
    "-fmad=false",                    # oracle operation order: no FMA contraction (R4)
    "-Xcompiler", "-fPIC,-O2,-ffp-contract=off",
    "-I", os.path.join(ROOT, "include"),
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


def _run(cmd, verbose):
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)


def _build_lib(out, extra_compile, extra_link, verbose):
    """Compile every translation unit in parallel (one nvcc per TU), then link the .so."""
    from concurrent.futures import ThreadPoolExecutor

    tag = os.path.basename(out).replace(".so", "")
    objdir = os.path.join(HERE, "build", tag)
    os.makedirs(objdir, exist_ok=True)
    objs = []
    cmds = []
    for src in SOURCES:
        obj = os.path.join(objdir, src + ".o")
        objs.append(obj)
        cmds.append([NVCC, *COMPILE_FLAGS, *extra_compile, *(["-Xptxas=-v"] if verbose else []),
                     "-c", os.path.join(CSRC, src), "-o", obj])
    with ThreadPoolExecutor(max_workers=min(len(cmds), os.cpu_count() or 1)) as ex:
        list(ex.map(lambda c: _run(c, verbose), cmds))
    tmp = out + f".tmp{os.getpid()}"
    _run([NVCC, *ARCH, *extra_compile[:1], "-shared", *objs, *extra_link, "-ldl", "-o", tmp], verbose)
    os.replace(tmp, out)


def build(force: bool = False, verbose: bool = False) -> str:
    from concurrent.futures import ThreadPoolExecutor

    jobs = []
    if force or needs_build(LIB):
        jobs.append((LIB, [], []))
    nv = nvshmem_home()
    if nv and (force or needs_build(LIB_NVSHMEM)):
        # N3 variant: same sources with -DJB_NVSHMEM, relocatable device code + NVSHMEM device lib
        jobs.append((LIB_NVSHMEM, ["-rdc=true", "-DJB_NVSHMEM", "-I", os.path.join(nv, "include")],
                     [os.path.join(nv, "lib", "libnvshmem_device.a"), "-L", os.path.join(nv, "lib"),
                      "-l:libnvshmem_host.so.3", "-L", "/usr/local/cuda/lib64/stubs", "-lcuda",
                      "-Xlinker", "-rpath," + os.path.join(nv, "lib")]))
    with ThreadPoolExecutor(max_workers=2) as ex:  # both libraries at once
        for f in [ex.submit(_build_lib, out, c, l, verbose) for out, c, l in jobs]:
            f.result()
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
