"""CPU oracle for the CPU-Free Jacobi hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_sc_baydamirlibu24_b200``) never imports it and shares no code with it.

Two independent implementations of the same definition (§2.1 Jacobi for
Laplace with Dirichlet boundary; P:355 fixed iteration count; P:394 previous-time-step,
out-of-place semantics; 2D5pt P:346, 3D7pt P:535):

* ``jacobi(field, iters, nthreads)`` — the plain C loop in ``jacobi_oracle.c`` (ctypes).
* ``jacobi_numpy(field, iters)`` — the same definition with numpy slicing.

Both use the operation order of DESIGN.md readings R2/R3: ((((x+1)+(x-1))+(y+1))+(y-1))
[+(z+1))+(z-1)] then ×0.25 (2D) or ×fl(1/6) (3D), IEEE fp64, no FMA, no FTZ.

Pins (tests/test_oracle.py, all ``-m "not gpu"``): exact rational arithmetic (2D),
closed-form eigenmode decay, convergence to scipy's sparse direct solve of the discrete
Laplace equation, one Jacobi step equal to the textbook matrix splitting
u' = D^{-1}(b - (A-D)u) built with scipy.sparse, stationary constant / linear / discrete-
harmonic fields, untouched boundary, maximum principle, mirror symmetry, run splitting.
The 3D association order is fixed by reading R2 and is "parity unpinned" by the paper
beyond the within-tolerance pins.

``jacobi_converge`` adds SURVEY §8(f) N4 (not in the paper, which runs a fixed count): the
L2 norm of the update sqrt(sum over interior cells of (u_new - u_old)^2) every `every` iterations
and stop once it is <= `tol` (reading R19).  Parity unpinned by the paper.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "jacobi_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
C6 = float.fromhex("0x1.5555555555555p-3")  # fl(1/6), reading R3

_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc -O2 -ffp-contract=off -fopenmp; no -ffast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        cmd = ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
               "-fPIC", "-shared", "-o", tmp, _SRC]
        subprocess.check_call(cmd)
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_jacobi.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
                                      ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
        lib.oracle_jacobi.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _dims(field: np.ndarray):
    if field.ndim == 2:
        ny, nx = field.shape
        return nx, ny, 1, 5
    if field.ndim == 3:
        nz, ny, nx = field.shape
        if nz == 1:
            return nx, ny, 1, 5
        return nx, ny, nz, 7
    raise ValueError("field must be (ny, nx) or (nz, ny, nx)")


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def jacobi(field: np.ndarray, iters: int, nthreads: int = 1) -> np.ndarray:
    """C oracle: `iters` Jacobi iterations of `field` (2D: (ny,nx) or (1,ny,nx); 3D: (nz,ny,nx))."""
    lib = _load()
    a = np.ascontiguousarray(field, dtype=np.float64)
    nx, ny, nz, st = _dims(a)
    out = np.empty_like(a)
    rc = lib.oracle_jacobi(nx, ny, nz, st, int(iters), a.ctypes.data, out.ctypes.data, int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_jacobi failed: {rc}")
    return out


def jacobi_numpy(field: np.ndarray, iters: int) -> np.ndarray:
    """Numpy-slicing oracle, same definition and operation order as the C oracle."""
    a = np.array(field, dtype=np.float64, copy=True)
    squeeze = False
    if a.ndim == 2:
        a = a[None]
        squeeze = True
    b = a.copy()
    three_d = a.shape[0] > 1
    for _ in range(int(iters)):
        if three_d:
            s = a[1:-1, 1:-1, 2:] + a[1:-1, 1:-1, :-2]   # x+1, x-1
            s = s + a[1:-1, 2:, 1:-1]                     # y+1
            s = s + a[1:-1, :-2, 1:-1]                    # y-1
            s = s + a[2:, 1:-1, 1:-1]                     # z+1
            s = s + a[:-2, 1:-1, 1:-1]                    # z-1
            b[1:-1, 1:-1, 1:-1] = C6 * s
        else:
            s = a[:, 1:-1, 2:] + a[:, 1:-1, :-2]          # x+1, x-1
            s = s + a[:, 2:, 1:-1]                        # y+1
            s = s + a[:, :-2, 1:-1]                       # y-1
            b[:, 1:-1, 1:-1] = 0.25 * s
        a, b = b, a
    return a[0] if squeeze else a


def jacobi_converge(field: np.ndarray, max_iters: int, tol: float, every: int):
    """Run up to `max_iters` Jacobi iterations (C oracle), checking the update norm
    sqrt(sum((u_new - u_old)**2)) over interior cells after every `every`-th iteration (counting
    from the first iteration of this call) and stopping after the first check with norm <= tol.
    Returns (field, iterations_done, [norm of each check])."""
    a = np.ascontiguousarray(field, dtype=np.float64)
    a3 = a if a.ndim == 3 else a[None]
    sl = (slice(None), slice(1, -1), slice(1, -1)) if a3.shape[0] == 1 else (slice(1, -1),) * 3
    norms = []
    done = 0
    cur = a3
    while done < max_iters:
        step = min(every, max_iters - done) if every > 0 else max_iters - done
        if step > 1:
            cur = jacobi(cur, step - 1)
        nxt = jacobi(cur, 1)
        done += step
        if every > 0 and step == every:
            d = (nxt[sl] - cur[sl]).reshape(-1)
            r = float(np.sqrt(np.sum(d * d)))
            norms.append(r)
            cur = nxt
            if r <= tol:
                break
        else:
            cur = nxt
    out = cur if a.ndim == 3 else cur[0]
    return out, done, norms
