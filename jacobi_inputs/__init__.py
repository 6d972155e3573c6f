"""Seeded synthetic input generators shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no stencil, no Jacobi update): it only
produces initial fields.  Both the oracle side (tests/, oracle/) and the CUDA side use the
same counter-based generator; the CUDA library implements U12 independently on the device
(``jacobi_create`` initialises the field with it), and a GPU test checks that the two
produce identical bits.

Grid convention (SURVEY.md §8 "Notation"): a global field is a C-contiguous numpy array of
shape ``(nz, ny, nx)`` (``nz == 1`` for 2D), x fastest, so the flat index is
``idx = (z*ny + y)*nx + x``.  Extents INCLUDE the one-cell Dirichlet layer on every face
(reading R7).

Generators
----------
``u12(shape, seed)``
    Every cell, boundary included, is ``1 + (splitmix64(seed + (idx+1)*GOLDEN) >> 12) * 2**-52``,
    i.e. the IEEE-754 double whose bit pattern is ``0x3FF0000000000000 | (z >> 12)``.
    Values are exact dyadics in [1, 2): no rounding anywhere, so two independent
    implementations agree bit for bit, and (maximum principle) the iterates never become
    subnormal.  The paper gives no value distribution (§6.1.1, P:524 only fixes
    domain sizes), so this is the recipe stated in DESIGN.md §3.
``nv_field(shape)``
    Zero interior, x-faces ``sin(2*pi*y/(ny-1))`` — the shape of the NVIDIA samples the
    paper's baselines come from; used only for subnormal-exposure tests.
``integer_field(shape, seed, lo, hi)``
    Uniform integers (as doubles) for exact-arithmetic tests.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
SEED_BENCH = 0x5C24
SEEDS_TEST = (1, 2, 3)

__all__ = ["splitmix64", "u12", "u12_flat", "nv_field", "integer_field", "SEED_BENCH", "SEEDS_TEST"]


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (mod 2**64 arithmetic)."""
    z = np.asarray(x, dtype=np.uint64).copy()
    with np.errstate(over="ignore"):
        z ^= z >> np.uint64(30)
        z *= np.uint64(0xBF58476D1CE4E5B9)
        z ^= z >> np.uint64(27)
        z *= np.uint64(0x94D049BB133111EB)
        z ^= z >> np.uint64(31)
    return z


def u12_flat(start: int, count: int, seed: int = SEED_BENCH) -> np.ndarray:
    """U12 values for flat indices [start, start+count) as float64."""
    idx = np.arange(start, start + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = np.uint64(seed) + (idx + np.uint64(1)) * GOLDEN
    bits = np.uint64(0x3FF0000000000000) | (splitmix64(x) >> np.uint64(12))
    return bits.view(np.float64)


def u12(shape, seed: int = SEED_BENCH) -> np.ndarray:
    """U12 field of the given (nz, ny, nx) or (ny, nx) shape."""
    shape = tuple(int(s) for s in shape)
    n = int(np.prod(shape))
    return u12_flat(0, n, seed).reshape(shape)


def nv_field(shape) -> np.ndarray:
    """Zero interior; x = 0 and x = nx-1 faces = sin(2*pi*y/(ny-1)); other faces 0."""
    shape = tuple(int(s) for s in shape)
    a = np.zeros(shape, dtype=np.float64)
    ny = shape[-2]
    prof = np.sin(2.0 * np.pi * np.arange(ny) / (ny - 1))
    a[..., :, 0] = prof
    a[..., :, -1] = prof
    return a


def integer_field(shape, seed: int, lo: int = -1000, hi: int = 1000) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.integers(lo, hi, size=tuple(shape)).astype(np.float64)
