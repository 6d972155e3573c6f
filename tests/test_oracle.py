"""Pins for the CPU oracle (oracle/) — all CPU-only ("not gpu").

The oracle follows PAPER.md P:195-197 (§2.1, Jacobi for Laplace, Dirichlet on ∂Ω)
(fixed iteration count), P:394 (previous-time-step semantics), P:346/P:535 (2D5pt/3D7pt).
Nothing here retypes the oracle's update formula as the expected value: each pin is fixed by
mathematics (eigenmode closed form, maximum principle, stationary harmonic fields, exact
rational arithmetic) or by an independent library construction (scipy.sparse discrete
Laplacian, scipy.sparse.linalg.spsolve).  Cross-checks between the two oracle
implementations and a hand loop are included as well, but they are not counted as pins.
"""
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.linalg as spla

from jacobi_inputs import integer_field, nv_field, u12


def both(oracle_mod, field, iters):
    a = oracle_mod.jacobi(field, iters)
    b = oracle_mod.jacobi_numpy(field, iters)
    assert np.array_equal(a.view(np.uint64), b.view(np.uint64)), "C and numpy oracles differ"
    return a


# ---------------------------------------------------------------- library / textbook pins

def laplacian_system(field):
    """Textbook discrete Laplace system A u = b on the interior (A = -Δ_h, 5/7-point),
    assembled with scipy.sparse Kronecker products; b carries the Dirichlet data."""
    f = field if field.ndim == 3 else field[None]
    nz, ny, nx = f.shape
    dims = [nx - 2, ny - 2] + ([nz - 2] if nz > 1 else [])

    def t1(n):
        return sp.diags([-np.ones(n - 1), 2 * np.ones(n), -np.ones(n - 1)], [-1, 0, 1], format="csr")

    eye = [sp.identity(n, format="csr") for n in dims]
    A = None
    for d in range(len(dims)):  # flat order: x fastest -> kron(..., I_y, T_x) etc.
        mats = [t1(dims[k]) if k == d else eye[k] for k in range(len(dims))]
        term = mats[-1]
        for m in reversed(mats[:-1]):
            term = sp.kron(term, m, format="csr")
        A = term if A is None else A + term
    # b: sum of Dirichlet neighbour values for cells adjacent to the boundary
    g = f.copy()
    g3 = g if nz > 1 else g
    inner = np.zeros_like(g3)
    if nz > 1:
        inner[1:-1, 1:-1, 1:-1] = 1
    else:
        inner[:, 1:-1, 1:-1] = 1
    bnd = np.where(inner == 1, 0.0, g3)
    if nz > 1:
        b = (bnd[1:-1, 1:-1, 2:] + bnd[1:-1, 1:-1, :-2] + bnd[1:-1, 2:, 1:-1] + bnd[1:-1, :-2, 1:-1]
             + bnd[2:, 1:-1, 1:-1] + bnd[:-2, 1:-1, 1:-1])
    else:
        b = bnd[:, 1:-1, 2:] + bnd[:, 1:-1, :-2] + bnd[:, 2:, 1:-1] + bnd[:, :-2, 1:-1]
    return A.tocsr(), b.reshape(-1), len(dims)


def interior(field):
    f = field if field.ndim == 3 else field[None]
    if f.shape[0] > 1:
        return f[1:-1, 1:-1, 1:-1].reshape(-1)
    return f[:, 1:-1, 1:-1].reshape(-1)


@pytest.mark.parametrize("shape", [(9, 12), (7, 8, 6), (1, 5, 17)])
def test_one_step_is_textbook_jacobi_splitting(oracle_mod, shape):
    """One sweep == Jacobi splitting u' = D^{-1}(b - (A - D) u) of the scipy-assembled system."""
    f = u12(shape, seed=1)
    A, b, nd = laplacian_system(f)
    D = 2.0 * nd
    u = interior(f)
    expect = (b - (A @ u - D * u)) / D
    got = interior(both(oracle_mod, f, 1))
    np.testing.assert_allclose(got, expect, rtol=0, atol=4e-16 * np.abs(expect).max())


@pytest.mark.parametrize("shape,iters", [((8, 7), 4000), ((6, 5, 7), 3000)])
def test_converges_to_sparse_direct_solve(oracle_mod, shape, iters):
    """Jacobi for Laplace converges to the discrete harmonic function with the same Dirichlet data
    (P:195-197); scipy's spsolve of the textbook system is the independent fixed point."""
    f = u12(shape, seed=2)
    A, b, _ = laplacian_system(f)
    sol = spla.spsolve(A.tocsc(), b)
    got = interior(both(oracle_mod, f, iters))
    np.testing.assert_allclose(got, sol, rtol=0, atol=1e-12)


@pytest.mark.parametrize("dims,modes,iters", [((66, 50), (3, 2), 1000), ((24, 22, 20), (2, 1, 3), 300),
                                              ((17, 40), (1, 5), 200)])
def test_eigenmode_closed_form(oracle_mod, dims, modes, iters):
    """u0 = prod_d sin(pi m_d i_d/(n_d-1)) with zero boundary decays as lambda^k u0,
    lambda = mean_d cos(pi m_d/(n_d-1)).  Pins the weights, the neighbour set and the axes."""
    if len(dims) == 2:
        ny, nx = dims
        my, mx = modes
        y = np.arange(ny)[:, None]
        x = np.arange(nx)[None, :]
        u0 = np.sin(np.pi * my * y / (ny - 1)) * np.sin(np.pi * mx * x / (nx - 1))
        u0[0, :] = u0[-1, :] = 0.0
        u0[:, 0] = u0[:, -1] = 0.0
        lam = (np.cos(np.pi * mx / (nx - 1)) + np.cos(np.pi * my / (ny - 1))) / 2
    else:
        nz, ny, nx = dims
        mz, my, mx = modes
        z = np.arange(nz)[:, None, None]
        y = np.arange(ny)[None, :, None]
        x = np.arange(nx)[None, None, :]
        u0 = (np.sin(np.pi * mz * z / (nz - 1)) * np.sin(np.pi * my * y / (ny - 1))
              * np.sin(np.pi * mx * x / (nx - 1)))
        for ax in range(3):
            idx = [slice(None)] * 3
            idx[ax] = 0
            u0[tuple(idx)] = 0
            idx[ax] = -1
            u0[tuple(idx)] = 0
        lam = (np.cos(np.pi * mx / (nx - 1)) + np.cos(np.pi * my / (ny - 1))
               + np.cos(np.pi * mz / (nz - 1))) / 3
    got = both(oracle_mod, u0, iters)
    np.testing.assert_allclose(got, lam ** iters * u0, rtol=0, atol=1e-14)


# ---------------------------------------------------------------- exact arithmetic pins

def exact_jacobi(field, iters, weight):
    """Exact rational Jacobi (Fraction) — the mathematical value without rounding."""
    f = field if field.ndim == 3 else field[None]
    nz, ny, nx = f.shape
    a = [[[Fraction(float(v)) for v in row] for row in pl] for pl in f]
    for _ in range(iters):
        b = [[row[:] for row in pl] for pl in a]
        zr = range(1, nz - 1) if nz > 1 else range(0, 1)
        for z in zr:
            for yy in range(1, ny - 1):
                for xx in range(1, nx - 1):
                    s = a[z][yy][xx + 1] + a[z][yy][xx - 1] + a[z][yy + 1][xx] + a[z][yy - 1][xx]
                    if nz > 1:
                        s += a[z + 1][yy][xx] + a[z - 1][yy][xx]
                    b[z][yy][xx] = s * weight
        a = b
    return a


def test_2d_exact_rational(oracle_mod):
    """Integer inputs in [-1000,1000): after k <= 20 sweeps every iterate is a dyadic with
    <= 10+2k significant bits, so IEEE fp64 must reproduce the exact rational value bit for bit."""
    f = integer_field((7, 9), seed=3)
    for iters in (1, 2, 7, 20):
        ex = exact_jacobi(f, iters, Fraction(1, 4))
        got = both(oracle_mod, f, iters)
        exp = np.array([[float(v) for v in row] for row in ex[0]])
        assert np.array_equal(got, exp)


def test_3d_within_rounding_of_exact(oracle_mod):
    """3D weight 1/6 is inexact in binary; the fp64 result must stay within a few ulps·k of
    the exact rational Jacobi value (error bound: 6 roundings + weight error per sweep)."""
    f = integer_field((5, 6, 7), seed=4).astype(np.float64) / 64.0
    iters = 6
    ex = exact_jacobi(f, iters, Fraction(1, 6))
    exp = np.array([[[float(v) for v in row] for row in pl] for pl in ex])
    got = both(oracle_mod, f, iters)
    scale = np.abs(f).max()
    assert np.max(np.abs(got - exp)) <= iters * 8 * np.finfo(np.float64).eps * scale


# ---------------------------------------------------------------- invariants

def test_constant_fields_stationary_2d(oracle_mod):
    rng = np.random.default_rng(11)
    consts = np.concatenate([rng.standard_normal(50) * 10.0 ** rng.integers(-300, 300, 50),
                             [0.0, -0.0, 1.0, np.pi, 5e-324, 1e300]])
    for c in consts:
        f = np.full((6, 7), c)
        assert np.array_equal(both(oracle_mod, f, 3), f)


def test_integer_constants_stationary_3d(oracle_mod):
    for c in (0.0, 1.0, -3.0, 12345.0, 2.0 ** 40):
        f = np.full((5, 6, 7), c)
        assert np.array_equal(both(oracle_mod, f, 5), f)


def _grid2(ny, nx):
    y, x = np.mgrid[0:ny, 0:nx].astype(np.float64)
    return x, y


def _grid3(nz, ny, nx):
    z, y, x = np.mgrid[0:nz, 0:ny, 0:nx].astype(np.float64)
    return x, y, z


@pytest.mark.parametrize("name", ["lin", "x2-y2", "xy"])
def test_harmonic_fields_stationary_2d(oracle_mod, name):
    x, y = _grid2(10, 12)
    f = {"lin": 3 + 2 * x - 5 * y, "x2-y2": x * x - y * y, "xy": x * y}[name]
    assert np.array_equal(both(oracle_mod, f, 1000), f)


@pytest.mark.parametrize("name", ["lin", "x2+y2-2z2", "xy+yz+zx"])
def test_harmonic_fields_stationary_3d(oracle_mod, name):
    x, y, z = _grid3(8, 9, 10)
    f = {"lin": 1 + x + 2 * y - 3 * z, "x2+y2-2z2": x * x + y * y - 2 * z * z,
         "xy+yz+zx": x * y + y * z + z * x}[name]
    assert np.array_equal(both(oracle_mod, f, 300), f)


def test_non_harmonic_field_moves(oracle_mod):
    """Guard against a no-op oracle: x^2 (Laplacian 2) must change."""
    x, _ = _grid2(8, 9)
    f = x * x
    assert not np.array_equal(both(oracle_mod, f, 1), f)


@pytest.mark.parametrize("shape", [(13, 17), (9, 10, 11)])
@pytest.mark.parametrize("iters", [1, 2, 5])
def test_boundary_untouched(oracle_mod, shape, iters):
    f = u12(shape, seed=1)
    g = both(oracle_mod, f, iters)
    if len(shape) == 2:
        m = np.ones(shape, bool)
        m[1:-1, 1:-1] = False
    else:
        m = np.ones(shape, bool)
        m[1:-1, 1:-1, 1:-1] = False
    assert np.array_equal(g[m], f[m])
    assert not np.array_equal(g[~m], f[~m])


@pytest.mark.parametrize("shape", [(20, 23), (9, 10, 11)])
def test_maximum_principle(oracle_mod, shape):
    f = u12(shape, seed=3)
    g = both(oracle_mod, f, 50)
    ulp = np.spacing(f.max())
    tol = 0.0 if len(shape) == 2 else ulp
    assert g.min() >= f.min() - tol and g.max() <= f.max() + tol


@pytest.mark.parametrize("shape", [(11, 16), (7, 8, 9)])
def test_x_mirror_symmetry(oracle_mod, shape):
    f = u12(shape, seed=2)
    f = f + f[..., ::-1]
    g = both(oracle_mod, f, 37)
    assert np.array_equal(g, g[..., ::-1])


def test_run_splitting_and_zero_iters(oracle_mod):
    f = u12((9, 10, 11), seed=1)
    assert np.array_equal(oracle_mod.jacobi(f, 0), f)
    a = oracle_mod.jacobi(oracle_mod.jacobi(f, 3), 4)
    assert np.array_equal(a, oracle_mod.jacobi(f, 7))


# ---------------------------------------------------------------- cross-checks (not pins)

def brute_force(field, iters):
    f = field if field.ndim == 3 else field[None]
    nz, ny, nx = f.shape
    a = f.tolist()
    c6 = float.fromhex("0x1.5555555555555p-3")
    for _ in range(iters):
        b = [[row[:] for row in pl] for pl in a]
        for z in (range(1, nz - 1) if nz > 1 else [0]):
            for y in range(1, ny - 1):
                for x in range(1, nx - 1):
                    s = a[z][y][x + 1] + a[z][y][x - 1]
                    s = s + a[z][y + 1][x]
                    s = s + a[z][y - 1][x]
                    if nz > 1:
                        s = s + a[z + 1][y][x]
                        s = s + a[z - 1][y][x]
                        b[z][y][x] = c6 * s
                    else:
                        b[z][y][x] = 0.25 * s
        a = b
    out = np.array(a)
    return out if field.ndim == 3 else out[0]


@pytest.mark.parametrize("shape", [(3, 3), (5, 6), (3, 3, 3), (4, 5, 6), (1, 4, 9)])
@pytest.mark.parametrize("iters", [0, 1, 4, 7])
def test_brute_force_bitwise(oracle_mod, shape, iters):
    f = u12(shape, seed=2)
    assert np.array_equal(both(oracle_mod, f, iters), brute_force(f, iters))


@pytest.mark.parametrize("nthreads", [2, 4, 8])
def test_thread_count_bitwise(oracle_mod, nthreads):
    f = u12((13, 40, 33), seed=3)
    assert np.array_equal(oracle_mod.jacobi(f, 9, nthreads), oracle_mod.jacobi(f, 9, 1))


def test_subnormals_kept(oracle_mod):
    """NV-shaped init on a wide grid produces subnormals; no FTZ/DAZ on either oracle."""
    f = nv_field((34, 2400))
    g = both(oracle_mod, f, 1000)
    sub = np.count_nonzero((g != 0) & (np.abs(g) < np.finfo(np.float64).tiny))
    assert sub > 0


def test_decomposition_invariance_model(oracle_mod):
    """a slab decomposition with halo copies equals the global sweep bit for bit.
    Model: chunks of q or q+1 outer planes (first r slabs get +1), 1 halo plane each side."""
    for shape in [(3 * 5 + 2, 9), (11, 7, 8)]:
        f = u12(shape, seed=3)
        ref = oracle_mod.jacobi(f, 6)
        n_out = shape[0]
        for P in range(1, 6):
            q, r = divmod(n_out - 2, P)
            if q < 1:
                continue
            starts = [1 + g * q + min(g, r) for g in range(P)]
            chunks = [q + (g < r) for g in range(P)]
            slabs = [f[s - 1:s + c + 1].copy() for s, c in zip(starts, chunks)]
            for _ in range(6):
                new = [oracle_mod.jacobi(s, 1) for s in slabs]
                for g in range(P):  # halo exchange
                    if g > 0:
                        new[g][0] = new[g - 1][-2]
                    if g < P - 1:
                        new[g][-1] = new[g + 1][1]
                slabs = new
            out = f.copy()
            for s, c, sl in zip(starts, chunks, slabs):
                out[s:s + c] = sl[1:-1]
            assert np.array_equal(out, ref), (shape, P)


def test_oracle_rejects_bad_args(oracle_mod):
    with pytest.raises(ValueError):
        oracle_mod.jacobi(np.zeros((2, 5)), 1)
    with pytest.raises(ValueError):
        oracle_mod.jacobi(np.zeros((5, 2)), 1)


# ---------------------------------------------------------------- N4: update norm (oracle side)
def test_update_norm_eigenmode_closed_form(oracle_mod):
    """For an eigenmode u_k = lam^k u0 the update norm after iteration k (1-based) is
    lam^(k-1) |lam - 1| ||u0||_2, and the run stops at the first check below tol."""
    ny, nx, my, mx = 34, 50, 2, 3
    y = np.arange(ny)[:, None]
    x = np.arange(nx)[None, :]
    u0 = np.sin(np.pi * my * y / (ny - 1)) * np.sin(np.pi * mx * x / (nx - 1))
    u0[0, :] = u0[-1, :] = 0.0
    u0[:, 0] = u0[:, -1] = 0.0
    lam = (np.cos(np.pi * mx / (nx - 1)) + np.cos(np.pi * my / (ny - 1))) / 2
    n0 = np.sqrt(np.sum(u0[1:-1, 1:-1] ** 2))
    every = 7
    tol = 0.05 * n0 * abs(lam - 1)
    out, done, norms = oracle_mod.jacobi_converge(u0, 5000, tol, every)
    exp = [lam ** (every * (i + 1) - 1) * abs(lam - 1) * n0 for i in range(len(norms))]
    np.testing.assert_allclose(norms, exp, rtol=1e-9)
    k_stop = next(k for k in range(every, 5000, every) if lam ** (k - 1) * abs(lam - 1) * n0 <= tol)
    assert done == k_stop
    np.testing.assert_allclose(out, lam ** done * u0, rtol=0, atol=1e-13)


def test_update_norm_zero_for_harmonic_field(oracle_mod):
    y, x = np.mgrid[0:12, 0:15].astype(np.float64)
    f = x * x - y * y
    out, done, norms = oracle_mod.jacobi_converge(f, 100, 0.0, 5)
    assert done == 5 and norms == [0.0] and np.array_equal(out, f)


def test_golden_digests(oracle_mod):
    """Regression pin: the oracle still reproduces the committed digests (tests/golden)."""
    import json
    import os
    import sys
    here = os.path.join(os.path.dirname(__file__), "golden")
    sys.path.insert(0, here)
    import make_golden
    gold = {}
    for fn in ("oracle_digests.json", "oracle_digests_latency.json"):  # (the C2 / C3 full set: too slow here)
        with open(os.path.join(here, fn)) as f:
            gold.update(json.load(f))
    for name, g in gold.items():
        r = make_golden.compute(tuple(g["shape"]), g["iters"])
        assert make_golden.digest(r) == g["sha256"], name
