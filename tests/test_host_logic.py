"""CPU-only tests of the C-ABI library: it loads, exports every symbol include/jacobi.h
declares, and its host-only planning logic (slab decomposition P:350, TB split P:398-404,
HBM geometry) is correct.  No kernel is launched here."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import paper_conf_sc_baydamirlibu24_b200 as jb


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sc_baydamirlibu24_b200 import build as b
    b.build()


def test_library_exports_every_header_symbol():
    names = jb.header_functions()
    assert len(names) == len(jb._SIGS) == 32
    L = ctypes.CDLL(jb.LIB_PATH)
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing
    # and the binding mirrors every one of them
    for n in names:
        assert n in jb._SIGS, n


def test_nvshmem_variant_exports_everything():
    """libjacobi_b200_nvshmem.so (N3) exports the whole ABI plus the NVSHMEM entry points.
    (nm, not dlopen: it links libcuda, which a GPU-less box does not have.)"""
    from paper_conf_sc_baydamirlibu24_b200 import build as b
    if b.nvshmem_home() is None:
        pytest.skip("no NVSHMEM wheel")
    out = subprocess.run(["nm", "-D", "--defined-only", jb.NVSHMEM_LIB_PATH], capture_output=True, text=True).stdout
    syms = {line.split()[-1] for line in out.splitlines() if line.strip()}
    want = jb.header_functions() + jb.header_functions(nvshmem=True)
    assert len(jb.header_functions(nvshmem=True)) == 4
    assert not [n for n in want if n not in syms]


def test_library_is_sm100a_only():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", jb.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    for bad in ("sm_80", "sm_90", "sm_103"):
        assert bad not in out


def test_sass_uses_bulk_copy_and_no_fma():
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", jb.LIB_PATH],
                          capture_output=True, text=True).stdout
    assert "UBLKCP" in sass, "persistent kernel must stream planes with cp.async.bulk (TMA)"
    # fp64 fused multiply-add would break the oracle's operation order.  The only exception is
    # the residual-norm variant (jb_sweep<*, false, true, NORM=true>), whose one sqrt of the
    # all-reduced sum is the library's correctly rounded DFMA-based sqrt (not stencil arithmetic).
    funcs = sass.split("Function : ")[1:]
    assert len(funcs) >= 8
    for f in funcs:
        name = f.split("\n", 1)[0]
        if "jb_sweepILi2ELb0ELb1ELb1E" in name or "jb_sweepILi3ELb0ELb1ELb1E" in name:
            continue
        assert "DFMA" not in f, name


def test_strerror_and_version():
    assert jb.strerror(0) == "ok"
    assert "timeout" in jb.strerror(jb.JACOBI_ETIMEOUT)
    assert jb.jacobi_version() >= 100


@pytest.mark.parametrize("n_out", [3, 4, 5, 17, 258, 16384, 514])
@pytest.mark.parametrize("P", [1, 2, 3, 4, 7, 8])
def test_decompose(n_out, P):
    inner = n_out - 2
    q, r = divmod(inner, P)
    nxt = 1
    total = 0
    for g in range(P):
        s, c = jb.jacobi_decompose(n_out, P, g)
        assert s == nxt
        assert c == q + (1 if g < r else 0)
        nxt = s + c
        total += c
    assert total == inner and nxt == n_out - 1


def test_decompose_rejects():
    with pytest.raises(jb.JacobiError):
        jb.jacobi_decompose(2, 1, 0)
    with pytest.raises(jb.JacobiError):
        jb.jacobi_decompose(10, 2, 2)


@pytest.mark.parametrize("ctas", [4, 18, 37, 74, 148])
@pytest.mark.parametrize("chunk", [2, 3, 16, 64, 255, 2048])
@pytest.mark.parametrize("sides", [(0, 0), (1, 0), (0, 1), (1, 1)])
def test_tb_split(ctas, chunk, sides):
    top, bot = sides
    units = 16
    lo, hi = (2 if top else 1), (chunk - 1 if bot else chunk)
    inner = hi - lo + 1
    try:
        nt, nb, ni = jb.jacobi_tb_split(ctas, chunk, top, bot, units)
    except jb.JacobiError:
        assert ctas < top + bot + (inner > 0)
        return
    assert nt + nb + ni == ctas
    assert (nt > 0) == bool(top) and (nb > 0) == bool(bot)
    if top and bot:
        assert nt == nb
    assert nt <= units and nb <= units
    if inner > 0:
        assert ni >= 1
    if not top and not bot:
        assert ni == ctas
    # the reconstructed P:400 formula: boundary share grows as the slab thins
    if top and bot and inner > 0 and ctas >= 37:
        thin = jb.jacobi_tb_split(ctas, 4, 1, 1, units)[0]
        thick = jb.jacobi_tb_split(ctas, 2048, 1, 1, units)[0]
        assert thin >= thick


def test_tb_split_override():
    assert jb.jacobi_tb_split(148, 100, 1, 1, 16, 3) == (3, 3, 142)


@pytest.mark.parametrize("nx", [3, 4, 5, 6, 7, 130, 256, 511, 512, 1024, 16384])
def test_geometry_alignment(nx):
    for st, ny, nz in ((5, 9, 1), (7, 9, 5)):
        g = jb.jacobi_geometry(nx, ny, nz, st)
        pitch = g["pitch"]
        assert pitch % 4 == 0 and pitch >= nx + 3
        tx = g["tile_x"]
        assert tx & (tx - 1) == 0 and tx >= 8
        assert g["units_x"] == -(-(nx - 2) // tx)
        for ux in range(g["units_x"]):
            x0 = 1 + ux * tx
            assert (x0 + 3) % 2 == 0          # first output cell 16-byte aligned
            xs = 2 + ux * tx
            xe = min(xs + tx + 4, pitch)
            assert xs % 2 == 0 and (xe - xs) % 2 == 0  # bulk copy: 16 B aligned, multiple of 16 B
            assert xs <= x0 - 1 + 3 and min(x0 + tx, nx - 1) + 3 < xe  # covers x0-1 .. last+1
        if st == 5:
            assert g["plane_elems"] == pitch and g["stage_rows"] == 1
        else:
            assert g["plane_elems"] == ny * pitch and g["stage_rows"] == g["tile_y"] + 2


def test_geometry_rejects():
    with pytest.raises(jb.JacobiError):
        jb.jacobi_geometry(2, 9, 1, 5)
    with pytest.raises(jb.JacobiError):
        jb.jacobi_geometry(9, 9, 3, 5)
    with pytest.raises(jb.JacobiError):
        jb.jacobi_geometry(9, 9, 1, 7)


def test_create_without_gpu_is_loud():
    """On a box without a CUDA device the product path must fail, never fall back."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(jb.JacobiError) as e:
        jb.Jacobi((10, 10))
    assert e.value.code == jb.JACOBI_ENODEV


def test_binding_rejects_bad_arrays():
    with pytest.raises(ValueError):
        jb._host_ptr(np.zeros(10, dtype=np.float32), 10, False)
    with pytest.raises(ValueError):
        jb._host_ptr(np.zeros(9), 10, False)


def test_product_package_does_not_import_oracle():
    pkg = os.path.dirname(jb.__file__)
    for root, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                src = open(os.path.join(root, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "jacobi_oracle" not in src, f


def test_slab_bytes_matches_layout():
    g = jb.jacobi_geometry(1000, 64, 1, 5)
    total = 0
    for slab in range(3):
        s, c = jb.jacobi_decompose(64, 3, slab)
        b = jb.jacobi_slab_bytes(1000, 64, 1, 5, 3, slab)
        # (chunk + 2) planes + the time-blocked kernel's edge-zone scratch: per side K-1 slots for
        # the neighbour's intermediate levels + 2K-m own level-m planes (m < K), for 2D K <= 5: 34
        kmax = 5
        scratch = (kmax - 1) + sum(2 * kmax - m for m in range(1, kmax))
        assert scratch == 34
        # + 8 doubles of read slack (JB_BUF_SLACK: vectorised edge-zone pair loads at the last column)
        assert b == ((c + 2 + scratch) * g["plane_elems"] + 8) * 8
        total += c
    assert total == 62
    # 3D: K <= 3: 2 slots + 5 level-1 + 4 level-2 planes
    g3 = jb.jacobi_geometry(40, 30, 64, 7)
    s, c = jb.jacobi_decompose(64, 3, 1)
    assert jb.jacobi_slab_bytes(40, 30, 64, 7, 3, 1) == ((c + 2 + 11) * g3["plane_elems"] + 8) * 8


def test_set_allocator_rejects_half():
    cb = jb.ALLOC_FN(lambda n, d, u: None)
    with pytest.raises(jb.JacobiError):
        jb.jacobi_set_allocator(cb, None)
    jb.jacobi_set_allocator(None, None)


def test_halo_spans_summary():
    """jb.halo_spans (host-side summary of a jacobi_halo_trace array): medians of wait, put
    (flag -> signal) and span per exchange over both sides, the signal period, and unrecorded
    (zero) entries ignored — checked on a synthetic trace with known spans."""
    n = 10
    tr = np.zeros((2, n, 3), dtype=np.uint64)
    for e in range(n):
        t0 = 1_000_000 + e * 5_000           # exchanges 5 us apart
        tr[0, e] = (t0, t0 + 1_000, t0 + 3_000)  # top: wait 1 us, put 2 us
    # bottom side never had a neighbour: all zero
    sp = jb.halo_spans(tr, skip=2)
    assert sp["wait_us"] == 1.0 and sp["put_us"] == 2.0 and sp["span_us"] == 3.0
    assert sp["period_us"] == 5.0 and sp["exchanges"] == n - 2
    assert jb.halo_spans(np.zeros((2, 4, 3), dtype=np.uint64))["span_us"] is None


# ---------------------------------------------------------------- auto policies
@pytest.mark.parametrize("shape,stencil,P,virtual,dyn,tb", [
    # measured choices of profiles/r02_sched_sweep_*.jsonl
    ((128, 128, 128), 7, 1, False, False, True),    # C5a: static schedule; one slab: time-blocked
    ((128, 128, 128), 7, 2, True, False, False),    # 2 virtual slabs: per-iteration, static
    ((256, 256, 256), 7, 2, True, False, False),    # 111 K cells per CTA: per-iteration
    ((384, 384, 384), 7, 2, True, True, True),      # 380 K: time-blocked
    ((384, 384, 384), 7, 4, True, True, False),     # 37 CTAs per slab < 64
    ((512, 512, 512), 7, 2, True, True, True),      # C3 with 2 virtual slabs
    ((512, 512, 512), 7, 8, True, True, False),     # 18 CTAs per slab
    ((512, 512, 512), 7, 2, False, True, True),     # C3 on 2 GPUs: 227 K per CTA
    ((512, 512, 512), 7, 8, False, False, False),   # C3 on 8 GPUs: 56 K per CTA
    ((1, 2048, 2048), 5, 2, True, False, False),    # 28 K: per-iteration
    ((1, 4096, 4096), 5, 2, True, False, True),     # 113 K: time-blocked, static interior (unused)
    ((1, 16384, 16384), 5, 8, False, True, True),   # C2 on 8 GPUs: 227 K per CTA
    ((1, 16384, 16384), 5, 8, True, True, True),    # C2 with 8 virtual slabs
])
def test_auto_policy_thresholds(shape, stencil, P, virtual, dyn, tb):
    nz, ny, nx = shape
    pol = jb.jacobi_auto_policy(nx, ny, nz, stencil, P, virtual)
    cells = (nx - 2) * (ny - 2) * (nz - 2 if stencil == 7 else 1)
    assert pol["cells_per_cta"] == cells // (148 if virtual else 148 * P)
    assert pol["dynamic_schedule"] == dyn, pol
    assert pol["tblock"] == tb, pol
    assert pol["min_slab_ctas"] == (148 // P if virtual else 148)


def test_auto_policy_rejects():
    for args in [(2, 9, 1, 5, 1, 0, 148), (9, 9, 3, 5, 1, 0, 148), (9, 9, 1, 5, 0, 0, 148), (9, 9, 1, 5, 1, 0, 0)]:
        with pytest.raises(jb.JacobiError):
            jb.jacobi_auto_policy(*args)
