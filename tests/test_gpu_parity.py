"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Bar (BASELINE.json north_star): bit-exact fp64 — the kernel uses the oracle's
operation order with contraction disabled — and the P-slab result bit-identical to P = 1.
Shapes span several tiles with ragged tails in x, y and the outer axis; slab counts include
remainders and the minimum chunk of 2 planes; modes cover CPU-Free, the memcpy baseline and
NCCL (P = 1), and the no-compute / watchdog paths.
"""
import numpy as np
import pytest

import oracle
import paper_conf_sc_baydamirlibu24_b200 as jb
from jacobi_inputs import SEED_BENCH, integer_field, nv_field, u12

pytestmark = pytest.mark.gpu
ROOT_DIR = __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__)))


def bits_equal(a, b):
    return np.array_equal(np.asarray(a).view(np.uint64), np.asarray(b).view(np.uint64))


def assert_bitwise(got, exp, what=""):
    if not bits_equal(got, exp):
        d = np.abs(got - exp)
        idx = np.unravel_index(np.argmax(d), d.shape)
        n = np.count_nonzero(got.view(np.uint64) != exp.view(np.uint64))
        raise AssertionError(f"{what}: {n} cells differ, max |diff| {d.max()} at {idx}")


def run_gpu(field, iters, virtual=0, mode=jb.MODE_CPUFREE, params=None, flags=0):
    """Run through the C ABI.  Unless `params` says otherwise the per-iteration streaming kernel
    is forced (resident=0, tblock=0), so these shapes exercise it; the resident and the
    temporally blocked kernels have their own tests (below, test_gpu_tblock.py)."""
    params = {"resident": 0, "tblock": 0, **(params or {})}
    with jb.Jacobi(field.shape, virtual=virtual) as j:
        for k, v in params.items():
            j.set_param(k, v)
        j.set_mode(mode, flags)
        j.scatter(field)
        j.run(iters)
        return j.gather()


# ---------------------------------------------------------------- 1 GPU
def test_device_init_is_u12():
    for shape in [(256, 256), (9, 37, 41)]:
        with jb.Jacobi(shape) as j:
            assert_bitwise(j.gather(), u12(shape, SEED_BENCH), "device U12 init")


def test_c1_256sq_1000_iters_vs_oracle():
    """BASELINE config C1: 2D 256x256, 1000 iterations, 1 GPU vs CPU oracle."""
    f = u12((256, 256), SEED_BENCH)
    with jb.Jacobi((256, 256)) as j:  # create initialises U12 on the device
        j.run(1000)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, 1000, 8), "C1")


@pytest.mark.parametrize("shape", [(3, 3), (4, 5), (37, 1500), (70, 2051), (300, 130)])
@pytest.mark.parametrize("iters", [1, 2, 7])
def test_2d_shapes(shape, iters):
    f = u12(shape, 1)
    exp = oracle.jacobi(f, iters)
    assert_bitwise(run_gpu(f, iters), exp, f"2D {shape}")
    assert_bitwise(run_gpu(f, iters, params={"tile_x": 64}), exp, f"2D {shape} tx64")


@pytest.mark.parametrize("shape", [(3, 3, 3), (5, 4, 9), (13, 30, 70), (20, 61, 130), (9, 17, 600)])
@pytest.mark.parametrize("iters", [1, 4])
def test_3d_shapes(shape, iters):
    f = u12(shape, 2)
    exp = oracle.jacobi(f, iters)
    assert_bitwise(run_gpu(f, iters), exp, f"3D {shape}")
    assert_bitwise(run_gpu(f, iters, params={"tile_y": 3, "tile_x": 16}), exp, f"3D {shape} ty3")


@pytest.mark.parametrize("sched", [0, 1, 2])
@pytest.mark.parametrize("stages", [4, 7])
def test_schedules_and_ring_depths(sched, stages):
    for shape in [(130, 333), (11, 40, 50)]:
        f = u12(shape, 3)
        exp = oracle.jacobi(f, 5)
        got = run_gpu(f, 5, params={"schedule": sched, "stages": stages, "ctas": 5})
        assert_bitwise(got, exp, f"{shape} sched={sched} stages={stages}")


# ---------------------------------------------------------------- virtual slabs (multi-GPU protocol)
@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
def test_virtual_2d(P):
    shape = (2 * P + 2 + 3, 777)  # chunk 2 for some slabs, remainder 3
    f = u12(shape, 1)
    for iters in (1, 6, 33):
        assert_bitwise(run_gpu(f, iters, virtual=P), oracle.jacobi(f, iters), f"virtual P={P} it={iters}")


@pytest.mark.parametrize("P", [2, 3, 8])
def test_virtual_3d(P):
    shape = (3 * P + 2 + 1, 21, 45)
    f = u12(shape, 2)
    for iters in (1, 9):
        assert_bitwise(run_gpu(f, iters, virtual=P), oracle.jacobi(f, iters), f"virtual3d P={P}")


def test_virtual_many_boundary_ctas():
    f = u12((40, 4100), 3)
    exp = oracle.jacobi(f, 11)
    for bc in (1, 2, 4):
        got = run_gpu(f, 11, virtual=4, params={"boundary_ctas": bc, "tile_x": 128})
        assert_bitwise(got, exp, f"boundary_ctas={bc}")


@pytest.mark.parametrize("min_block,help_", [(1, 1), (3, 0), (64, 1)])
def test_dynamic_schedule_knobs(min_block, help_):
    for shape, P in [((70, 1030), 3), ((23, 40, 130), 2), ((300, 77), 1)]:
        f = u12(shape, 4)
        exp = oracle.jacobi(f, 7)
        got = run_gpu(f, 7, virtual=P, params={"schedule": 2, "min_block": min_block, "dyn_help": help_})
        assert_bitwise(got, exp, f"{shape} P={P} min_block={min_block} help={help_}")


def test_virtual_c5_latency_shapes_long():
    """C5 shapes (3D 128^3, 2D 1024^2) at P = 8 slabs, 100 iterations, vs P = 1 and the oracle."""
    for shape in [(128, 128, 128), (1024, 1024)]:
        f = u12(shape, SEED_BENCH)
        exp = oracle.jacobi(f, 100, 8)
        assert_bitwise(run_gpu(f, 100, virtual=8), exp, f"C5 {shape} P=8")
        assert_bitwise(run_gpu(f, 100), exp, f"C5 {shape} P=1")


# ---------------------------------------------------------------- baselines
@pytest.mark.parametrize("P", [1, 2, 4])
def test_baseline_memcpy_virtual(P):
    f = u12((4 * P + 5, 300), 1)
    exp = oracle.jacobi(f, 13)
    assert_bitwise(run_gpu(f, 13, virtual=P, mode=jb.MODE_BASELINE_MEMCPY), exp, f"memcpy P={P}")
    g = u12((3 * P + 3, 12, 33), 2)
    assert_bitwise(run_gpu(g, 5, virtual=P, mode=jb.MODE_BASELINE_MEMCPY), oracle.jacobi(g, 5), "memcpy 3d")


@pytest.mark.parametrize("mode", ["MODE_BASELINE_OVERLAP", "MODE_BASELINE_P2P", "MODE_BASELINE_GRAPH"])
@pytest.mark.parametrize("P", [1, 2, 4])
def test_baselines_n1(mode, P):
    """SURVEY §8(f) N1 baselines (Copy-Overlap, P2P, CUDA graph) are bit-identical too."""
    m = getattr(jb, mode)
    f = u12((4 * P + 7, 520), 1)
    assert_bitwise(run_gpu(f, 11, virtual=P, mode=m), oracle.jacobi(f, 11), f"{mode} P={P}")
    g = u12((3 * P + 4, 13, 70), 2)
    assert_bitwise(run_gpu(g, 6, virtual=P, mode=m), oracle.jacobi(g, 6), f"{mode} 3d P={P}")


def test_graph_baseline_cache_and_mixing():
    f = u12((30, 200), 3)
    with jb.Jacobi(f.shape, virtual=3) as j:
        j.scatter(f)
        j.set_mode(jb.MODE_BASELINE_GRAPH)
        j.run(4).run(4).run(5)           # cached graph reused for equal (iters, parity)
        j.set_mode(jb.MODE_CPUFREE).run(3)
        j.set_mode(jb.MODE_BASELINE_P2P).run(2)
        j.set_mode(jb.MODE_BASELINE_OVERLAP).run(2)
        assert_bitwise(j.gather(), oracle.jacobi(f, 20), "graph cache + mixing")


def test_baseline_nccl_single_gpu():
    f = u12((65, 300), 1)
    assert_bitwise(run_gpu(f, 9, mode=jb.MODE_BASELINE_NCCL), oracle.jacobi(f, 9), "nccl P=1")


def test_mode_switching_and_run_splitting():
    f = u12((50, 310), 2)
    exp = oracle.jacobi(f, 20)
    with jb.Jacobi(f.shape, virtual=3) as j:
        j.scatter(f)
        j.run(3)
        j.set_mode(jb.MODE_BASELINE_MEMCPY).run(4)
        j.set_mode(jb.MODE_CPUFREE).run(0).run(5)
        j.set_mode(jb.MODE_BASELINE_MEMCPY).run(1)
        j.set_mode(jb.MODE_CPUFREE).run(7)
        assert j.iterations == 20
        assert_bitwise(j.gather(), exp, "mixed modes")


# ---------------------------------------------------------------- invariants through the C ABI
def test_harmonic_and_constant_fields_stationary():
    y, x = np.mgrid[0:40, 0:70].astype(np.float64)
    for f in (3 + 2 * x - 5 * y, x * x - y * y, x * y, np.full((40, 70), np.pi)):
        assert_bitwise(run_gpu(f, 101, virtual=3), f, "2D stationary")
    z, y, x = np.mgrid[0:12, 0:13, 0:30].astype(np.float64)
    for f in (1 + x + 2 * y - 3 * z, x * x + y * y - 2 * z * z, x * y + y * z + z * x):
        assert_bitwise(run_gpu(f, 51, virtual=2), f, "3D stationary")


def test_exact_integer_rational_field():
    f = integer_field((33, 70), 5)
    assert_bitwise(run_gpu(f, 20, virtual=2), oracle.jacobi(f, 20), "integer field")


def test_subnormals_not_flushed():
    f = nv_field((34, 2400))
    exp = oracle.jacobi(f, 1000, 8)
    got = run_gpu(f, 1000)
    assert np.count_nonzero((exp != 0) & (np.abs(exp) < np.finfo(np.float64).tiny)) > 0
    assert_bitwise(got, exp, "subnormals")


def test_gather_scatter_roundtrip_and_run_zero():
    f = u12((7, 19, 23), 9)
    with jb.Jacobi(f.shape, virtual=2) as j:
        j.scatter(f)
        j.run(0)
        assert_bitwise(j.gather(), f, "roundtrip")


@pytest.mark.parametrize("shape", [(20, 64), (11, 9, 40)])
def test_no_compute_halo_slots_hold_neighbour_edges(shape):
    """after a no-compute run each slab's halo planes hold the neighbour's edge
    planes (P:550-552 measurement mode still moves every halo byte)."""
    f = u12(shape, 4)
    P = 3
    with jb.Jacobi(shape, virtual=P) as j:
        j.scatter(f)
        j.set_param("resident", 0)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE).run(3)
        par = j.iterations & 1
        slabs = [j.read_slab(i, par) for i in range(P)]
        chunks = [j.describe(i)["chunk"] for i in range(P)]
    for g in range(P):
        if g > 0:      # my top halo (plane 0) == top neighbour's last owned plane
            assert np.array_equal(slabs[g][0], slabs[g - 1][chunks[g - 1]])
        if g < P - 1:  # my bottom halo == bottom neighbour's first owned plane
            assert np.array_equal(slabs[g][chunks[g] + 1], slabs[g + 1][1])


def test_no_compute_mode_moves_halos_only():
    f = u12((20, 64), 4)
    with jb.Jacobi(f.shape, virtual=2) as j:
        j.scatter(f)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE).run(3)
        g = j.gather()
    # owned planes untouched (no arithmetic), only halos (not gathered) change
    assert_bitwise(g, f, "no-compute leaves owned planes")


# ---------------------------------------------------------------- errors
def test_errors():
    with pytest.raises(jb.JacobiError) as e:
        jb.Jacobi((2, 10))
    assert e.value.code == jb.JACOBI_EINVAL
    with pytest.raises(jb.JacobiError) as e:
        jb.Jacobi((5, 10), virtual=2)  # chunk 1.5 < 2
    assert e.value.code == jb.JACOBI_EINVAL
    with pytest.raises(jb.JacobiError) as e:
        jb.Jacobi((1000, 64), ngpus=64)
    assert e.value.code == jb.JACOBI_ENODEV
    with jb.Jacobi((10, 10)) as j:
        with pytest.raises(jb.JacobiError):
            j.set_mode(7)
        with pytest.raises(jb.JacobiError):
            j.run(-1)
        with pytest.raises(jb.JacobiError):
            j.set_param("nope", 1)


def test_watchdog_timeout_without_hang():
    with jb.Jacobi((40, 200), virtual=2) as j:
        j.set_param("timeout_ms", 300)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_DROP_SIGNAL)
        with pytest.raises(jb.JacobiError) as e:
            j.run(10)
        assert e.value.code == jb.JACOBI_ETIMEOUT
    # the device is still healthy afterwards
    f = u12((40, 200), 1)
    assert_bitwise(run_gpu(f, 3, virtual=2), oracle.jacobi(f, 3), "after timeout")


# ---------------------------------------------------------------- resident (on-chip) kernel, N2
@pytest.mark.parametrize("shape", [(3, 3), (9, 70), (300, 131), (1024, 1024), (5, 4, 9), (13, 30, 70),
                                   (20, 61, 130), (40, 40, 40)])
@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("sync", [0, 1])
def test_resident_vs_oracle(shape, P, sync):
    n_out = shape[0]
    if P > 1 and (n_out - 2) // P < 2:
        pytest.skip("slab too thin")
    f = u12(shape, 5)
    for iters in (1, 2, 9):
        with jb.Jacobi(shape, virtual=P) if P > 1 else jb.Jacobi(shape) as j:
            j.set_param("resident", 1)
            j.set_param("block_sync", sync)
            j.scatter(f)
            j.run(iters)
            assert jb.jacobi_get_param(j.h, "last_resident") == 1
            assert_bitwise(j.gather(), oracle.jacobi(f, iters), f"resident {shape} P={P} it={iters}")


def test_resident_auto_mixing_and_splitting():
    f = u12((66, 400), 6)
    exp = oracle.jacobi(f, 30)
    with jb.Jacobi(f.shape, virtual=4) as j:
        j.scatter(f)
        j.run(5)                                              # auto -> resident (fits)
        assert jb.jacobi_get_param(j.h, "last_resident") == 1
        j.set_param("resident", 0).run(6)                     # streaming
        j.set_mode(jb.MODE_BASELINE_MEMCPY).run(4)
        j.set_mode(jb.MODE_CPUFREE).set_param("resident", 1).run(7).run(8)
        assert j.iterations == 30
        assert_bitwise(j.gather(), exp, "resident mixed")


def test_resident_rejects_when_too_big():
    with jb.Jacobi((1024, 4096)) as j:  # 32 MB slab: does not fit on chip
        j.set_param("resident", 1)
        with pytest.raises(jb.JacobiError):
            j.run(1)
        j.set_param("resident", -1).run(1)
        assert jb.jacobi_get_param(j.h, "last_resident") == 0


def test_resident_watchdog():
    with jb.Jacobi((40, 200), virtual=2) as j:
        j.set_param("timeout_ms", 300)
        j.set_param("resident", 1)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_DROP_SIGNAL)
        with pytest.raises(jb.JacobiError) as e:
            j.run(10)
        assert e.value.code == jb.JACOBI_ETIMEOUT


def test_torch_allocator_owns_device_memory():
    """With use_torch_allocator() the slab buffers are PyTorch tensors; results are unchanged."""
    import torch
    f = u12((70, 300), 8)
    exp = oracle.jacobi(f, 9)
    before = torch.cuda.memory_allocated(0)
    jb.use_torch_allocator()
    try:
        with jb.Jacobi(f.shape, virtual=3) as j:
            assert torch.cuda.memory_allocated(0) > before  # our buffers live in torch's allocator
            j.scatter(f)
            j.run(4)
            j.set_param("resident", 0).run(5)
            assert_bitwise(j.gather(), exp, "torch allocator")
    finally:
        jb.use_torch_allocator(False)
    assert torch.cuda.memory_allocated(0) == before


# ---------------------------------------------------------------- N4: residual norm + convergence
def _converge_gpu(f, max_iters, tol, every, virtual=0, pre=0):
    with jb.Jacobi(f.shape, virtual=virtual) if virtual else jb.Jacobi(f.shape) as j:
        j.scatter(f)
        if pre:
            j.run(pre)  # a plain run first: the norm protocol must continue from any state
        j.set_tolerance(tol, every)
        t0 = j.iterations
        j.run(max_iters)
        return j.gather(), j.iterations - t0, j.last_norm


@pytest.mark.parametrize("shape", [(40, 130), (300, 77), (12, 30, 45), (33, 20, 20)])
@pytest.mark.parametrize("P", [1, 2, 4])
def test_converge_vs_oracle(shape, P):
    if (shape[0] - 2) // P < 2:
        pytest.skip("slab too thin")
    f = u12(shape, 9)
    _, _, norms = oracle.jacobi_converge(f, 400, 0.0, 10)
    tol = norms[len(norms) // 2] * (1 + 1e-9)  # stop at a check in the middle of the run
    exp, done, enorms = oracle.jacobi_converge(f, 400, tol, 10)
    got, gdone, gnorm = _converge_gpu(f, 400, tol, 10, virtual=P)
    assert gdone == done
    assert_bitwise(got, exp, f"converge {shape} P={P}")
    assert abs(gnorm - enorms[-1]) <= 1e-12 * enorms[-1]


def test_converge_never_and_split_runs():
    f = u12((50, 200), 10)
    exp, done, enorms = oracle.jacobi_converge(f, 55, 0.0, 5)  # tol 0: never stops
    assert done == 55
    got, gdone, gnorm = _converge_gpu(f, 55, 0.0, 5, virtual=3, pre=7)
    assert gdone == 55
    assert_bitwise(got, oracle.jacobi(f, 62), "converge after a plain run")
    with jb.Jacobi(f.shape, virtual=2) as j:  # repeated norm runs: monotone slots across runs
        j.scatter(f).set_tolerance(0.0, 4)
        for _ in range(3):
            j.run(8)
        assert j.iterations == 24
        assert_bitwise(j.gather(), oracle.jacobi(f, 24), "norm runs x3")


def test_gpu_matches_golden_digests():
    """The CUDA path (device U12 init, create -> run -> gather) reproduces the committed oracle
    digests of tests/golden bit for bit, with no oracle run."""
    import hashlib
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "oracle_digests.json")) as f:
        gold = json.load(f)
    for name, g in gold.items():
        for virtual in (0, 2):
            with jb.Jacobi(tuple(g["shape"]), virtual=virtual) as j:  # created with U12 seed 0x5C24
                j.run(g["iters"])
                r = j.gather()
            assert hashlib.sha256(np.ascontiguousarray(r).tobytes()).hexdigest() == g["sha256"], (name, virtual)


@pytest.mark.parametrize("virtual", [0, 2, 4, 8])
@pytest.mark.parametrize("mode", ["auto", "graph"])
def test_gpu_matches_latency_digests(virtual, mode):
    """C5 latency workloads (3D 128^3, 2D 1024^2) at 1000 iterations with 1-8 slabs, the auto
    kernel (time-blocked / static-schedule streaming / resident) and the CUDA-graph baseline: the
    whole field equals the committed oracle digest (tests/golden/oracle_digests_latency.json)."""
    import hashlib
    import json
    import os
    with open(os.path.join(os.path.dirname(__file__), "golden", "oracle_digests_latency.json")) as f:
        gold = json.load(f)
    for name, g in gold.items():
        with jb.Jacobi(tuple(g["shape"]), virtual=virtual) as j:  # created with U12 seed 0x5C24
            if mode == "graph":
                j.set_mode(jb.MODE_BASELINE_GRAPH)
            j.run(g["iters"])
            r = j.gather()
        assert hashlib.sha256(np.ascontiguousarray(r).tobytes()).hexdigest() == g["sha256"], (name, virtual, mode)


def test_nccl_baseline_then_import_torch():
    """The NCCL baseline loads the same libnccl.so.2 PyTorch ships (JACOBI_NCCL_LIB, set by the
    binding): running it BEFORE `import torch` must not leave a different NCCL in the process
    (a system NCCL of the same soname would be reused by torch and miss its symbols)."""
    import subprocess
    import sys
    code = ("import sys; sys.path.insert(0, %r)\n"
            "import numpy as np, paper_conf_sc_baydamirlibu24_b200 as jb\n"
            "with jb.Jacobi((40, 64)) as j:\n"
            "    j.set_mode(jb.MODE_BASELINE_NCCL); j.run(3)\n"
            "import torch\n"
            "print('TORCH_OK', torch.cuda.is_available())\n") % ROOT_DIR
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300)
    assert "TORCH_OK True" in r.stdout, (r.stdout + r.stderr)[-3000:]


# ---------------------------------------------------------------- halo flag scope
@pytest.mark.parametrize("shape,virtual", [((66, 300), 3), ((23, 20, 70), 2), ((130, 1030), 4)])
@pytest.mark.parametrize("kernel", [{"resident": 0, "tblock": 0}, {"resident": 1}, {"resident": 0, "tblock": 1},
                                    {"resident": 0, "tblock": 0, "halo_ll": 1}])
@pytest.mark.parametrize("scope", [0, 1])
def test_flag_scope_virtual_bitwise(shape, virtual, kernel, scope):
    """Virtual slabs with halo flags at .sys (flag_scope 0) and .gpu scope (1; auto for virtual
    slabs): the same bits as the oracle, for the streaming, resident, time-blocked and LL kernels."""
    f = u12(shape, 11)
    got = run_gpu(f, 23, virtual=virtual, params={**kernel, "flag_scope": scope})
    assert_bitwise(got, oracle.jacobi(f, 23), f"{shape} P={virtual} {kernel} scope={scope}")


def test_flag_scope_knob():
    """.gpu scope is refused for a handle whose slabs may live on other GPUs / processes."""
    with jb.Jacobi((40, 40)) as j:
        assert j.get_param("flag_scope") == -1
        with pytest.raises(jb.JacobiError):
            j.set_param("flag_scope", 1)
        j.set_param("flag_scope", 0)
    with jb.Jacobi((40, 40), virtual=2) as j:
        j.set_param("flag_scope", 1)


@pytest.mark.parametrize("params,flags", [({"resident": 0, "tblock": 0}, 0),
                                          ({"resident": 0, "tblock": 0}, jb.FLAG_NO_COMPUTE),
                                          ({"resident": 1}, 0), ({"resident": 1, "block_sync": 1}, 0),
                                          ({"resident": 0, "tblock": 1}, 0)])
@pytest.mark.parametrize("scope", [0, 1])
def test_watchdog_every_kernel(params, flags, scope):
    """DROP_SIGNAL on slab 0 with every CPU-Free kernel and both flag scopes: the waits that moved
    into the barrier (pre-wait) and the no-compute signal folded into the arrival still end in
    JACOBI_ETIMEOUT, not a hang, and the next run on a new handle is bitwise."""
    with jb.Jacobi((40, 200), virtual=2) as j:
        j.set_param("timeout_ms", 300)
        j.set_param("flag_scope", scope)
        for k, v in params.items():
            j.set_param(k, v)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_DROP_SIGNAL | flags)
        with pytest.raises(jb.JacobiError) as e:
            j.run(10)
        assert e.value.code == jb.JACOBI_ETIMEOUT
    f = u12((40, 200), 1)
    assert_bitwise(run_gpu(f, 5, virtual=2, params=params), oracle.jacobi(f, 5), f"after timeout {params}")
