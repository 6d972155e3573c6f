"""Real multi-GPU parity (BASELINE.json north_star: "the 2/4/8-GPU result must
be bitwise identical to the 1-GPU result"): the single-process path jacobi_create(ngpus=P) —
one slab per physical device, cudaDeviceEnablePeerAccess, UVA peer stores of the halo planes
and sys-scope release flags across devices — and the one-process-per-GPU
path (CUDA IPC between ranks on different devices).

Every test is gated on torch.cuda.device_count() >= P and skips cleanly on the 1-GPU pool; on an
8-GPU node they all run.  The halo-trace test at the end uses virtual slabs and runs everywhere.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import paper_conf_sc_baydamirlibu24_b200 as jb
from jacobi_inputs import u12

pytestmark = pytest.mark.gpu


def ndev():
    import torch
    return torch.cuda.device_count()


def need(P):
    if ndev() < P:
        pytest.skip(f"needs {P} GPUs, {ndev()} visible")


def bits_equal(a, b):
    return np.array_equal(np.asarray(a).view(np.uint64), np.asarray(b).view(np.uint64))


def assert_bitwise(got, exp, what=""):
    if not bits_equal(got, exp):
        d = np.abs(got - exp)
        n = np.count_nonzero(got.view(np.uint64) != exp.view(np.uint64))
        raise AssertionError(f"{what}: {n} cells differ, max |diff| {d.max()}")


def run_multi(field, iters, P, mode=jb.MODE_CPUFREE, params=None, flags=0, splits=None):
    with jb.Jacobi(field.shape, ngpus=P) as j:
        j.set_param("timeout_ms", 60000)
        for k, v in (params or {}).items():
            j.set_param(k, v)
        j.set_mode(mode, flags)
        j.scatter(field)
        for n in (splits or [iters]):
            j.run(n)
        return j.gather(), j


PS = [2, 4, 8]
STREAM = {"resident": 0, "tblock": 0}
TB = {"resident": 0, "tblock": 1}


@pytest.mark.parametrize("P", PS)
def test_create_places_one_slab_per_device(P):
    need(P)
    with jb.Jacobi((4 * P + 5, 300), ngpus=P) as j:
        assert j.local_slabs == P and j.total_slabs == P
        assert [j.describe(i)["device"] for i in range(P)] == list(range(P))


def test_create_more_gpus_than_visible_is_enodev():
    n = ndev()
    with pytest.raises(jb.JacobiError) as e:
        jb.Jacobi((64, 64), ngpus=n + 1)
    assert e.value.code == jb.JACOBI_ENODEV


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("params", [STREAM, TB, {}], ids=["streaming", "tblock", "auto"])
def test_ragged_2d_vs_oracle(P, params):
    """Remainder chunks (first r slabs one row more), a tail tile in x, 2D."""
    need(P)
    rows = 2 + 10 * P + (P - 1)  # chunk 10 or 11 (>= 2K = 10 for the K = 5 edge zones)
    f = u12((rows, 2051), 11)
    got, _ = run_multi(f, 23, P, params=params)
    assert_bitwise(got, oracle.jacobi(f, 23), f"2D P={P} {params}")


@pytest.mark.parametrize("P", PS)
def test_chunk2_slabs_vs_oracle(P):
    """The minimum chunk of 2 planes per GPU (no interior work at all: only boundary roles)."""
    need(P)
    f = u12((2 + 2 * P, 700), 12)
    got, _ = run_multi(f, 9, P, params=STREAM)
    assert_bitwise(got, oracle.jacobi(f, 9), f"chunk 2, P={P}")
    f3 = u12((2 + 2 * P, 20, 70), 13)
    got, _ = run_multi(f3, 5, P, params=STREAM)
    assert_bitwise(got, oracle.jacobi(f3, 5), f"3D chunk 2, P={P}")


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("params", [STREAM, TB, {}], ids=["streaming", "tblock", "auto"])
def test_ragged_3d_vs_oracle(P, params):
    need(P)
    f = u12((2 + 6 * P + 1, 29, 133), 14)
    got, _ = run_multi(f, 12, P, params=params)
    assert_bitwise(got, oracle.jacobi(f, 12), f"3D P={P} {params}")


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("mode", [jb.MODE_BASELINE_MEMCPY, jb.MODE_BASELINE_NCCL, jb.MODE_BASELINE_OVERLAP,
                                  jb.MODE_BASELINE_P2P, jb.MODE_BASELINE_GRAPH])
def test_cpu_controlled_baselines_with_real_peers(P, mode):
    """a10 / N1: cudaMemcpyPeerAsync, NCCL send/recv (single-process ncclCommInitAll), Overlap,
    P2P stores and the CUDA graph — halos moved between physical devices."""
    need(P)
    f = u12((2 + 7 * P, 515), 15)
    got, _ = run_multi(f, 11, P, mode=mode)
    assert_bitwise(got, oracle.jacobi(f, 11), f"mode {mode} P={P}")
    f3 = u12((2 + 3 * P, 18, 40), 16)
    got, _ = run_multi(f3, 6, P, mode=mode)
    assert_bitwise(got, oracle.jacobi(f3, 6), f"3D mode {mode} P={P}")


@pytest.mark.parametrize("P", [2, 8])
def test_mode_mixing_and_run_splitting_across_devices(P):
    """run(a); run(b) == run(a+b) across CPU-Free (time-blocked, streaming) and baseline runs."""
    need(P)
    f = u12((2 + 12 * P, 600), 17)
    exp = oracle.jacobi(f, 5 + 3 + 10 + 7 + 4)
    with jb.Jacobi(f.shape, ngpus=P) as j:
        j.scatter(f)
        j.run(5)                              # time-blocked (K = 5)
        j.set_param("tblock", 0).run(3)       # streaming
        j.set_mode(jb.MODE_BASELINE_NCCL).run(10)
        j.set_mode(jb.MODE_CPUFREE).set_param("tblock", -1).run(7)
        j.set_mode(jb.MODE_BASELINE_MEMCPY).run(4)
        assert_bitwise(j.gather(), exp, f"mixed P={P}")


@pytest.mark.parametrize("P", PS)
def test_c2_1000_iters_p_gpus_equals_one_gpu(P):
    """C2 (16384^2, 1000 iterations): P physical GPUs (time-blocked edge zones over NVLink) ==
    1 GPU, bitwise on every one of the 268 M cells."""
    need(P)
    shape = (16384, 16384)
    with jb.Jacobi(shape, ngpus=1) as j1:
        j1.run(1000)
        ref = j1.gather()
    with jb.Jacobi(shape, ngpus=P) as j:
        j.run(1000)
        assert j.get_param("last_tblock") == 1000
        assert_bitwise(j.gather(), ref, f"C2 P={P}")


@pytest.mark.parametrize("P", PS)
def test_c3_1000_iters_p_gpus_equals_one_gpu(P):
    """C3 (512^3, 1000 iterations): P physical GPUs == 1 GPU, bitwise."""
    need(P)
    shape = (512, 512, 512)
    with jb.Jacobi(shape, ngpus=1) as j1:
        j1.run(1000)
        ref = j1.gather()
    with jb.Jacobi(shape, ngpus=P) as j:
        j.run(1000)
        assert_bitwise(j.gather(), ref, f"C3 P={P}")
    with jb.Jacobi(shape, ngpus=P) as j:
        j.set_mode(jb.MODE_BASELINE_NCCL).run(1000)
        assert_bitwise(j.gather(), ref, f"C3 NCCL baseline P={P}")


@pytest.mark.parametrize("P", PS)
def test_watchdog_across_devices(P):
    """A GPU that never signals (DROP_SIGNAL on slab 0) -> JACOBI_ETIMEOUT on the waiting devices,
    no hang; the handle stays usable for a clean run afterwards."""
    need(P)
    f = u12((2 + 12 * P, 300), 18)
    for params in (STREAM, TB):
        with jb.Jacobi(f.shape, ngpus=P) as j:
            for k, v in params.items():
                j.set_param(k, v)
            j.set_param("timeout_ms", 300)
            j.set_mode(jb.MODE_CPUFREE, jb.FLAG_DROP_SIGNAL)
            j.scatter(f)
            with pytest.raises(jb.JacobiError) as e:
                j.run(10)
            assert e.value.code == jb.JACOBI_ETIMEOUT


@pytest.mark.parametrize("P", [2, 4])
def test_norm_all_reduce_across_devices(P):
    """N4: the device-side norm all-reduce over NVLink stops every GPU after the same check."""
    need(P)
    f = u12((2 + 10 * P, 96), 7)
    _, _, norms = oracle.jacobi_converge(f, 200, 0.0, 5)
    tol = norms[7] * (1 + 1e-9)
    exp, done, _ = oracle.jacobi_converge(f, 200, tol, 5)
    with jb.Jacobi(f.shape, ngpus=P) as j:
        j.scatter(f)
        j.set_tolerance(tol, 5)
        j.run(200)
        assert j.iterations == done
        assert_bitwise(j.gather(), exp, f"norm P={P}")


@pytest.mark.parametrize("P", PS)
def test_halo_trace_on_real_devices(P):
    need(P)
    f = u12((2 + 20 * P, 4096), 19)
    with jb.Jacobi(f.shape, ngpus=P) as j:
        j.scatter(f)
        j.set_param("halo_trace", 50)
        j.set_param("tblock", 0).set_param("resident", 0)
        j.run(50)
        for i in range(P):
            tr = j.halo_trace(i, 50).astype(np.int64)
            for side, has in ((0, i > 0), (1, i < P - 1)):
                if has:
                    assert (tr[side, 1:, 0] > 0).all() and (tr[side, 1:, 1] >= tr[side, 1:, 0]).all()
                    assert (tr[side, 1:, 2] >= tr[side, 1:, 1]).all()
                else:
                    assert (tr[side] == 0).all()


# ---------------------------------------------------------------- one process per GPU
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shape, iters, q, params, nccl_mode):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(rank)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        f = u12(shape, 21)
        jb.use_torch_allocator()
        j = jb.Jacobi(shape, dist=(rank, world), device=rank)
        j.set_param("timeout_ms", 60000)
        for k, v in (params or {}).items():
            j.set_param(k, v)
        jb.exchange_peers(j, nccl=True)
        j.scatter(f)
        dist.barrier()
        if nccl_mode:
            j.set_mode(jb.MODE_BASELINE_NCCL)
        j.run(iters)
        out = np.full(f.shape, np.nan)
        j.gather(out)
        dist.barrier()
        j.close()
        dist.destroy_process_group()
        q.put((rank, out, None))
    except Exception as e:
        q.put((rank, None, repr(e)))


@pytest.mark.parametrize("P", PS)
@pytest.mark.parametrize("shape,params,nccl_mode", [((61, 1030), None, False), ((61, 1030), TB, False),
                                                    ((23, 20, 70), None, False), ((23, 20, 70), TB, False),
                                                    ((61, 1030), None, True)])
def test_one_process_per_gpu_ipc(P, shape, params, nccl_mode):
    """torchrun-style ranks on P distinct devices: CUDA IPC peer stores between GPUs, the NCCL
    baseline between processes; result merged from all ranks == oracle."""
    need(P)
    if (shape[0] - 2) // P < (10 if params else 2):
        pytest.skip("slabs too thin for this P")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, P, port, shape, 17, q, params, nccl_mode)) for r in range(P)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(P):
        rank, out, err = q.get(timeout=300)
        assert err is None, err
        res[rank] = out
    for p in procs:
        p.join(timeout=60)
    merged = res[0]
    for r in range(1, P):
        merged = np.where(np.isnan(merged), res[r], merged)
    assert not np.isnan(merged).any()
    assert_bitwise(merged, oracle.jacobi(u12(shape, 21), 17), f"IPC P={P}")


# ---------------------------------------------------------------- runs on one GPU too
@pytest.mark.parametrize("params", [STREAM, TB, {"resident": 1, "tblock": 0}], ids=["streaming", "tblock", "resident"])
def test_halo_trace_virtual_slabs(params):
    """jacobi_halo_trace: every exchange of every side with a neighbour is recorded in order
    (wait begins <= flag acquired <= signal released), sides without one stay zero."""
    P = 3
    f = u12((2 + 20 * P, 1000), 20)
    n = 40
    with jb.Jacobi(f.shape, virtual=P) as j:
        for k, v in params.items():
            j.set_param(k, v)
        j.scatter(f)
        j.set_param("halo_trace", n)
        j.run(n)
        got = j.gather()
        for i in range(P):
            tr = j.halo_trace(i, n).astype(np.int64)
            for side, has in ((0, i > 0), (1, i < P - 1)):
                t = tr[side]
                if not has:
                    assert (t == 0).all()
                    continue
                first = 1 if params.get("resident") == 1 else 0  # resident: no wait before iteration 0
                assert (t[first:, 0] > 0).all() and (t[:, 2] > 0).all(), (i, side)
                assert (t[first:, 1] >= t[first:, 0]).all() and (t[first:, 2] >= t[first:, 1]).all()
                assert (np.diff(t[:, 2]) > 0).all()  # signals in iteration order
            sp = jb.halo_spans(tr, skip=2)
            assert sp["span_us"] is not None and sp["span_us"] >= 0
        with pytest.raises(jb.JacobiError):
            j.halo_trace(0, n + 1)
    assert_bitwise(got, oracle.jacobi(f, n), "traced run")
