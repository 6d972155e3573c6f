"""N3: the NVSHMEM variant of the CPU-Free kernel (libjacobi_b200_nvshmem.so) —
halos delivered with nvshmemx_putmem_signal_nbi_warp + signals, the paper's own layer (P:323,
P:394).  Two PEs share the pool's single GPU (NVSHMEM_DISABLE_NVLS=1; the driver time-slices their
persistent kernels), 2D and 3D, plain and convergence-terminated runs, bitwise vs the oracle."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shape, iters, tol, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), NVSHMEM_DISABLE_NVLS="1",
                          NVSHMEM_BOOTSTRAP_UID_SOCK_IFNAME="lo")
        import torch.distributed as dist
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import paper_conf_sc_baydamirlibu24_b200 as jb
        from jacobi_inputs import u12
        f = u12(shape, 11)
        outs = []
        j = jb.create_nvshmem(shape)
        j.set_param("timeout_ms", 60000)
        for mode_tol in (None, tol, "baseline"):
            j.scatter(f)
            if mode_tol == "baseline":  # P:531 "Baseline NVSHMEM": discrete kernels + sync kernel
                j.set_tolerance(0.0, 0)
                j.set_mode(jb.MODE_BASELINE_NVSHMEM)
            elif mode_tol is not None:
                j.set_tolerance(mode_tol, 5)
            t0 = j.iterations
            dist.barrier()
            j.run(iters)
            out = np.full(f.shape, np.nan)
            j.gather(out)
            outs.append((out, j.iterations - t0))
            dist.barrier()
        j.close()
        jb.nvshmem_finalize()
        dist.destroy_process_group()
        q.put((rank, outs, None))
    except Exception as e:
        q.put((rank, None, repr(e)))


@pytest.mark.parametrize("shape", [(40, 96), (12, 13, 40)])
def test_nvshmem_two_pes(shape):
    import oracle
    from jacobi_inputs import u12
    from paper_conf_sc_baydamirlibu24_b200 import build as b
    if b.nvshmem_home() is None:
        pytest.skip("no NVSHMEM")
    f = u12(shape, 11)
    iters = 30
    _, _, norms = oracle.jacobi_converge(f, iters, 0.0, 5)
    tol = norms[2] * (1 + 1e-9)
    exp_conv, done, _ = oracle.jacobi_converge(f, iters, tol, 5)
    exp_plain = oracle.jacobi(f, iters)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, shape, iters, tol, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        rank, outs, err = q.get(timeout=300)
        assert err is None, err
        res[rank] = outs
    for p in procs:
        p.join(timeout=60)
    for k, (exp, n_exp) in enumerate([(exp_plain, iters), (exp_conv, done), (exp_plain, iters)]):
        a, na = res[0][k]
        bb, nb = res[1][k]
        assert na == nb == n_exp
        merged = np.where(np.isnan(a), bb, a)
        assert np.array_equal(merged.view(np.uint64), exp.view(np.uint64)), k
