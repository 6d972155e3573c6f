"""World-size-2 gloo tests of the multi-process host plumbing (CPU only): the IPC-blob
exchange that wires slab g to g-1 / g+1, the NCCL-id broadcast, the max-over-ranks timing
reduction bench.py uses, and the per-rank slab bookkeeping (jacobi_decompose)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_baydamirlibu24_b200 as jb
    blob = f"blob-of-rank-{rank}".encode() * 3
    top, bot = jb.exchange_blobs(blob)
    uid = jb.broadcast_blob(b"unique-id-from-rank-0" if rank == 0 else None)
    t = torch.tensor([float(10 * rank + 1)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    start, chunk = jb.jacobi_decompose(16384, world, rank)
    q.put((rank, top, bot, uid, t.item(), start, chunk))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_exchange(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    nxt = 1
    for rank, top, bot, uid, mx, start, chunk in res:
        assert top == (f"blob-of-rank-{rank - 1}".encode() * 3 if rank > 0 else None)
        assert bot == (f"blob-of-rank-{rank + 1}".encode() * 3 if rank < world - 1 else None)
        assert uid == b"unique-id-from-rank-0"
        assert mx == 10 * (world - 1) + 1
        assert start == nxt
        nxt = start + chunk
    assert nxt == 16383
