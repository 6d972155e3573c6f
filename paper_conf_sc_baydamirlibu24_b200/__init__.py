"""Thin Python binding of libjacobi_b200.so (include/jacobi.h) — argument marshalling only.

Every step of the hot path runs in the CUDA library; this module never computes the stencil
and has no CPU fallback: if the extension is missing it raises.  Function names mirror the C
ABI (``jacobi_create``, ``jacobi_run``, ...); ``Jacobi`` is a small convenience wrapper over a
handle used by tests, ``bench.py`` and ``__graft_entry__``.  PyTorch is used only as plumbing
(torch.distributed to exchange CUDA IPC handles / the NCCL unique id between ranks).
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("JACOBI_LIB") or os.path.join(_HERE, "libjacobi_b200.so")  # env: A/B measurement aid
NVSHMEM_LIB_PATH = os.path.join(_HERE, "libjacobi_b200_nvshmem.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "jacobi.h")

JACOBI_OK = 0
JACOBI_EINVAL = -1
JACOBI_ENODEV = -2
JACOBI_ENOPEER = -3
JACOBI_ENOCOOP = -4
JACOBI_ENOMEM = -5
JACOBI_ECUDA = -6
JACOBI_ETIMEOUT = -7
JACOBI_ENCCL = -8
JACOBI_ESTATE = -9

MODE_CPUFREE = 0
MODE_BASELINE_MEMCPY = 1
MODE_BASELINE_NCCL = 2
MODE_BASELINE_OVERLAP = 3
MODE_BASELINE_P2P = 4
MODE_BASELINE_GRAPH = 5
MODE_BASELINE_NVSHMEM = 6
FLAG_NO_COMPUTE = 1
FLAG_DROP_SIGNAL = 2

_c = ctypes
_i64 = _c.c_int64
_p = _c.c_void_p
_SIGS = {
    "jacobi_create": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.POINTER(_p)], _c.c_int),
    "jacobi_create_virtual": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_p)], _c.c_int),
    "jacobi_create_rank": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_p)], _c.c_int),
    "jacobi_ipc_handle_bytes": ([], _c.c_int),
    "jacobi_get_ipc_handle": ([_p, _p], _c.c_int),
    "jacobi_open_peers": ([_p, _p, _p], _c.c_int),
    "jacobi_nccl_unique_id": ([_p], _c.c_int),
    "jacobi_nccl_init": ([_p, _p], _c.c_int),
    "jacobi_run": ([_p, _i64], _c.c_int),
    "jacobi_set_mode": ([_p, _c.c_int, _c.c_int], _c.c_int),
    "jacobi_set_param": ([_p, _c.c_char_p, _i64], _c.c_int),
    "jacobi_get_param": ([_p, _c.c_char_p, _c.POINTER(_i64)], _c.c_int),
    "jacobi_scatter": ([_p, _p], _c.c_int),
    "jacobi_gather": ([_p, _p], _c.c_int),
    "jacobi_last_time": ([_p, _c.POINTER(_c.c_double), _c.POINTER(_c.c_double)], _c.c_int),
    "jacobi_iterations": ([_p, _c.POINTER(_i64)], _c.c_int),
    "jacobi_num_slabs": ([_p, _c.POINTER(_c.c_int), _c.POINTER(_c.c_int)], _c.c_int),
    "jacobi_describe": ([_p, _c.c_int, _c.POINTER(_i64)], _c.c_int),
    "jacobi_strerror": ([_c.c_int], _c.c_char_p),
    "jacobi_destroy": ([_p], _c.c_int),
    "jacobi_decompose": ([_i64, _c.c_int, _c.c_int, _c.POINTER(_i64), _c.POINTER(_i64)], _c.c_int),
    "jacobi_tb_split": ([_c.c_int, _i64, _c.c_int, _c.c_int, _i64, _c.c_int, _c.POINTER(_c.c_int)], _c.c_int),
    "jacobi_geometry": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_i64)], _c.c_int),
    "jacobi_auto_policy": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_i64)], _c.c_int),
    "jacobi_version": ([], _c.c_int),
    "jacobi_set_allocator": ([_p, _p, _p], _c.c_int),
    "jacobi_open_ranks": ([_p, _p, _c.c_int], _c.c_int),
    "jacobi_set_tolerance": ([_p, _c.c_double], _c.c_int),
    "jacobi_last_norm": ([_p, _c.POINTER(_c.c_double)], _c.c_int),
    "jacobi_slab_bytes": ([_i64, _i64, _i64, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_i64)], _c.c_int),
    "jacobi_read_slab": ([_p, _c.c_int, _c.c_int, _p], _c.c_int),
    "jacobi_halo_trace": ([_p, _c.c_int, _p, _i64], _c.c_int),
}
# exported only by the NVSHMEM variant (libjacobi_b200_nvshmem.so)
_SIGS_NVSHMEM = {
    "jacobi_nvshmem_uid_bytes": ([], _c.c_int),
    "jacobi_nvshmem_uid": ([_p], _c.c_int),
    "jacobi_create_nvshmem": ([_i64, _i64, _i64, _c.c_int, _p, _c.c_int, _c.c_int, _c.c_int, _c.POINTER(_p)],
                              _c.c_int),
    "jacobi_nvshmem_finalize": ([], _c.c_int),
}

ALLOC_FN = _c.CFUNCTYPE(_c.c_void_p, _c.c_size_t, _c.c_int, _c.c_void_p)
FREE_FN = _c.CFUNCTYPE(None, _c.c_void_p, _c.c_int, _c.c_void_p)

_lib = None


class JacobiError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = int(code)
        super().__init__(f"{what}: {strerror(code)} ({code})" if what else f"{strerror(code)} ({code})")


def _torch_nccl() -> str | None:
    """Path of the libnccl.so.2 PyTorch ships (nvidia-nccl wheel), if any — without importing torch."""
    import importlib.util
    try:
        spec = importlib.util.find_spec("nvidia.nccl")
    except (ImportError, ValueError):
        return None
    for base in (spec.submodule_search_locations or []) if spec else []:
        p = os.path.join(base, "lib", "libnccl.so.2")
        if os.path.exists(p):
            return p
    return None


def lib() -> ctypes.CDLL:
    """Load the CUDA extension.  Fails loudly if it has not been built (no fallback)."""
    global _lib
    if _lib is None:
        nccl = _torch_nccl()  # the NCCL baseline uses the same libnccl as PyTorch (one per process)
        if nccl and "JACOBI_NCCL_LIB" not in os.environ:
            os.environ["JACOBI_NCCL_LIB"] = nccl
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"CUDA extension missing: {LIB_PATH} (run __graft_entry__.build())")
        L = ctypes.CDLL(LIB_PATH)
        sigs = dict(_SIGS, **(_SIGS_NVSHMEM if LIB_PATH == NVSHMEM_LIB_PATH else {}))
        for name, (args, res) in sigs.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def use_nvshmem() -> None:
    """Switch this process to the NVSHMEM variant of the library (N3).  Must be called before the
    library is first used; every call of this module then goes through that library."""
    global LIB_PATH
    if _lib is not None and LIB_PATH != NVSHMEM_LIB_PATH:
        raise RuntimeError("use_nvshmem() must precede the first use of the library")
    if not os.path.exists(NVSHMEM_LIB_PATH):
        raise RuntimeError(f"NVSHMEM variant missing: {NVSHMEM_LIB_PATH}")
    LIB_PATH = NVSHMEM_LIB_PATH


def header_functions(nvshmem: bool = False) -> list[str]:
    """Names of the functions declared in include/jacobi.h: those of the main library, or (with
    nvshmem=True) those exported only by the NVSHMEM variant."""
    with open(HEADER_PATH) as f:
        src = f.read()
    names = re.findall(r"^\s*(?:int|const char \*)\s*(jacobi_\w+)\s*\(", src, flags=re.M)
    return [n for n in names if (n in _SIGS_NVSHMEM) == nvshmem]


def strerror(code: int) -> str:
    return lib().jacobi_strerror(int(code)).decode()


def _check(rc: int, what: str) -> None:
    if rc != JACOBI_OK:
        raise JacobiError(rc, what)


# ---------------------------------------------------------------- C-ABI mirrors
def jacobi_create(nx, ny, nz, stencil, ngpus) -> int:
    h = _p()
    _check(lib().jacobi_create(nx, ny, nz, stencil, ngpus, _c.byref(h)), "jacobi_create")
    return h.value


def jacobi_create_virtual(nx, ny, nz, stencil, nslabs, device=0) -> int:
    h = _p()
    _check(lib().jacobi_create_virtual(nx, ny, nz, stencil, nslabs, device, _c.byref(h)), "jacobi_create_virtual")
    return h.value


def jacobi_create_rank(nx, ny, nz, stencil, world_size, rank, device) -> int:
    h = _p()
    _check(lib().jacobi_create_rank(nx, ny, nz, stencil, world_size, rank, device, _c.byref(h)),
           "jacobi_create_rank")
    return h.value


def jacobi_get_ipc_handle(h) -> bytes:
    n = lib().jacobi_ipc_handle_bytes()
    buf = _c.create_string_buffer(n)
    _check(lib().jacobi_get_ipc_handle(h, buf), "jacobi_get_ipc_handle")
    return buf.raw


def jacobi_open_peers(h, top: bytes | None, bottom: bytes | None) -> None:
    _check(lib().jacobi_open_peers(h, top, bottom), "jacobi_open_peers")


def jacobi_open_ranks(h, blobs: list) -> None:
    _check(lib().jacobi_open_ranks(h, b"".join(blobs), len(blobs)), "jacobi_open_ranks")


def jacobi_set_tolerance(h, tol: float) -> None:
    _check(lib().jacobi_set_tolerance(h, float(tol)), "jacobi_set_tolerance")


def jacobi_last_norm(h) -> float:
    v = _c.c_double()
    _check(lib().jacobi_last_norm(h, _c.byref(v)), "jacobi_last_norm")
    return v.value


def jacobi_nccl_unique_id() -> bytes:
    buf = _c.create_string_buffer(128)
    _check(lib().jacobi_nccl_unique_id(buf), "jacobi_nccl_unique_id")
    return buf.raw


def jacobi_nccl_init(h, uid: bytes) -> None:
    _check(lib().jacobi_nccl_init(h, uid), "jacobi_nccl_init")


def jacobi_run(h, iters: int) -> None:
    _check(lib().jacobi_run(h, int(iters)), "jacobi_run")


def jacobi_set_mode(h, mode: int, flags: int = 0) -> None:
    _check(lib().jacobi_set_mode(h, int(mode), int(flags)), "jacobi_set_mode")


def jacobi_set_param(h, name: str, value: int) -> None:
    _check(lib().jacobi_set_param(h, name.encode(), int(value)), f"jacobi_set_param({name})")


def jacobi_get_param(h, name: str) -> int:
    v = _i64()
    _check(lib().jacobi_get_param(h, name.encode(), _c.byref(v)), f"jacobi_get_param({name})")
    return v.value


def _host_ptr(a: np.ndarray, n: int, writable: bool) -> int:
    if not isinstance(a, np.ndarray) or a.dtype != np.float64 or not a.flags["C_CONTIGUOUS"] or a.size != n:
        raise ValueError(f"expected a C-contiguous float64 array of {n} elements")
    if writable and not a.flags["WRITEABLE"]:
        raise ValueError("output array is read-only")
    return a.ctypes.data


def jacobi_scatter(h, field: np.ndarray, n: int) -> None:
    _check(lib().jacobi_scatter(h, _host_ptr(field, n, False)), "jacobi_scatter")


def jacobi_gather(h, out: np.ndarray, n: int) -> None:
    _check(lib().jacobi_gather(h, _host_ptr(out, n, True)), "jacobi_gather")


def jacobi_scatter_ptr(h, ptr: int) -> None:
    _check(lib().jacobi_scatter(h, _p(ptr)), "jacobi_scatter")


def jacobi_gather_ptr(h, ptr: int) -> None:
    _check(lib().jacobi_gather(h, _p(ptr)), "jacobi_gather")


def jacobi_last_time(h, nslabs: int):
    mx = _c.c_double()
    per = (_c.c_double * max(nslabs, 1))()
    _check(lib().jacobi_last_time(h, _c.byref(mx), per), "jacobi_last_time")
    return mx.value, list(per)[:nslabs]


def jacobi_halo_trace(h, slab: int, n: int) -> np.ndarray:
    """Raw halo-exchange trace of the last CPU-Free run: uint64 array [2 sides][n exchanges][3]
    (%globaltimer ns at wait begin / flag acquired / signal released; 0 = not recorded)."""
    out = np.zeros((2, n, 3), dtype=np.uint64)
    _check(lib().jacobi_halo_trace(h, int(slab), out.ctypes.data, int(n)), "jacobi_halo_trace")
    return out


def halo_spans(trace: np.ndarray, skip: int = 0) -> dict:
    """Summary (median µs over exchanges >= skip, both sides) of a jacobi_halo_trace array:
    wait = flag acquired - wait begin, put = signal - flag acquired (edge plane compute + peer
    stores + release), span = signal - wait begin (the boundary block's whole exchange), period =
    time between consecutive signals of a side (the per-iteration halo cadence)."""
    t = trace.astype(np.int64)
    out = {}
    for key, (i, j) in {"wait_us": (0, 1), "put_us": (1, 2), "span_us": (0, 2)}.items():
        v = []
        for side in range(2):
            a, b = t[side, skip:, i], t[side, skip:, j]
            m = (a > 0) & (b > 0)
            v.extend(((b[m] - a[m]) / 1e3).tolist())
        out[key] = float(np.median(v)) if v else None
    per = []
    for side in range(2):
        sg = t[side, skip:, 2]
        sg = sg[sg > 0]
        if len(sg) > 1:
            per.extend((np.diff(sg) / 1e3).tolist())
    out["period_us"] = float(np.median(per)) if per else None
    out["exchanges"] = int(((t[:, skip:, 2] > 0)).sum())
    return out


def jacobi_iterations(h) -> int:
    t = _i64()
    _check(lib().jacobi_iterations(h, _c.byref(t)), "jacobi_iterations")
    return t.value


def jacobi_num_slabs(h):
    a, b = _c.c_int(), _c.c_int()
    _check(lib().jacobi_num_slabs(h, _c.byref(a), _c.byref(b)), "jacobi_num_slabs")
    return a.value, b.value


DESCRIBE_KEYS = ("start", "chunk", "pitch", "plane_elems", "tile_x", "tile_y", "units_x", "units_y",
                 "stages", "n_top", "n_bot", "n_interior", "ctas", "k_planes", "smem_bytes", "device")


def jacobi_describe(h, i: int) -> dict:
    o = (_i64 * 16)()
    _check(lib().jacobi_describe(h, int(i), o), "jacobi_describe")
    return dict(zip(DESCRIBE_KEYS, list(o)))


def jacobi_destroy(h) -> None:
    _check(lib().jacobi_destroy(h), "jacobi_destroy")


def jacobi_decompose(n_out: int, nslabs: int, slab: int):
    s, c = _i64(), _i64()
    _check(lib().jacobi_decompose(n_out, nslabs, slab, _c.byref(s), _c.byref(c)), "jacobi_decompose")
    return s.value, c.value


def jacobi_tb_split(ctas, chunk, has_top, has_bottom, units, override_per_side=0):
    o = (_c.c_int * 3)()
    _check(lib().jacobi_tb_split(ctas, chunk, int(has_top), int(has_bottom), units, override_per_side, o),
           "jacobi_tb_split")
    return tuple(o)


GEOMETRY_KEYS = ("pitch", "plane_elems", "tile_x", "tile_y", "units_x", "units_y", "stage_rows", "stage_row_doubles")


def jacobi_geometry(nx, ny, nz, stencil, tile_x=0, tile_y=0) -> dict:
    o = (_i64 * 8)()
    _check(lib().jacobi_geometry(nx, ny, nz, stencil, tile_x, tile_y, o), "jacobi_geometry")
    return dict(zip(GEOMETRY_KEYS, list(o)))


def jacobi_auto_policy(nx, ny, nz, stencil, nslabs, virtual=False, sms=148) -> dict:
    """Host-only auto policies of the C ABI: cells per CTA of the job, dynamic
    interior schedule, time-blocked kernel, CTAs of the smallest slab."""
    o = (_i64 * 4)()
    _check(lib().jacobi_auto_policy(nx, ny, nz, stencil, nslabs, 1 if virtual else 0, sms, o), "jacobi_auto_policy")
    return {"cells_per_cta": o[0], "dynamic_schedule": bool(o[1]), "tblock": bool(o[2]), "min_slab_ctas": o[3]}


def jacobi_version() -> int:
    return lib().jacobi_version()


def jacobi_slab_bytes(nx, ny, nz, stencil, nslabs, slab) -> int:
    b = _i64()
    _check(lib().jacobi_slab_bytes(nx, ny, nz, stencil, nslabs, slab, _c.byref(b)), "jacobi_slab_bytes")
    return b.value


def jacobi_set_allocator(alloc_fn, free_fn, user=None) -> None:
    """Install C-callable alloc/free callbacks (ctypes ALLOC_FN / FREE_FN) or (None, None)."""
    _check(lib().jacobi_set_allocator(_c.cast(alloc_fn, _p) if alloc_fn else None,
                                      _c.cast(free_fn, _p) if free_fn else None, user), "jacobi_set_allocator")


_torch_blocks: dict = {}
_torch_cbs = None


def use_torch_allocator(enable: bool = True) -> None:
    """Let PyTorch own the device memory of handles created from now on: the library's slab
    buffers and control blocks become torch tensors from the CUDA caching allocator (kept alive
    here until the library frees them)."""
    global _torch_cbs
    if not enable:
        jacobi_set_allocator(None, None)
        return
    import torch

    def _alloc(nbytes, device, _user):
        try:
            t = torch.empty(int(nbytes), dtype=torch.uint8, device=f"cuda:{device}")
        except Exception:
            return None
        _torch_blocks[t.data_ptr()] = t
        return t.data_ptr()

    def _free(ptr, _device, _user):
        _torch_blocks.pop(ptr, None)

    _torch_cbs = (ALLOC_FN(_alloc), FREE_FN(_free))  # keep the thunks alive
    jacobi_set_allocator(*_torch_cbs)


# ---------------------------------------------------------------- convenience wrapper
class Jacobi:
    """One handle of the library.  shape = (nz, ny, nx) or (ny, nx) including the boundary."""

    def _init_shape(self, shape):
        shape = tuple(int(s) for s in shape)
        if len(shape) == 2:
            shape = (1,) + shape
        self.shape = shape
        nz, ny, nx = shape
        self.nx, self.ny, self.nz = nx, ny, nz
        self.stencil = 5 if nz == 1 else 7
        self.n = nx * ny * nz

    def __init__(self, shape, ngpus: int = 1, virtual: int = 0, device: int = 0, dist=None):
        self._init_shape(shape)
        nz, ny, nx = self.shape
        if dist is not None:
            rank, world = dist
            self.h = jacobi_create_rank(nx, ny, nz, self.stencil, world, rank, device)
        elif virtual:
            self.h = jacobi_create_virtual(nx, ny, nz, self.stencil, virtual, device)
        else:
            self.h = jacobi_create(nx, ny, nz, self.stencil, ngpus)
        self.local_slabs, self.total_slabs = jacobi_num_slabs(self.h)

    def run(self, iters: int) -> "Jacobi":
        jacobi_run(self.h, iters)
        return self

    def set_mode(self, mode: int, flags: int = 0) -> "Jacobi":
        jacobi_set_mode(self.h, mode, flags)
        return self

    def set_param(self, name: str, value: int) -> "Jacobi":
        jacobi_set_param(self.h, name, value)
        return self

    def get_param(self, name: str) -> int:
        return jacobi_get_param(self.h, name)

    def scatter(self, field: np.ndarray) -> "Jacobi":
        a = np.ascontiguousarray(field, dtype=np.float64)
        jacobi_scatter(self.h, a.reshape(-1), self.n)
        return self

    def gather(self, out: np.ndarray | None = None) -> np.ndarray:
        if out is None:
            out = np.empty(self.shape, dtype=np.float64)
        jacobi_gather(self.h, out.reshape(-1), self.n)
        return out if self.nz > 1 else out.reshape(self.ny, self.nx)

    def set_tolerance(self, tol: float, every: int) -> "Jacobi":
        """Convergence-terminated runs (N4): check the update norm every `every` iterations."""
        jacobi_set_tolerance(self.h, tol)
        jacobi_set_param(self.h, "norm_every", every)
        return self

    @property
    def last_norm(self) -> float:
        return jacobi_last_norm(self.h)

    def last_time_ms(self) -> float:
        return jacobi_last_time(self.h, self.local_slabs)[0]

    @property
    def iterations(self) -> int:
        return jacobi_iterations(self.h)

    def read_slab(self, i: int, parity: int) -> np.ndarray:
        """Raw slab buffer (chunk+2 planes incl. halos) as (planes, [ny,] pitch)."""
        d = self.describe(i)
        planes = d["chunk"] + 2
        out = np.empty(planes * d["plane_elems"], dtype=np.float64)
        _check(lib().jacobi_read_slab(self.h, i, parity, out.ctypes.data), "jacobi_read_slab")
        if self.nz > 1:
            return out.reshape(planes, self.ny, d["pitch"])
        return out.reshape(planes, d["pitch"])

    def describe(self, i: int = 0) -> dict:
        return jacobi_describe(self.h, i)

    def halo_trace(self, slab: int, n: int) -> np.ndarray:
        return jacobi_halo_trace(self.h, slab, n)

    def close(self) -> None:
        if getattr(self, "h", None):
            jacobi_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def create_nvshmem(shape, group=None, device: int = 0) -> "Jacobi":
    """N3: one NVSHMEM PE per rank of `group` (torch.distributed carries the unique id)."""
    import torch.distributed as dist

    use_nvshmem()
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = None
    if rank == 0:
        buf = _c.create_string_buffer(lib().jacobi_nvshmem_uid_bytes())
        _check(lib().jacobi_nvshmem_uid(buf), "jacobi_nvshmem_uid")
        uid = buf.raw
    uid = broadcast_blob(uid, group)
    j = Jacobi.__new__(Jacobi)
    j._init_shape(shape)
    h = _p()
    _check(lib().jacobi_create_nvshmem(j.nx, j.ny, j.nz, j.stencil, uid, world, rank, device, _c.byref(h)),
           "jacobi_create_nvshmem")
    j.h = h.value
    j.local_slabs, j.total_slabs = jacobi_num_slabs(j.h)
    return j


def nvshmem_finalize() -> None:
    lib().jacobi_nvshmem_finalize()


def exchange_blobs(blob: bytes, group=None):
    """All-gather one opaque blob per rank over torch.distributed; return (top, bottom): the
    blobs of ranks rank-1 and rank+1 (None at the ends of the slab chain)."""
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    blobs = [None] * world
    dist.all_gather_object(blobs, blob, group=group)
    top = blobs[rank - 1] if rank > 0 else None
    bot = blobs[rank + 1] if rank < world - 1 else None
    return top, bot


def broadcast_blob(blob_on_rank0, group=None):
    import torch.distributed as dist

    obj = [blob_on_rank0]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def all_blobs(blob: bytes, group=None) -> list:
    """All-gather one opaque blob per rank (rank order) over torch.distributed."""
    import torch.distributed as dist

    blobs = [None] * dist.get_world_size(group)
    dist.all_gather_object(blobs, blob, group=group)
    return blobs


def exchange_peers(j: Jacobi, group=None, nccl: bool = True) -> None:
    """Dist mode plumbing: all-gather every rank's IPC blob over torch.distributed, attach the
    neighbours and every rank's control block, and (optionally) set up the NCCL communicator of
    the baseline."""
    import torch.distributed as dist

    jacobi_open_ranks(j.h, all_blobs(jacobi_get_ipc_handle(j.h), group))
    if nccl:
        uid = broadcast_blob(jacobi_nccl_unique_id() if dist.get_rank(group) == 0 else None, group)
        jacobi_nccl_init(j.h, uid)
