// multiproc.cu — multi-process plumbing of the C ABI: CUDA IPC blobs (one process per GPU),
// NCCL communicators of the baseline, the caller device-memory allocator, and the NVSHMEM
// variant's creation (built only with -DJB_NVSHMEM).
#include "runtime_internal.h"

namespace jbrt {
NcclApi g_nccl;
Allocator g_alloc;
size_t alloc_offset(const void *p) {
  static PFN_getAddressRange fn = nullptr;
  if (!fn) {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess || !f) return 0;
    fn = reinterpret_cast<PFN_getAddressRange>(f);
  }
  unsigned long long base = 0;
  size_t size = 0;
  if (fn(&base, &size, (unsigned long long)p) != 0) return 0;
  return (size_t)((unsigned long long)p - base);
}
}  // namespace jbrt

extern "C" {
int jacobi_create_rank(int64_t nx, int64_t ny, int64_t nz, int stencil, int world_size, int rank,
                       int device, jacobi_t *out) {
  if (!out) return JACOBI_EINVAL;
  *out = nullptr;
  if (rank < 0 || rank >= world_size) return JACOBI_EINVAL;
  int rc = validate(nx, ny, nz, stencil, world_size);
  if (rc) return rc;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return JACOBI_ENODEV;
  jacobi_ctx *h = new_ctx(nx, ny, nz, stencil, world_size);
  h->kind = KIND_DIST;
  h->rank = rank;
  h->slabs.resize(1);
  Slab &s = h->slabs[0];
  s.device = device;
  s.id = rank;
  jbplan::decompose(h->n_out, world_size, rank, &s.start, &s.chunk);
  rc = alloc_slab(h, s);
  if (rc) { jacobi_destroy(h); return rc; }
  s.has_top = rank > 0;
  s.has_bot = rank < world_size - 1;
  h->peers_ready = world_size == 1;
  *out = h;
  return JACOBI_OK;
}

int jacobi_set_allocator(jacobi_alloc_fn alloc, jacobi_free_fn free_fn, void *user) {
  if ((alloc == nullptr) != (free_fn == nullptr)) return JACOBI_EINVAL;
  g_alloc.alloc = alloc;
  g_alloc.free = free_fn;
  g_alloc.user = user;
  return JACOBI_OK;
}

int jacobi_slab_bytes(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs, int slab, int64_t *bytes) {
  if (!bytes || slab < 0 || slab >= nslabs) return JACOBI_EINVAL;
  int rc = validate(nx, ny, nz, stencil, nslabs);
  if (rc) return rc;
  JbGeom g;
  if (jbplan::geometry(nx, ny, nz, stencil == 5 ? 2 : 3, 8, 1, JB_SMEM_DEFAULT, 0, &g)) return JACOBI_EINVAL;
  int64_t start, chunk;
  jbplan::decompose(stencil == 5 ? ny : nz, nslabs, slab, &start, &chunk);
  *bytes = jb_buf_doubles(chunk, g.dim, g.plane_elems) * (int64_t)sizeof(double);
  return JACOBI_OK;
}

int jacobi_ipc_handle_bytes(void) { return (int)sizeof(IpcBlob); }

int jacobi_get_ipc_handle(jacobi_t h, void *out) {
  if (!h || !out || h->kind != KIND_DIST) return JACOBI_EINVAL;
  Slab &s = h->slabs[0];
  IpcBlob b;
  std::memset(&b, 0, sizeof(b));
  b.magic = kIpcMagic;
  b.rank = h->rank;
  b.chunk = s.chunk;
  b.plane_elems = h->geom.plane_elems;
  CK(cudaDeviceGetAttribute(&b.sms, cudaDevAttrMultiProcessorCount, s.device));
  CK(cudaSetDevice(s.device));
  CK(cudaIpcGetMemHandle(&b.buf[0], s.buf[0]));
  CK(cudaIpcGetMemHandle(&b.buf[1], s.buf[1]));
  CK(cudaIpcGetMemHandle(&b.ctrl, s.ctrl));
  b.off[0] = alloc_offset(s.buf[0]);
  b.off[1] = alloc_offset(s.buf[1]);
  b.off[2] = alloc_offset(s.ctrl);
  std::memcpy(out, &b, sizeof(b));
  return JACOBI_OK;
}

int jacobi_open_peers(jacobi_t h, const void *top_blob, const void *bottom_blob) {
  if (!h || h->kind != KIND_DIST) return JACOBI_EINVAL;
  Slab &s = h->slabs[0];
  if ((s.has_top && !top_blob) || (s.has_bot && !bottom_blob)) return JACOBI_EINVAL;
  CK(cudaSetDevice(s.device));
  const int64_t pe = h->geom.plane_elems;
  auto open = [&](const void *blob, int expect_rank, double **bufs, JbCtrl **ctrl, int64_t *chunk) -> int {
    IpcBlob b;
    std::memcpy(&b, blob, sizeof(b));
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, s.device));
    if (b.magic != kIpcMagic || b.rank != expect_rank || b.plane_elems != pe || b.sms != sms) return JACOBI_EINVAL;
    for (int p = 0; p < 2; ++p) {
      void *ptr = nullptr;
      CK(cudaIpcOpenMemHandle(&ptr, b.buf[p], cudaIpcMemLazyEnablePeerAccess));
      s.ipc_opened.push_back(ptr);
      bufs[p] = reinterpret_cast<double *>(static_cast<char *>(ptr) + b.off[p]);
    }
    void *c = nullptr;
    CK(cudaIpcOpenMemHandle(&c, b.ctrl, cudaIpcMemLazyEnablePeerAccess));
    s.ipc_opened.push_back(c);
    *ctrl = reinterpret_cast<JbCtrl *>(static_cast<char *>(c) + b.off[2]);
    *chunk = b.chunk;
    return JACOBI_OK;
  };
  if (s.has_top) {
    double *bufs[2];
    JbCtrl *ctrl;
    int64_t chunk;
    int rc = open(top_blob, h->rank - 1, bufs, &ctrl, &chunk);
    if (rc) return rc;
    for (int p = 0; p < 2; ++p) s.peer_top[p] = bufs[p] + (chunk + 1) * pe;
    for (int p = 0; p < 2; ++p) s.ll_out_top[p] = jb_ll_area(bufs[p], chunk, h->dim, pe, 1);
    s.mid_top_out = bufs[1] + (chunk + 2) * pe;
    s.flag_out_top = &ctrl->flag_in[1][0];
  }
  if (s.has_bot) {
    double *bufs[2];
    JbCtrl *ctrl;
    int64_t chunk;
    int rc = open(bottom_blob, h->rank + 1, bufs, &ctrl, &chunk);
    if (rc) return rc;
    for (int p = 0; p < 2; ++p) s.peer_bot[p] = bufs[p];
    for (int p = 0; p < 2; ++p) s.ll_out_bot[p] = jb_ll_area(bufs[p], chunk, h->dim, pe, 0);
    s.mid_bot_out = bufs[0] + (chunk + 2) * pe;
    s.flag_out_bot = &ctrl->flag_in[0][0];
  }
  h->peers_ready = true;
  return JACOBI_OK;
}

int jacobi_open_ranks(jacobi_t h, const void *blobs, int world) {
  if (!h || !blobs || h->kind != KIND_DIST || world != h->total) return JACOBI_EINVAL;
  const size_t B = sizeof(IpcBlob);
  const char *base = static_cast<const char *>(blobs);
  const int r = h->rank;
  int rc = jacobi_open_peers(h, r > 0 ? base + (r - 1) * B : nullptr, r < world - 1 ? base + (r + 1) * B : nullptr);
  if (rc) return rc;
  Slab &s = h->slabs[0];
  CK(cudaSetDevice(s.device));
  h->all_ctrl.assign(world, nullptr);
  for (int g = 0; g < world; ++g) {
    if (g == r) {
      h->all_ctrl[g] = s.ctrl;
      continue;
    }
    IpcBlob b;
    std::memcpy(&b, base + g * B, B);
    if (b.magic != kIpcMagic || b.rank != g) return JACOBI_EINVAL;
    void *c = nullptr;
    CK(cudaIpcOpenMemHandle(&c, b.ctrl, cudaIpcMemLazyEnablePeerAccess));
    s.ipc_opened.push_back(c);
    h->all_ctrl[g] = reinterpret_cast<JbCtrl *>(static_cast<char *>(c) + b.off[2]);
  }
  return JACOBI_OK;
}

#ifdef JB_NVSHMEM
namespace {
bool g_shm_init = false;
void *shm_alloc(size_t bytes, int, void *) { return nvshmem_malloc(bytes); }
void shm_free(void *p, int, void *) { nvshmem_free(p); }
}  // namespace

int jacobi_nvshmem_uid_bytes(void) { return (int)sizeof(nvshmemx_uniqueid_t); }

int jacobi_nvshmem_uid(void *out) {
  if (!out) return JACOBI_EINVAL;
  nvshmemx_uniqueid_t uid = NVSHMEMX_UNIQUEID_INITIALIZER;
  if (nvshmemx_get_uniqueid(&uid) != 0) return JACOBI_ECUDA;
  std::memcpy(out, &uid, sizeof(uid));
  return JACOBI_OK;
}

// N3: one PE per process, bootstrapped from a unique id (created by rank 0, shared by the caller),
// slab buffers and control blocks on the NVSHMEM symmetric heap; halos are delivered with
// nvshmemx_putmem_signal_nbi_warp by the boundary CTAs of the CPU-Free kernel.
// Collective: every rank creates (and later destroys) its handle in the same order.
int jacobi_create_nvshmem(int64_t nx, int64_t ny, int64_t nz, int stencil, const void *uid, int world_size,
                          int rank, int device, jacobi_t *out) {
  if (!out || !uid || rank < 0 || rank >= world_size || world_size > 32) return JACOBI_EINVAL;
  *out = nullptr;
  int rc = validate(nx, ny, nz, stencil, world_size);
  if (rc) return rc;
  CK(cudaSetDevice(device));
  if (!g_shm_init) {
    if (!getenv("NVSHMEM_SYMMETRIC_SIZE")) {  // room for two field buffers + control block
      JbGeom g;
      jbplan::geometry(nx, ny, nz, stencil == 5 ? 2 : 3, 8, 1, JB_SMEM_DEFAULT, 0, &g);
      int64_t st, chunk_max;
      jbplan::decompose(stencil == 5 ? ny : nz, world_size, 0, &st, &chunk_max);
      const int64_t need = 2 * jb_buf_doubles(chunk_max, g.dim, g.plane_elems) * 8 + (64 << 20);
      const int64_t sz = std::max<int64_t>(need + need / 4, (int64_t)1 << 30);
      setenv("NVSHMEM_SYMMETRIC_SIZE", std::to_string(sz).c_str(), 0);
    }
    nvshmemx_uniqueid_t id;
    std::memcpy(&id, uid, sizeof(id));
    nvshmemx_init_attr_t attr = NVSHMEMX_INIT_ATTR_INITIALIZER;
    nvshmemx_set_attr_uniqueid_args(rank, world_size, &id, &attr);
    if (nvshmemx_init_attr(NVSHMEMX_INIT_WITH_UNIQUEID, &attr) != 0) return JACOBI_ECUDA;
    g_shm_init = true;
  }
  if (nvshmem_my_pe() != rank || nvshmem_n_pes() != world_size) return JACOBI_ESTATE;
  jacobi_ctx *h = new_ctx(nx, ny, nz, stencil, world_size);
  h->kind = KIND_SHMEM;
  h->rank = rank;
  h->alloc.alloc = shm_alloc;
  h->alloc.free = shm_free;
  h->alloc.user = nullptr;
  h->slabs.resize(1);
  Slab &s = h->slabs[0];
  s.device = device;
  s.id = rank;
  jbplan::decompose(h->n_out, world_size, rank, &s.start, &s.chunk);
  rc = alloc_slab(h, s);
  if (rc) { delete h; return rc; }
  const int64_t pe = h->geom.plane_elems;
  s.has_top = rank > 0;
  s.has_bot = rank < world_size - 1;
  if (s.has_top) {  // symmetric addresses of the neighbour's bottom halo plane and flag slots
    int64_t st, ct;
    jbplan::decompose(h->n_out, world_size, rank - 1, &st, &ct);
    for (int p = 0; p < 2; ++p) s.peer_top[p] = s.buf[p] + (ct + 1) * pe;
    s.flag_out_top = &s.ctrl->flag_in[1][0];
    s.shm_pe_top = rank - 1;
  }
  if (s.has_bot) {
    for (int p = 0; p < 2; ++p) s.peer_bot[p] = s.buf[p];
    s.flag_out_bot = &s.ctrl->flag_in[0][0];
    s.shm_pe_bot = rank + 1;
  }
  h->all_ctrl.assign(world_size, nullptr);  // raw NVLink pointers for the norm all-reduce (N4)
  for (int g = 0; g < world_size; ++g)
    h->all_ctrl[g] = static_cast<JbCtrl *>(nvshmem_ptr(s.ctrl, g));
  for (int g = 0; g < world_size; ++g)
    if (!h->all_ctrl[g]) h->all_ctrl.clear();
  h->peers_ready = true;
  nvshmem_barrier_all();
  *out = h;
  return JACOBI_OK;
}

int jacobi_nvshmem_finalize(void) {
  if (g_shm_init) nvshmem_finalize();
  g_shm_init = false;
  return JACOBI_OK;
}
#endif

int jacobi_nccl_unique_id(void *out128) {
  if (!out128) return JACOBI_EINVAL;
  if (!g_nccl.load()) return JACOBI_ENCCL;
  ncclUniqueId id;
  if (g_nccl.GetUniqueId(&id) != ncclSuccess) return JACOBI_ENCCL;
  std::memcpy(out128, &id, sizeof(id));
  return JACOBI_OK;
}

int jacobi_nccl_init(jacobi_t h, const void *id128) {
  if (!h || !id128 || h->kind != KIND_DIST) return JACOBI_EINVAL;
  if (!g_nccl.load()) return JACOBI_ENCCL;
  Slab &s = h->slabs[0];
  CK(cudaSetDevice(s.device));
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof(id));
  if (g_nccl.CommInitRank(&s.comm, h->total, id, h->rank) != ncclSuccess) return JACOBI_ENCCL;
  h->nccl_ready = true;
  return JACOBI_OK;
}
}  // extern "C"
