// runtime.cu — host runtime behind the C ABI in include/jacobi.h: slabs (HBM buffers + control
// blocks), planning (tiles, block split, schedules), the CPU-Free run, data movement.  The
// CPU-controlled baselines live in baselines.cu, multi-process plumbing in multiproc.cu.  All
// device work is done by the kernels in sweep.cu / resident.cu / util.cu.
#include "runtime_internal.h"

namespace jbrt {
int64_t slab_elems(const jacobi_ctx *h, const Slab &s) { return (s.chunk + 2) * h->geom.plane_elems; }

int validate(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs) {
  if (nx < 3 || ny < 3 || nslabs < 1) return JACOBI_EINVAL;
  if (!((stencil == 5 && nz == 1) || (stencil == 7 && nz >= 3))) return JACOBI_EINVAL;
  const int64_t n_out = stencil == 5 ? ny : nz;
  if (nslabs > 1 && (n_out - 2) / nslabs < 2) return JACOBI_EINVAL;  // every chunk >= 2 planes
  if (nslabs > 1 && nx + 3 > (int64_t)1 << 40) return JACOBI_EINVAL;
  return JACOBI_OK;
}

jacobi_ctx *new_ctx(int64_t nx, int64_t ny, int64_t nz, int stencil, int total) {
  jacobi_ctx *h = new jacobi_ctx();
  h->nx = nx; h->ny = ny; h->nz = nz; h->stencil = stencil;
  h->dim = stencil == 5 ? 2 : 3;
  h->n_out = h->dim == 2 ? ny : nz;
  h->total = total;
  h->alloc = g_alloc;
  JbGeom g;
  // Layout only depends on pitch / plane_elems; tile parameters are re-planned per launch.
  jbplan::geometry(nx, ny, nz, h->dim, 8, 1, JB_SMEM_DEFAULT, 0, &g);
  h->geom = g;
  return h;
}

int alloc_slab(jacobi_ctx *h, Slab &s) {
  CK(cudaSetDevice(s.device));
  // (chunk + 2) planes of the slab + jb_edge_planes(h->dim) scratch planes (time-blocked edge zones)
  size_t bytes = (size_t)jb_buf_doubles(s.chunk, h->dim, h->geom.plane_elems) * sizeof(double);
  if (h->kind == KIND_SHMEM) {  // symmetric heap: every PE allocates the largest slab
    int64_t st, chunk_max;
    jbplan::decompose(h->n_out, h->total, 0, &st, &chunk_max);
    bytes = (size_t)jb_buf_doubles(chunk_max, h->dim, h->geom.plane_elems) * sizeof(double);
  }
  if (h->alloc.alloc) {
    s.buf[0] = static_cast<double *>(h->alloc.alloc(bytes, s.device, h->alloc.user));
    s.buf[1] = static_cast<double *>(h->alloc.alloc(bytes, s.device, h->alloc.user));
    s.ctrl = static_cast<JbCtrl *>(h->alloc.alloc(sizeof(JbCtrl), s.device, h->alloc.user));
    if (!s.buf[0] || !s.buf[1] || !s.ctrl) return JACOBI_ENOMEM;
    CK(cudaSetDevice(s.device));  // the callback may have switched devices
    for (const void *p : {(const void *)s.buf[0], (const void *)s.buf[1], (const void *)s.ctrl})
      if ((uintptr_t)p % 16) return JACOBI_EINVAL;  // bulk copies and 16-byte stores need alignment
  } else {
    CK(cudaMalloc(&s.buf[0], bytes));
    CK(cudaMalloc(&s.buf[1], bytes));
    CK(cudaMalloc(&s.ctrl, sizeof(JbCtrl)));
  }
  CK(cudaMemset(s.ctrl, 0, sizeof(JbCtrl)));
  CK(cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s.stream2, cudaStreamNonBlocking));
  CK(cudaEventCreate(&s.ev0));
  CK(cudaEventCreate(&s.ev1));
  CK(cudaEventCreateWithFlags(&s.ev_sync, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&s.ev_copy, cudaEventDisableTiming));
  // Deterministic U12 initial field, both buffers, padding = 0.
  CK(jbk::launch_init(s.buf[0], s.buf[1], s.chunk + 2, h->geom, s.start - 1, kSeedBench, s.stream));
  CK(cudaStreamSynchronize(s.stream));
  return JACOBI_OK;
}

void free_slab(Slab &s, const Allocator &a) {
  cudaSetDevice(s.device);
  if (s.comm && g_nccl.CommDestroy) g_nccl.CommDestroy(s.comm);
  for (void *p : s.ipc_opened) cudaIpcCloseMemHandle(p);
  s.ipc_opened.clear();
  for (void *p : {(void *)s.buf[0], (void *)s.buf[1], (void *)s.ctrl}) {
    if (!p) continue;
    if (a.free) a.free(p, s.device, a.user);
    else if (!a.alloc) cudaFree(p);
  }
  for (auto &t : s.tabs)
    if (t.ptr) cudaFree(t.ptr);
  if (s.blk_flags) cudaFree(s.blk_flags);
  if (s.partials) cudaFree(s.partials);
  if (s.norm_peers) cudaFree(s.norm_peers);
  if (s.tmap) cudaFree(s.tmap);
  if (s.trace) cudaFree(s.trace);
  if (s.bar_flags) cudaFree(s.bar_flags);
  if (s.ev0) cudaEventDestroy(s.ev0);
  if (s.ev1) cudaEventDestroy(s.ev1);
  if (s.ev_sync) cudaEventDestroy(s.ev_sync);
  if (s.ev_copy) cudaEventDestroy(s.ev_copy);
  if (s.stream2) cudaStreamDestroy(s.stream2);
  if (s.stream) cudaStreamDestroy(s.stream);
  s = Slab();
}

// Link slabs that live in this process (single / virtual mode).
void link_local(jacobi_ctx *h) {
  const int64_t pe = h->geom.plane_elems;
  const int n = (int)h->slabs.size();
  for (int i = 0; i < n; ++i) {
    Slab &s = h->slabs[i];
    s.has_top = i > 0;
    s.has_bot = i < n - 1;
    if (s.has_top) {
      Slab &o = h->slabs[i - 1];
      for (int p = 0; p < 2; ++p) s.peer_top[p] = o.buf[p] + (o.chunk + 1) * pe;
      for (int p = 0; p < 2; ++p) s.ll_out_top[p] = jb_ll_area(o.buf[p], o.chunk, h->dim, pe, 1);
      s.mid_top_out = o.buf[1] + (o.chunk + 2) * pe;  // its E_bot (slot 0)
      s.flag_out_top = &o.ctrl->flag_in[1][0];
      s.peer_top_dev = o.device;
    }
    if (s.has_bot) {
      Slab &o = h->slabs[i + 1];
      for (int p = 0; p < 2; ++p) s.peer_bot[p] = o.buf[p];
      for (int p = 0; p < 2; ++p) s.ll_out_bot[p] = jb_ll_area(o.buf[p], o.chunk, h->dim, pe, 0);
      s.mid_bot_out = o.buf[0] + (o.chunk + 2) * pe;  // its E_top (slot 0)
      s.flag_out_bot = &o.ctrl->flag_in[0][0];
      s.peer_bot_dev = o.device;
    }
  }
  h->peers_ready = true;
}

// Tensor maps (TMA descriptors) of a slab's two buffers, viewed as [planes][ny][pitch] fp64, box
// = one plane's `rows` x `cols` window; out-of-bounds elements are zero-filled (they only feed
// Dirichlet / discarded cells).  Encoded with the driver's cuTensorMapEncodeTiled (entry point
// via the runtime, no -lcuda) and kept in device memory for the kernel.
int slab_tensor_maps(jacobi_ctx *h, Slab &s, int cols, int rows) {
  if (s.tmap && s.tmap_key[0] == cols && s.tmap_key[1] == rows) return JACOBI_OK;
  using EncodeFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  static EncodeFn encode = nullptr;
  if (!encode) {
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess) return JACOBI_ECUDA;
    encode = reinterpret_cast<EncodeFn>(fn);
  }
  const JbGeom &g = h->geom;
  const int64_t planes = s.chunk + 2 + jb_edge_planes(h->dim);
  CUtensorMap maps[2];
  for (int b = 0; b < 2; ++b) {
    const cuuint64_t dims[3] = {(cuuint64_t)g.pitch, (cuuint64_t)h->ny, (cuuint64_t)planes};
    const cuuint64_t strides[2] = {(cuuint64_t)g.pitch * 8, (cuuint64_t)g.plane_elems * 8};
    const cuuint32_t box[3] = {(cuuint32_t)cols, (cuuint32_t)rows, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    const CUresult r = encode(&maps[b], CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, s.buf[b], dims, strides, box, estr,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return JACOBI_ECUDA;
  }
  CK(cudaSetDevice(s.device));
  if (!s.tmap) CK(cudaMalloc(&s.tmap, sizeof(maps)));
  CK(cudaMemcpy(s.tmap, maps, sizeof(maps), cudaMemcpyHostToDevice));
  s.tmap_key[0] = cols;
  s.tmap_key[1] = rows;
  return JACOBI_OK;
}

// Device copy of the guided-schedule block table of a slab.  Two cached entries (LRU): a
// time-blocked run plans the per-iteration launch too, so the two tables alternate within every
// jacobi_run; rebuilding them each time cost a cudaFree (an implicit device sync) + cudaMalloc
// per run.  An evicted entry's allocation is reused when it is large enough.
int upload_table(Slab &s, int64_t npl, int units, int n, int min_blk, int64_t nb) {
  const int64_t key[4] = {npl, units, n, min_blk};
  ++s.tab_clock;
  for (auto &t : s.tabs)
    if (t.ptr && std::memcmp(key, t.key, sizeof(key)) == 0) {
      t.used = s.tab_clock;
      s.dyn_table = t.ptr;
      return JACOBI_OK;
    }
  auto &t = s.tabs[0].used <= s.tabs[1].used ? s.tabs[0] : s.tabs[1];
  std::vector<int32_t> tab(nb + 1);
  jbplan::dyn_blocks(npl, units, n, min_blk, tab.data());
  if (t.cap < nb + 1) {
    if (t.ptr) cudaFree(t.ptr);
    t.ptr = nullptr;
    t.cap = 0;
    CK(cudaMalloc(&t.ptr, tab.size() * sizeof(int32_t)));
    t.cap = nb + 1;
  }
  CK(cudaMemcpy(t.ptr, tab.data(), tab.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
  std::memcpy(t.key, key, sizeof(key));
  t.used = s.tab_clock;
  s.dyn_table = t.ptr;
  return JACOBI_OK;
}

// CTAs of one launch on a GPU with `sms` SMs (all slabs of a virtual group share it).
int launch_ctas(const jacobi_ctx *h, int sms) {
  int total = sms;
  const int nslab = h->kind == KIND_VIRTUAL ? h->total : 1;
  if (h->ctas > 0) total = (int)std::min<int64_t>(h->ctas * nslab, sms);
  return total;
}

// Interior cells of the whole grid per CTA of the whole job (every slab's CTAs on every GPU):
// the same number on every rank, so the policies below agree across processes.
int64_t cells_per_cta(const jacobi_ctx *h, int sms) {
  const int64_t devices = h->kind == KIND_VIRTUAL ? 1 : h->total;
  return jbplan::cells_per_cta(h->nx, h->ny, h->nz, h->dim, (int64_t)launch_ctas(h, sms) * devices);
}

// Interior schedule of the per-iteration kernel: knob "schedule" 0 / 1 static, 2 dynamic; auto
// (-1): dynamic guided self-scheduling for large grids (it absorbs the B200's per-SM speed spread
// on HBM-bound sweeps: C2 / C3 0.93-0.99 of copy), static linear for grids of < JB_DYN_MIN_CELLS
// interior cells per CTA, whose L2-resident iterations are latency-bound and where every claim
// (an atomic plus the block-table reads) sits on the critical path: 3D 128^3 18.0 -> 12.5 us,
// 2D 2048^2 with 2-8 virtual slabs 15.7 -> 11.1-12.2 us per iteration.
bool schedule_dynamic(const jacobi_ctx *h, int sms) {
  if (h->schedule >= 0) return h->schedule == 2;
  return jbplan::schedule_dynamic_auto(cells_per_cta(h, sms));
}

// CTAs of slab `id` in its CPU-Free launch.
int slab_ctas(const jacobi_ctx *h, int id, int sms) {
  const int total = launch_ctas(h, sms);
  if (h->kind != KIND_VIRTUAL) return total;
  return total / h->total + (id < total % h->total ? 1 : 0);
}

// Boundary / interior split of a slab's CTAs (reconstructed P:398-404; R11).
void split_roles(const jacobi_ctx *h, int sms, int count, int64_t inner, bool top, bool bot, int units, int *nt,
                 int *nb, int *ni) {
  const bool dynamic = schedule_dynamic(h, sms);
  const bool nocomp = (h->flags & JACOBI_FLAG_NO_COMPUTE) != 0;
  int override_ps = (int)h->boundary_ctas;
  if (override_ps <= 0 && ((dynamic && h->dyn_help) || nocomp) && inner > 0 && (top || bot)) {
    // Boundary CTAs join the dynamic interior after signalling (or, without compute, the
    // interior has nothing to do), so give every boundary unit its own CTA (shortest halo
    // critical path), up to a quarter of the grid per side.
    override_ps = (int)std::max<int64_t>(1, std::min<int64_t>(units, count / 4));
  }
  override_ps = std::min(override_ps, JB_MAXK);
  jbplan::tb_split(count, inner, top, bot, units, override_ps, nt, nb, ni);
  *nt = std::min(*nt, JB_MAXK);
  *nb = std::min(*nb, JB_MAXK);
  *ni = count - *nt - *nb;
}

// The CPU-Free split of slab `id` as that slab computes it (same inputs, same function).
void neighbour_roles(const jacobi_ctx *h, int id, int sms, int units, int *nt_out, int *nb_out) {
  int64_t start, chunk;
  jbplan::decompose(h->n_out, h->total, id, &start, &chunk);
  const bool top = id > 0, bot = id < h->total - 1;
  const int64_t inner = (bot ? chunk - 1 : chunk) - (top ? 2 : 1) + 1;
  int nt, nb, ni;
  split_roles(h, sms, slab_ctas(h, id, sms), inner, top, bot, units, &nt, &nb, &ni);
  if (nt_out) *nt_out = nt;
  if (nb_out) *nb_out = nb;
}



// Plan one launch on one device over the local slabs `idx` (1 slab per GPU, or all slabs in
// virtual mode).  persist=false plans the discrete baseline kernel (no boundary roles).


// JB_PFLAG_GPU_SCOPE when every slab of the launch lives on one GPU in this process (virtual
// slabs): the halo flags then need only .gpu scope (knob flag_scope).
static int flag_scope_bits(const jacobi_ctx *h) {
  const bool gpu = h->kind == KIND_VIRTUAL && h->flag_scope != 0;
  return gpu ? JB_PFLAG_GPU_SCOPE : 0;
}

int plan_launch(jacobi_ctx *h, const std::vector<int> &idx, LaunchKind lk, bool nocomp, LaunchPlan &L,
                int grid_override) {
  const bool persist = lk == LK_PERSIST;
  Slab &s0 = h->slabs[idx[0]];
  L.device = s0.device;
  L.stream = s0.stream;
  L.slab_idx = idx;
  CK(cudaSetDevice(s0.device));
  int sms = 0, smem_optin = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, s0.device));
  CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, s0.device));
  smem_optin = std::min(smem_optin, JB_SMEM_DEFAULT) - 1024;  // static smem + reserve

  JbGeom g;
  // First pass with the default ty to learn units_x / stage size.
  if (jbplan::geometry(h->nx, h->ny, h->nz, h->dim, (int)h->tile_x, (int)h->tile_y, smem_optin,
                       (int)h->stages, &g))
    return JACOBI_EINVAL;
  const int nslab = (int)idx.size();
  int total_ctas = launch_ctas(h, sms);  // one CTA per SM (occupancy verified below)
  if (grid_override > 0) total_ctas = std::min(grid_override, lk == LK_PERSIST ? 2 * sms : sms);
  const int per = total_ctas / nslab;
  if (h->dim == 3 && h->tile_y <= 0) {
    // Pick ty so that the tile count divides the CTA count well: a whole number of plane blocks
    // per scheduling round keeps neighbouring tiles on the same planes, so their y-halo rows
    // are L2 hits (measured C3: ty=7 -> 73 tiles, 2 per round of 148 CTAs, 0.97 of copy BW).
    // Small (latency-bound) slabs prefer the tallest tile: fewer, larger items.
    const int64_t planes_per_cta = (h->ny - 2) * (h->n_out - 2) / std::max<int64_t>(1, h->total) / per;
    const bool small = planes_per_cta < 64 * 8;  // (rows x planes) per CTA below 64 planes of ty=8 tiles
    int ty = (h->schedule == 0 || small) ? jbplan::tallest_ty(h->ny, smem_optin, g.ws)
                                         : jbplan::choose_ty(h->ny, g.units_x, per, smem_optin, g.ws);
    if (jbplan::geometry(h->nx, h->ny, h->nz, h->dim, (int)h->tile_x, ty, smem_optin, (int)h->stages, &g))
      return JACOBI_EINVAL;
  }
  g.l2hint = (int32_t)(h->l2hint < 0 ? 0 : h->l2hint);
  L.smem = jbplan::smem_bytes(g);
  CK(jbk::prepare(h->dim, nocomp, persist, L.smem));
  int occ = 0;
  CK(jbk::occupancy(h->dim, nocomp, persist, L.smem, &occ));
  if (occ < 1) return JACOBI_ENOCOOP;
  L.grid = total_ctas;

  JbParams &P = L.P;
  std::memset(&P, 0, sizeof(P));
  P.g = g;
  P.nslabs = nslab;
  P.flags = h->flags | flag_scope_bits(h);
  P.timeout_ns = (unsigned long long)h->timeout_ms * 1000000ull;
  P.status = s0.ctrl->status;
  int begin = 0;
  for (int k = 0; k < nslab; ++k) {
    Slab &s = h->slabs[idx[k]];
    JbSlab &d = P.s[k];
    const int count = per + (k < total_ctas % nslab ? 1 : 0);
    d.buf[0] = s.buf[0]; d.buf[1] = s.buf[1];
    d.peer_top[0] = s.peer_top[0]; d.peer_top[1] = s.peer_top[1];
    d.peer_bot[0] = s.peer_bot[0]; d.peer_bot[1] = s.peer_bot[1];
    d.flag_in_top = &s.ctrl->flag_in[0][0];
    d.flag_in_bot = &s.ctrl->flag_in[1][0];
    d.flag_out_top = s.flag_out_top;
    d.flag_out_bot = s.flag_out_bot;
    d.side_ctr = s.ctrl->side_ctr;
    d.barrier = &s.ctrl->barrier;
    d.chunk = s.chunk;
    d.cta_begin = begin;
    d.cta_count = count;
    d.slab_id = s.id;
    d.use_shm = h->kind == KIND_SHMEM ? 1 : 0;
    d.shm_pe_top = s.shm_pe_top;
    d.shm_pe_bot = s.shm_pe_bot;
    begin += count;
    const bool roles = lk == LK_PERSIST || lk == LK_P2P || lk == LK_EDGES;
    const bool top = roles && s.has_top, bot = roles && s.has_bot;
    if (lk == LK_EDGES) {  // boundary planes only: CTAs split between the sides, no interior
      d.peer_top[0] = d.peer_top[1] = d.peer_bot[0] = d.peer_bot[1] = nullptr;
      const int sides = (top ? 1 : 0) + (bot ? 1 : 0);
      d.n_top = top ? std::max(1, count / std::max(sides, 1)) : 0;
      d.n_bot = bot ? count - d.n_top : 0;
      d.cta_count = d.n_top + d.n_bot;
      d.work_ctr = s.ctrl->work;
      s.desc = d;
      s.grid = d.cta_count;
      s.smem = L.smem;
      continue;
    }
    if (lk == LK_INNER) {
      d.excl_top = s.has_top ? 1 : 0;
      d.excl_bot = s.has_bot ? 1 : 0;
    }
    const int64_t lo = (top || d.excl_top) ? 2 : 1, hi = (bot || d.excl_bot) ? s.chunk - 1 : s.chunk;
    const int64_t inner = hi - lo + 1;
    int nt, nb, ni;
    if (count < (top ? 1 : 0) + (bot ? 1 : 0) + (inner > 0 ? 1 : 0)) return JACOBI_ENOCOOP;
    const bool dynamic = schedule_dynamic(h, sms);
    split_roles(h, sms, count, inner, top, bot, g.units, &nt, &nb, &ni);
    d.n_top = nt;
    d.n_bot = nb;
    if (persist || lk == LK_P2P) {
      // The facing boundary-CTA counts of the neighbours (how many flag slots to wait for) are
      // recomputed here with the neighbours' own chunk and CTA count: the split is deterministic.
      int kt = 0, kb = 0;
      if (s.has_top) neighbour_roles(h, s.id - 1, sms, g.units, nullptr, &kt);
      if (s.has_bot) neighbour_roles(h, s.id + 1, sms, g.units, &kb, nullptr);
      d.k_in_top = kt;
      d.k_in_bot = kb;
      if (kt > JB_MAXK || kb > JB_MAXK || nt > JB_MAXK || nb > JB_MAXK) return JACOBI_EINVAL;
    }
    const bool lockstep = h->schedule == 1;
    d.k_planes = lockstep ? jbplan::lockstep_k(g.units, ni, inner) : 0;
    d.work_ctr = s.ctrl->work;
    if (dynamic && inner > 0) {
      // Guided self-scheduling over every CTA of the slab (boundary CTAs join after signalling).
      d.dyn_min_blk = (int)std::max<int64_t>(1, h->min_block);
      d.dyn_help = (h->dyn_help != 0) ? 1 : 0;
      d.dyn_n = d.dyn_help ? count : ni;
      const int64_t nblk = jbplan::dyn_blocks(inner, g.units, d.dyn_n, d.dyn_min_blk);
      d.dyn_items = (int64_t)g.units * nblk;
      d.dyn_first = (int)std::min<int64_t>(ni, d.dyn_items);
      int rc = upload_table(s, inner, g.units, d.dyn_n, d.dyn_min_blk, nblk);
      if (rc) return rc;
      d.dyn_table = s.dyn_table;
    }
    s.desc = d;
    s.grid = count;
    s.smem = L.smem;
  }
  return JACOBI_OK;
}

// Zero the per-run counters of a slab: barrier, side counters, status, claim counters.
cudaError_t reset_run_counters(Slab &s, cudaStream_t st) {
  static_assert(offsetof(JbCtrl, work) + sizeof(JbCtrl::work) - offsetof(JbCtrl, barrier) == 32,
                "JbCtrl per-run counters must be contiguous");
  return cudaMemsetAsync(&s.ctrl->barrier, 0, 32, st);
}

int read_status(Slab &s) {
  int st[2] = {0, 0};
  CK(cudaSetDevice(s.device));
  CK(cudaMemcpy(st, s.ctrl->status, sizeof(st), cudaMemcpyDeviceToHost));
  return st[0] ? st[0] : JACOBI_OK;
}

// Launch groups of this context: one launch per device slab, or one for all (virtual).
std::vector<std::vector<int>> launch_groups(jacobi_ctx *h) {
  std::vector<std::vector<int>> groups;
  if (h->kind == KIND_VIRTUAL) {
    std::vector<int> all;
    for (int i = 0; i < (int)h->slabs.size(); ++i) all.push_back(i);
    groups.push_back(all);
  } else {
    for (int i = 0; i < (int)h->slabs.size(); ++i) groups.push_back({i});
  }
  return groups;
}

// Plan a resident (on-chip) launch over the slabs `idx` of one device.
// Returns JACOBI_OK, or JACOBI_EINVAL when some slab does not fit on chip.
int plan_resident(jacobi_ctx *h, const std::vector<int> &idx, LaunchPlan &L) {
  Slab &s0 = h->slabs[idx[0]];
  L.device = s0.device;
  L.stream = s0.stream;
  L.slab_idx = idx;
  CK(cudaSetDevice(s0.device));
  int sms = 0, smem_optin = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, s0.device));
  CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, s0.device));
  smem_optin = std::min(smem_optin, JB_SMEM_DEFAULT) - 1024;
  JbParams &P = L.P;
  std::memset(&P, 0, sizeof(P));
  if (jbplan::geometry(h->nx, h->ny, h->nz, h->dim, 8, 1, JB_SMEM_DEFAULT, 0, &P.g)) return JACOBI_EINVAL;
  P.g.res_rs = (int)((h->nx + 2) / 2 * 2);  // round_up(nx + 1, 2)
  if ((h->slabs[idx[0]].chunk + 3) * P.g.plane_elems >= ((int64_t)1 << 31)) return JACOBI_EINVAL;
  P.nslabs = (int)idx.size();
  P.flags = h->flags | flag_scope_bits(h);
  P.timeout_ns = (unsigned long long)h->timeout_ms * 1000000ull;
  P.status = s0.ctrl->status;
  auto tiling = [&](int id, int *nbz, int *nby, int *cpp, size_t *sm) {
    int64_t st, ch;
    jbplan::decompose(h->n_out, h->total, id, &st, &ch);
    return jbplan::resident_tiling(h->nx, h->ny, h->dim, ch, slab_ctas(h, id, sms), smem_optin, nbz, nby, cpp, sm);
  };
  int cpp_max = 1, begin = 0;
  size_t smem = 0;
  for (size_t k = 0; k < idx.size(); ++k) {
    Slab &s = h->slabs[idx[k]];
    JbSlab &d = P.s[k];
    int nbz, nby, cpp;
    size_t sm;
    if (tiling(s.id, &nbz, &nby, &cpp, &sm)) return JACOBI_EINVAL;
    cpp_max = std::max(cpp_max, cpp);
    smem = std::max(smem, sm);
    d.buf[0] = s.buf[0]; d.buf[1] = s.buf[1];
    d.peer_top[0] = s.peer_top[0]; d.peer_top[1] = s.peer_top[1];
    d.peer_bot[0] = s.peer_bot[0]; d.peer_bot[1] = s.peer_bot[1];
    d.flag_in_top = &s.ctrl->flag_in[0][0];
    d.flag_in_bot = &s.ctrl->flag_in[1][0];
    d.flag_out_top = s.flag_out_top;
    d.flag_out_bot = s.flag_out_bot;
    d.barrier = &s.ctrl->barrier;
    d.chunk = s.chunk;
    d.slab_id = s.id;
    d.res_nbz = nbz;
    d.res_nby = nby;
    d.res_relaxed = h->block_sync == 0 ? 0 : 1;
    if (d.res_relaxed) {
      if (nbz * nby > JB_MAX_BLOCKS) return JACOBI_EINVAL;
      if (!s.blk_flags) {
        CK(cudaMalloc(&s.blk_flags, JB_MAX_BLOCKS * sizeof(unsigned long long)));
        CK(cudaMemset(s.blk_flags, 0, JB_MAX_BLOCKS * sizeof(unsigned long long)));
      }
      d.blk_flags = s.blk_flags;
    }
    d.cta_begin = begin;
    d.cta_count = nbz * nby;
    begin += d.cta_count;
    // facing boundary blocks of the neighbours = their nby (one flag slot per boundary block)
    int nz2, ny2, c2;
    size_t sm2;
    d.k_in_top = (s.has_top && !tiling(s.id - 1, &nz2, &ny2, &c2, &sm2)) ? ny2 : 0;
    d.k_in_bot = (s.has_bot && !tiling(s.id + 1, &nz2, &ny2, &c2, &sm2)) ? ny2 : 0;
    if ((s.has_top && d.k_in_top == 0) || (s.has_bot && d.k_in_bot == 0)) return JACOBI_EINVAL;
    s.desc = d;
    s.grid = d.cta_count;
    s.smem = smem;
  }
  int occ = 0;
  CK(jbk::prepare_resident(h->dim, cpp_max, smem, &occ));
  if (occ < 1 || begin > sms * occ) return JACOBI_EINVAL;
  L.grid = begin;
  L.smem = smem;
  L.cpp = cpp_max;
  return JACOBI_OK;
}

// Whether EVERY slab of the run (all ids 0..total-1, not only this process's) fits the resident
// kernel.  One process per GPU decides on its own, so the choice must be a deterministic function
// of the global problem: a rank picking the resident kernel while its neighbour streams would
// disagree on the flag slots and their meaning (per iteration vs per phase).  Same inputs as
// plan_resident (decompose, resident_tiling with the slab's CTA count, the 2^31 element limit,
// occupancy of the chosen variant); ranks run on equal GPUs (SM count checked in the IPC blob).
bool resident_fits_all(jacobi_ctx *h) {
  const int dev = h->slabs[0].device;
  if (cudaSetDevice(dev) != cudaSuccess) return false;
  int sms = 0, smem_optin = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return false;
  if (cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) return false;
  smem_optin = std::min(smem_optin, JB_SMEM_DEFAULT) - 1024;
  int64_t group_ctas = 0;
  for (int id = 0; id < h->total; ++id) {
    int64_t st, ch;
    jbplan::decompose(h->n_out, h->total, id, &st, &ch);
    if ((ch + 3) * h->geom.plane_elems >= ((int64_t)1 << 31)) return false;
    int nbz, nby, cpp;
    size_t sm;
    if (jbplan::resident_tiling(h->nx, h->ny, h->dim, ch, slab_ctas(h, id, sms), smem_optin, &nbz, &nby, &cpp, &sm))
      return false;
    int occ = 0;
    if (jbk::prepare_resident(h->dim, cpp, sm, &occ) != cudaSuccess || occ < 1) return false;
    if (h->block_sync && nbz * nby > JB_MAX_BLOCKS) return false;
    group_ctas = h->kind == KIND_VIRTUAL ? group_ctas + nbz * nby : nbz * nby;
    if (group_ctas > (int64_t)sms * occ) return false;
  }
  return true;
}

// N4: wire the residual-norm all-reduce into a planned launch (partials + every slab's ctrl).
int setup_norm(jacobi_ctx *h, LaunchPlan &L) {
  if (h->total > 32) return JACOBI_EINVAL;  // one polling lane per slab
  // every slab stores its sum into every other slab's control block: all pairs must be mapped
  if (h->kind == KIND_SINGLE && !h->all_peers) return JACOBI_ENOPEER;
  for (size_t k = 0; k < L.slab_idx.size(); ++k) {
    Slab &s = h->slabs[L.slab_idx[k]];
    JbSlab &d = L.P.s[k];
    const int64_t n = d.dyn_items + 2 * (int64_t)L.P.g.units;
    if (n > s.partials_cap) {
      if (s.partials) cudaFree(s.partials);
      s.partials = nullptr;
      CK(cudaMalloc(&s.partials, n * sizeof(double)));
      s.partials_cap = n;
    }
    CK(cudaMemset(s.partials, 0, n * sizeof(double)));
    std::vector<JbCtrl *> ctrls(h->total, nullptr);
    if (h->kind == KIND_DIST || h->kind == KIND_SHMEM) {
      if ((int)h->all_ctrl.size() != h->total) return JACOBI_ESTATE;  // needs jacobi_open_ranks
      ctrls = h->all_ctrl;
    } else {
      for (auto &o : h->slabs) ctrls[o.id] = o.ctrl;
    }
    ctrls[s.id] = s.ctrl;
    if (!s.norm_peers) CK(cudaMalloc(&s.norm_peers, JB_MAX_NORM * sizeof(JbCtrl *)));
    CK(cudaMemcpy(s.norm_peers, ctrls.data(), h->total * sizeof(JbCtrl *), cudaMemcpyHostToDevice));
    d.partials = s.partials;
    d.norm_peers = s.norm_peers;
    d.n_partials = (int32_t)n;
    d.norm_slabs = h->total;
  }
  L.P.norm_every = (int32_t)h->norm_every;
  L.P.tol = h->tol;
  L.P.k0 = h->norm_checks;
  return JACOBI_OK;
}

// Halo-exchange trace (param halo_trace = n): a zeroed per-slab buffer of 2 sides x n exchanges
// x 3 timestamps, wired into a planned CPU-Free launch (streaming, resident or time-blocked).
int setup_trace(jacobi_ctx *h, LaunchPlan &L) {
  const int64_t n = h->halo_trace;
  L.P.halo_trace_n = (int32_t)n;
  for (size_t k = 0; k < L.slab_idx.size(); ++k) {
    Slab &s = h->slabs[L.slab_idx[k]];
    L.P.s[k].halo_trace = nullptr;
    if (n <= 0) continue;
    CK(cudaSetDevice(s.device));
    if (s.trace_cap < n) {
      if (s.trace) cudaFree(s.trace);
      s.trace = nullptr;
      s.trace_cap = 0;
      CK(cudaMalloc(&s.trace, (size_t)n * 6 * sizeof(unsigned long long)));
      s.trace_cap = n;
    }
    CK(cudaMemsetAsync(s.trace, 0, (size_t)n * 6 * sizeof(unsigned long long), L.stream));
    s.trace_n = n;
    L.P.s[k].halo_trace = s.trace;
  }
  // grid-barrier form (knob "barrier"): per-CTA arrival flags, allocated once and zeroed; their
  // epochs (global iteration counts) only grow, so stale slots never satisfy a later barrier
  for (size_t k = 0; k < L.slab_idx.size(); ++k) {
    Slab &s = h->slabs[L.slab_idx[k]];
    L.P.s[k].bar_flags = nullptr;
    if (h->barrier != 1) continue;
    if (L.P.s[k].cta_count > JB_MAX_BLOCKS) return JACOBI_EINVAL;
    CK(cudaSetDevice(s.device));
    if (!s.bar_flags) {
      CK(cudaMalloc(&s.bar_flags, JB_MAX_BLOCKS * sizeof(unsigned long long)));
      CK(cudaMemset(s.bar_flags, 0, JB_MAX_BLOCKS * sizeof(unsigned long long)));
    }
    L.P.s[k].bar_flags = s.bar_flags;
  }
  return JACOBI_OK;
}

// LL halo protocol (knob "halo_ll") for a streaming CPU-Free launch: the
// receive areas of this launch's slabs and the neighbours' (set at link time); null = flags.
bool ll_enabled(const jacobi_ctx *h) {
  if (h->kind == KIND_SHMEM || h->halo_ll == 0) return false;
  return h->halo_ll > 0 || JB_LL_AUTO;
}
void setup_ll(jacobi_ctx *h, LaunchPlan &L) {
  const bool on = ll_enabled(h);
  const int64_t pe = h->geom.plane_elems;
  for (size_t k = 0; k < L.slab_idx.size(); ++k) {
    Slab &s = h->slabs[L.slab_idx[k]];
    JbSlab &d = L.P.s[k];
    for (int p = 0; p < 2; ++p) {
      d.ll_out_top[p] = on && s.has_top ? s.ll_out_top[p] : nullptr;
      d.ll_out_bot[p] = on && s.has_bot ? s.ll_out_bot[p] : nullptr;
      d.ll_in_top[p] = on && s.has_top ? jb_ll_area(s.buf[p], s.chunk, h->dim, pe, 0) : nullptr;
      d.ll_in_bot[p] = on && s.has_bot ? jb_ll_area(s.buf[p], s.chunk, h->dim, pe, 1) : nullptr;
    }
    if (on && ((s.has_top && !s.ll_out_top[0]) || (s.has_bot && !s.ll_out_bot[0])))
      for (int p = 0; p < 2; ++p) d.ll_out_top[p] = d.ll_out_bot[p] = nullptr, d.ll_in_top[p] = d.ll_in_bot[p] = nullptr;
  }
}

int run_cpufree_k1(jacobi_ctx *h, int64_t iters) {
  const bool nocomp = h->flags & JACOBI_FLAG_NO_COMPUTE;
  const bool norm = !nocomp && h->norm_every > 0;
  auto groups = launch_groups(h);
  std::vector<LaunchPlan> plans(groups.size());
  // Resident (on-chip) kernel when every slab fits (auto) or when forced (not with the norm).
  bool resident = !nocomp && !norm && h->resident != 0 && h->kind != KIND_SHMEM;
  if (resident && !resident_fits_all(h)) {
    if (h->resident == 1) return JACOBI_EINVAL;
    resident = false;
  }
  if (resident) {
    for (size_t i = 0; i < groups.size() && resident; ++i)
      if (plan_resident(h, groups[i], plans[i]) != JACOBI_OK) resident = false;
    if (!resident && h->resident == 1) return JACOBI_EINVAL;
  }
  if (norm && h->resident == 1) return JACOBI_EINVAL;
  h->last_resident = resident ? 1 : 0;
  for (size_t i = 0; i < groups.size(); ++i) {
    if (!resident) {
      const int64_t sched = h->schedule;
      if (norm) h->schedule = 2;  // the norm's partial sums are indexed by dynamic items
      int rc = plan_launch(h, groups[i], LK_PERSIST, nocomp, plans[i]);
      h->schedule = sched;
      if (rc) return rc;
      if (norm && (rc = setup_norm(h, plans[i]))) return rc;
      if (!norm) setup_ll(h, plans[i]);
    }
    plans[i].P.t0 = h->t;
    plans[i].P.iters = iters;
  }
  for (auto &L : plans) {
    int rc = setup_trace(h, L);
    if (rc) return rc;
  }
  // Reset per-run counters (barrier, status, claim counters).  Flags are monotonic across runs:
  // raise every inbound slot to the current iteration (atomicMax: a neighbour that already
  // signalled this run is kept), so slots unused by an earlier split never hold stale values.
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    for (int k : L.slab_idx) {
      Slab &s = h->slabs[k];
      CK(reset_run_counters(s, L.stream));
      CK(jbk::launch_flag_max(&s.ctrl->flag_in[0][0], 2 * JB_MAXK, (unsigned long long)h->t, L.stream));
      ++h->last_launches;
      if (s.blk_flags) {
        CK(jbk::launch_flag_max(s.blk_flags, JB_MAX_BLOCKS, (unsigned long long)h->t, L.stream));
        ++h->last_launches;
      }
    }
  }
  // Debug: JACOBI_TRACE=1 records when each CTA finished its work in the first 8 iterations.
  unsigned long long *trace = nullptr;
  const bool tracing = getenv("JACOBI_TRACE") && plans.size() == 1;
  if (tracing) {
    CK(cudaMalloc(&trace, 8 * plans[0].grid * sizeof(unsigned long long)));
    CK(cudaMemset(trace, 0, 8 * plans[0].grid * sizeof(unsigned long long)));
    plans[0].P.trace = trace;
  }
  // One host thread launches every GPU's persistent kernel back to back (co-residency across
  // GPUs only needs every kernel to start; the device watchdog bounds any wait).
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    Slab &s0 = h->slabs[L.slab_idx[0]];
    CK(cudaEventRecord(s0.ev0, L.stream));
    if (resident) CK(jbk::launch_resident(L.P, L.cpp, L.grid, L.smem, L.stream));
    else CK(jbk::launch_sweep(L.P, nocomp, true, L.grid, L.smem, L.stream));
    ++h->last_launches;
    CK(cudaEventRecord(s0.ev1, L.stream));
  }
  int rc_all = JACOBI_OK;
  double mx = 0;
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    Slab &s0 = h->slabs[L.slab_idx[0]];
    CK(cudaEventSynchronize(s0.ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, s0.ev0, s0.ev1));
    for (int k : L.slab_idx) h->slabs[k].last_ms = ms;
    mx = std::max(mx, (double)ms);
    int rc = read_status(s0);
    if (rc && !rc_all) rc_all = rc;
  }
  h->last_ms_max = mx;
  if (tracing) {
    const int n = plans[0].grid;
    std::vector<unsigned long long> tr(8 * n);
    CK(cudaMemcpy(tr.data(), trace, tr.size() * 8, cudaMemcpyDeviceToHost));
    cudaFree(trace);
    for (int it = 1; it < 8 && it < iters; ++it) {
      std::vector<double> d;
      unsigned long long t0 = ~0ull;
      for (int c = 0; c < n; ++c) t0 = std::min(t0, tr[(it - 1) * n + c]);
      for (int c = 0; c < n; ++c) d.push_back((tr[it * n + c] - t0) / 1e3);
      std::vector<double> s = d;
      std::sort(s.begin(), s.end());
      fprintf(stderr, "[trace] it %d work-end us after prev barrier: min %.1f med %.1f max %.1f | slowest ctas:",
              it, s[0], s[n / 2], s[n - 1]);
      for (int k = 0; k < 4; ++k) {
        int arg = (int)(std::max_element(d.begin(), d.end()) - d.begin());
        fprintf(stderr, " %d(%.1f)", arg, d[arg]);
        d[arg] = -1;
      }
      fprintf(stderr, "\n");
    }
  }
  if (rc_all) return rc_all;
  int64_t done = iters;
  if (norm) {  // every slab stopped after the same iteration: read it (and the norm) from slab 0
    Slab &s0 = h->slabs[0];
    CK(cudaSetDevice(s0.device));
    long long d = 0;
    double r = 0;
    CK(cudaMemcpy(&d, &s0.ctrl->done_iters, sizeof(d), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&r, &s0.ctrl->norm_out, sizeof(r), cudaMemcpyDeviceToHost));
    done = d;
    h->norm_checks += done / h->norm_every;
    if (done >= h->norm_every) h->last_norm = r;
  }
  h->t += done;
  return JACOBI_OK;
}

// Temporally blocked CPU-Free launch (tblock.cu) of `iters` (a multiple of 2K)
// iterations: per launch group the roles and flags of plan_launch (boundary CTAs run the edge
// zones with the per-iteration exchange, then join the interior), the guided dynamic schedule
// over the interior planes the edge zones leave, and the ring shortened to the smem budget.
// (K, pairs per lane, variant) of the time-blocked kernel for this handle; K = 0: none fits.
// variant: 2D odd K = the wavefront lag (1, 2); 3D odd K = rows per warp of the tile.
void tblock_choice(const jacobi_ctx *h, int *k_out, int *ppt_out, int *var_out, int *ws_out) {
  const int kmax = h->dim == 2 ? JB_TB_KMAX2 : JB_TB_KMAX3;
  int k = h->tb_k >= 2 ? (int)std::min<int64_t>(h->tb_k, kmax) : (h->dim == 2 ? JB_TB_K2D : JB_TB_K3D);
  // every slab needs its edge zones (2K planes) when it has neighbours: shallower blocks otherwise
  const int64_t chunk_min = (h->n_out - 2) / h->total;
  auto fits = [&](int kk) { return h->total == 1 || chunk_min >= 2 * kk; };
  auto dflt_ppt = [&](int kk) { return h->dim == 3 ? (kk == 2 ? 4 : 1) : kk == 5 ? JB_TB_PPT5 : 4; };
  auto dflt_var = [&](int kk) { return kk == 2 ? 1 : h->dim == 3 ? JB_TB_RPW3 : JB_TB_LAG; };
  while (k > 2 && !(fits(k) && jbk::tblock_ncw(h->dim, k, dflt_ppt(k), dflt_var(k), 1) > 0)) k -= (k == 3 ? 1 : 2);
  int ppt = dflt_ppt(k), var = dflt_var(k);
  const int64_t var_req = h->dim == 3 ? h->tb_rpw : h->tb_lag;
  if (h->tb_ppt > 0 && jbk::tblock_ncw(h->dim, k, (int)h->tb_ppt, var, 1) > 0) ppt = (int)h->tb_ppt;
  if (var_req > 0 && jbk::tblock_ncw(h->dim, k, ppt, (int)var_req, 1) > 0) var = (int)var_req;
  if (h->tb_ppt > 0 && var_req > 0 && jbk::tblock_ncw(h->dim, k, (int)h->tb_ppt, (int)var_req, 1) > 0) {
    ppt = (int)h->tb_ppt;
    var = (int)var_req;
  }
  if (jbk::tblock_ncw(h->dim, k, ppt, var, 1) == 0) {
    ppt = dflt_ppt(k);
    var = dflt_var(k);
  }
  if (!fits(k)) k = 0;
  *ws_out = (h->tb_ws != 0 && k > 0 && jbk::tblock_ncw(h->dim, k, ppt, var, 1, 1) > 0) ? 1 : 0;
  *k_out = k;
  *ppt_out = ppt;
  *var_out = var;
}

int run_tblock(jacobi_ctx *h, int64_t iters, int K, int ppt, int lag, int ws) {
  auto groups = launch_groups(h);
  std::vector<LaunchPlan> plans(groups.size());
  // roles must match across slabs; two CTAs per SM only for K = 2
  const int per_sm = (h->tb_ctas >= 2 && h->total == 1 && K == 2) ? 2 : 1;
  for (size_t gi = 0; gi < groups.size(); ++gi) {
    LaunchPlan &L = plans[gi];
    const int64_t sched = h->schedule;
    h->schedule = 2;
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->slabs[groups[gi][0]].device));
    int rc = plan_launch(h, groups[gi], LK_PERSIST, false, L, per_sm == 2 ? launch_ctas(h, sms) * 2 : 0);
    h->schedule = sched;
    if (rc) return rc;
    JbGeom &g = L.P.g;
    if (h->dim == 3 && K > 2) {  // odd K: NCW warps x RPW rows x 64 ppt columns, outputs shrink by 2(K-1)
      const int ncw = jbk::tblock_ncw(3, K, ppt, lag, 1, ws), ty_all = ncw * lag;
      g.tx = 64 * ppt - 2 * (K - 1);
      g.ty = ty_all - 2 * (K - 1);
      g.rh = ty_all + 2;
      g.ws = 64 * ppt + 4;
      g.units_x = (int)((h->nx - 2 + g.tx - 1) / g.tx);
      g.units_y = (int)((h->ny - 2 + g.ty - 1) / g.ty);
      g.units = g.units_x * g.units_y;
      g.stage_doubles = (g.rh * g.ws + 15) / 16 * 16;  // TMA box destinations: 128-byte aligned
      g.xch_doubles = (K - 1) * 2 * ncw * 2 * 64 * ppt;
    } else if (h->dim == 3) {  // tiles of TY rows; stages hold rows y0-2 .. y0+TY+1
      g.ty = jbk::tblock_ty();
      g.rh = g.ty + 4;
      g.units_y = (int)((h->ny - 2 + g.ty - 1) / g.ty);
      g.units = g.units_x * g.units_y;
      g.stage_doubles = g.rh * g.ws;
    } else if (K > 2) {  // odd K: JB_NCW warps x (64 ppt - 2(K-1)) output columns per strip
      g.tx = jbk::tblock_ncw(2, K, ppt, lag, 1, ws) * (64 * ppt - 2 * (K - 1));
      g.ws = g.tx + 2 * K + 2;
      g.units_x = (int)((h->nx - 2 + g.tx - 1) / g.tx);
      g.units_y = 1;
      g.units = g.units_x;
      g.stage_doubles = g.ws;
    } else {  // K = 2: the strip of plan_launch (tile_x), ppt pairs per thread cover it
      ppt = g.tx >= 4 * JB_NC * 2 ? 4 : g.tx >= 2 * JB_NC * 2 ? 2 : 1;
    }
    g.stages = (int)(h->stages > 0 ? std::min<int64_t>(h->stages, JB_MAX_STAGES) : JB_MAX_STAGES);
    const int min_blk = (int)std::max<int64_t>(1, h->tb_min_block);
    for (size_t k = 0; k < groups[gi].size(); ++k) {
      Slab &s = h->slabs[groups[gi][k]];
      JbSlab &d = L.P.s[k];
      d.tb_lo = s.has_top ? K + 1 : 1;  // edge zones: level-K planes 1..K (top), C-K+1..C (bottom)
      d.tb_hi = s.has_bot ? s.chunk - K : s.chunk;
      d.mid_top_out = s.mid_top_out;
      d.mid_bot_out = s.mid_bot_out;
      d.tmap = nullptr;
      if (h->dim == 3 && K > 2) {  // one TMA box copy per plane: the tile's rh rows x ws columns
        rc = slab_tensor_maps(h, s, g.ws, g.rh);
        if (rc) return rc;
        d.tmap = s.tmap;
      }
      if (per_sm == 1 && (s.has_top || s.has_bot)) {
        // Boundary roles of the time-blocked plan: plan_launch split the CTAs by the per-iteration
        // tiles (C2: 8 strips of 2048), but the edge zones are distributed over THIS geometry's
        // units (C2: 25 strips of 672 with the register split) — one CTA per unit, up to a quarter
        // of the slab per side.  Every slab computes its own and its neighbours' counts with the
        // same deterministic function (neighbour_roles), so the flag slots agree.
        const int64_t sch = h->schedule;
        h->schedule = 2;
        int nt = 0, nb = 0, kt = 0, kb = 0;
        neighbour_roles(h, s.id, sms, g.units, &nt, &nb);
        if (s.has_top) neighbour_roles(h, s.id - 1, sms, g.units, nullptr, &kt);
        if (s.has_bot) neighbour_roles(h, s.id + 1, sms, g.units, &kb, nullptr);
        h->schedule = sch;
        d.n_top = s.has_top ? nt : 0;
        d.n_bot = s.has_bot ? nb : 0;
        d.k_in_top = kt;
        d.k_in_bot = kb;
        if (d.n_top + d.n_bot >= d.cta_count) return JACOBI_ENOCOOP;
      }
      const int64_t npl = d.tb_hi - d.tb_lo + 1;
      const int ni = d.cta_count - d.n_top - d.n_bot;
      d.dyn_items = 0;
      d.dyn_first = 0;
      if (npl > 0) {
        d.dyn_min_blk = min_blk;
        d.dyn_n = d.dyn_help ? d.cta_count : ni;
        const int64_t nblk = jbplan::dyn_blocks(npl, g.units, d.dyn_n, min_blk);
        d.dyn_items = (int64_t)g.units * nblk;
        d.dyn_first = (int)std::min<int64_t>(ni, d.dyn_items);
        rc = upload_table(s, npl, g.units, d.dyn_n, min_blk, nblk);
        if (rc) return rc;
        d.dyn_table = s.dyn_table;
      }
      s.desc = d;
    }
    int smem_optin = 0;
    CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, L.device));
    smem_optin = std::min(smem_optin, JB_SMEM_DEFAULT) - 1024;
    if (per_sm == 2) {  // two CTAs share the SM's shared memory (1 KB reserved per CTA + static)
      int smem_sm = 0;
      CK(cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, L.device));
      smem_optin = std::min(smem_optin, smem_sm / 2 - 1024 - 512);
    }
    while (g.stages > 3 && jbk::tblock_smem(g) > (size_t)smem_optin) --g.stages;
    if (jbk::tblock_smem(g) > (size_t)smem_optin) return JACOBI_EINVAL;
    L.smem = jbk::tblock_smem(g);
    int occ = 0;
    CK(jbk::prepare_tblock(g, K, ppt, lag, per_sm, ws, L.smem, &occ));
    if (occ < per_sm) {
      if (getenv("JACOBI_DEBUG")) fprintf(stderr, "[jacobi] tblock: occupancy %d < %d (smem %zu)\n", occ, per_sm, L.smem);
      return JACOBI_ENOCOOP;
    }
    for (int k : groups[gi]) h->slabs[k].smem = L.smem;
    L.P.t0 = h->t;
    L.P.iters = iters;
  }
  for (auto &L : plans) {
    int rc = setup_trace(h, L);
    if (rc) return rc;
  }
  // per-run counters; flags raised to the current iteration (as run_cpufree_k1)
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    for (int k : L.slab_idx) {
      Slab &s = h->slabs[k];
      CK(reset_run_counters(s, L.stream));
      CK(jbk::launch_flag_max(&s.ctrl->flag_in[0][0], 2 * JB_MAXK, (unsigned long long)h->t, L.stream));
      ++h->last_launches;
    }
  }
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    Slab &s0 = h->slabs[L.slab_idx[0]];
    CK(cudaEventRecord(s0.ev0, L.stream));
    CK(jbk::launch_tblock(L.P, K, ppt, lag, per_sm, ws, L.grid, L.smem, L.stream));
    ++h->last_launches;
    CK(cudaEventRecord(s0.ev1, L.stream));
  }
  int rc_all = JACOBI_OK;
  double mx = 0;
  for (auto &L : plans) {
    CK(cudaSetDevice(L.device));
    Slab &s0 = h->slabs[L.slab_idx[0]];
    CK(cudaEventSynchronize(s0.ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, s0.ev0, s0.ev1));
    for (int k : L.slab_idx) h->slabs[k].last_ms = ms;
    mx = std::max(mx, (double)ms);
    int rc = read_status(s0);
    if (rc && !rc_all) rc_all = rc;
  }
  h->last_ms_max = mx;
  if (rc_all) return rc_all;
  h->t += iters;
  return JACOBI_OK;
}

// CPU-Free run: the temporally blocked kernel for as many whole pairs of time blocks as fit when
// the run is eligible (one slab without neighbours, 2D, compute, no norm, not on-chip resident),
// the per-iteration kernels (streaming / resident) for the rest.  Device times add up.
// One-cluster on-chip kernel (cluster.cu) for a single 2D slab that fits in the
// shared memory of one thread-block cluster: cluster size (0: not eligible) and shared memory.
int cluster_plan(jacobi_ctx *h, size_t *smem) {
  if (h->total != 1 || h->slabs.size() != 1 || h->dim != 2 || h->kind == KIND_SHMEM) return 0;
  if ((h->flags & JACOBI_FLAG_NO_COMPUTE) || h->norm_every > 0) return 0;
  Slab &s = h->slabs[0];
  CK(cudaSetDevice(s.device));
  int optin = 0;
  CK(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, s.device));
  return jbk::cluster_choice(h->geom, s.chunk, std::min(optin, JB_SMEM_DEFAULT) - 1024, smem);
}

int run_cluster(jacobi_ctx *h, int64_t iters, int nc, size_t smem) {
  Slab &s = h->slabs[0];
  CK(cudaSetDevice(s.device));
  JbParams P;
  std::memset(&P, 0, sizeof(P));
  P.g = h->geom;
  P.nslabs = 1;
  P.flags = h->flags | flag_scope_bits(h);
  P.t0 = h->t;
  P.iters = iters;
  P.timeout_ns = (unsigned long long)h->timeout_ms * 1000000ull;
  P.status = s.ctrl->status;
  JbSlab &d = P.s[0];
  d.buf[0] = s.buf[0];
  d.buf[1] = s.buf[1];
  d.chunk = s.chunk;
  d.cta_count = nc;
  CK(reset_run_counters(s, s.stream));
  ++h->last_launches;
  CK(cudaEventRecord(s.ev0, s.stream));
  CK(jbk::launch_cluster(P, nc, smem, s.stream));
  ++h->last_launches;
  CK(cudaEventRecord(s.ev1, s.stream));
  CK(cudaEventSynchronize(s.ev1));
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, s.ev0, s.ev1));
  s.last_ms = ms;
  h->last_ms_max = ms;
  int rc = read_status(s);
  if (rc) return rc;
  h->t += iters;
  return JACOBI_OK;
}

int run_cpufree(jacobi_ctx *h, int64_t iters) {
  h->last_launches = 0;
  h->last_tblock = 0;
  h->last_tb_k = 0;
  h->last_tb_ws = 0;
  h->last_resident = 0;
  h->last_cluster = 0;
  if (h->cluster != 0) {  // auto (JB_CLUSTER_AUTO): only while the other kernel knobs are auto too
    size_t smem = 0;
    const int nc = cluster_plan(h, &smem);
    if (h->cluster == 1 && nc == 0) return JACOBI_EINVAL;
    const bool use = nc > 0 && (h->cluster == 1 || (JB_CLUSTER_AUTO && h->tblock < 0 && h->resident < 0));
    if (use) {
      int rc = run_cluster(h, iters, nc, smem);
      if (rc) return rc;
      h->last_cluster = nc;
      return JACOBI_OK;
    }
  }
  const bool nocomp = h->flags & JACOBI_FLAG_NO_COMPUTE;
  // P > 1: every slab needs the two edge zones (>= 2K planes); the NVSHMEM variant keeps jb_sweep
  int K = 0, ppt = 0, lag = 1, ws = 0;
  tblock_choice(h, &K, &ppt, &lag, &ws);
  const bool eligible = h->tblock != 0 && !nocomp && h->norm_every <= 0 && h->kind != KIND_SHMEM && K >= 2;
  if (h->tblock == 1 && !eligible) return JACOBI_EINVAL;
  // auto picks it where it measured faster than the per-iteration kernel: always for a slab
  // without neighbours; with neighbours the K phases of edge zones (each waiting for the
  // neighbour's previous phase) must be amortised by enough interior work per CTA — 2D >= 2^16
  // interior cells per CTA of the job (2048^2 with 2-8 virtual slabs, 28 K: 17.3 vs 11.0-12.2
  // us/iteration per-iteration; 4096^2, 113 K: 22.6-28.0 vs 42-44), 3D >= 3 * 2^16 and >= 64
  // CTAs per slab (256^3 with 2 virtual slabs, 111 K: 57.9 vs 49.8 us; 384^3, 380 K: 139 vs 191;
  // C3 with 2 virtual slabs 467 vs 384 Gcell/s; with 8, 18 CTAs per slab: 251 vs 340 — DESIGN.md
  // §5.9, §5.14).
  bool use_tb = h->total == 1;
  if (!use_tb) {
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->slabs[0].device));
    int min_ctas = sms;
    for (int id = 0; id < h->total; ++id) min_ctas = std::min(min_ctas, slab_ctas(h, id, sms));
    use_tb = jbplan::tblock_neighbours_auto(h->dim, cells_per_cta(h, sms), min_ctas);
  }
  const bool use = eligible && (h->tblock == 1 || use_tb);
  int64_t tb_iters = 0;
  if (use) {
    // odd K: any block count; K = 2: an even one (the result stays in buf[t & 1], R10)
    const int64_t step = (K & 1) ? K : 2 * K;
    tb_iters = iters / step * step;
    // auto: slabs that fit on chip run the resident kernel (faster for those small grids:
    // C1 2D 256^2 2.2 vs 3.1 us/iteration) — except a single slab of >= 2^18 interior cells,
    // where the time-blocked kernel's K iterations per barrier win (C5b 2D 1024^2: 3.3 vs 4.6
    // us/iteration); decided over every slab of the run so that all ranks take
    // the same kernel
    const int64_t cells = (h->nx - 2) * (h->dim == 3 ? (h->ny - 2) * (h->nz - 2) : (h->ny - 2));
    const bool big_single = h->total == 1 && cells >= ((int64_t)1 << 18);
    if (h->tblock < 0 && h->resident != 0 && !big_single && resident_fits_all(h)) tb_iters = 0;
  }
  double ms = 0;
  if (tb_iters > 0) {
    int rc = run_tblock(h, tb_iters, K, ppt, lag, ws);
    if (rc) return rc;
    ms = h->last_ms_max;
    h->last_tblock = tb_iters;
    h->last_tb_k = K;
    h->last_tb_ws = ws;
  }
  if (iters - tb_iters > 0) {
    int rc = run_cpufree_k1(h, iters - tb_iters);
    if (rc) return rc;
    ms += h->last_ms_max;
  }
  h->last_ms_max = ms;
  for (auto &s : h->slabs) s.last_ms = ms;
  return JACOBI_OK;
}
}  // namespace jbrt

extern "C" {
int jacobi_create(int64_t nx, int64_t ny, int64_t nz, int stencil, int ngpus, jacobi_t *out) {
  if (!out) return JACOBI_EINVAL;
  *out = nullptr;
  int rc = validate(nx, ny, nz, stencil, ngpus);
  if (rc) return rc;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < ngpus) return JACOBI_ENODEV;
  for (int g = 0; g + 1 < ngpus; ++g) {
    int a = 0, b = 0;
    cudaDeviceCanAccessPeer(&a, g, g + 1);
    cudaDeviceCanAccessPeer(&b, g + 1, g);
    if (!a || !b) return JACOBI_ENOPEER;
  }
  jacobi_ctx *h = new_ctx(nx, ny, nz, stencil, ngpus);
  h->kind = KIND_SINGLE;
  h->slabs.resize(ngpus);
  for (int g = 0; g < ngpus; ++g) {
    Slab &s = h->slabs[g];
    s.device = g;
    s.id = g;
    jbplan::decompose(h->n_out, ngpus, g, &s.start, &s.chunk);
    rc = alloc_slab(h, s);
    if (rc) { jacobi_destroy(h); return rc; }
  }
  for (int g = 0; g < ngpus; ++g) {
    cudaSetDevice(g);
    for (int o = 0; o < ngpus; ++o) {  // neighbours required; all pairs for the norm (NVSwitch)
      if (o == g) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, g, o);
      if (!can) {
        h->all_peers = false;  // neighbours were checked above; only the norm needs this pair
        continue;
      }
      cudaError_t e = cudaDeviceEnablePeerAccess(o, 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
      else if (e != cudaSuccess && (o == g - 1 || o == g + 1)) { jacobi_destroy(h); return JACOBI_ENOPEER; }
      else if (e != cudaSuccess) { cudaGetLastError(); h->all_peers = false; }
    }
  }
  link_local(h);
  *out = h;
  return JACOBI_OK;
}

int jacobi_create_virtual(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs, int device,
                          jacobi_t *out) {
  if (!out) return JACOBI_EINVAL;
  *out = nullptr;
  if (nslabs > JB_MAX_SLABS) return JACOBI_EINVAL;
  int rc = validate(nx, ny, nz, stencil, nslabs);
  if (rc) return rc;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return JACOBI_ENODEV;
  jacobi_ctx *h = new_ctx(nx, ny, nz, stencil, nslabs);
  h->kind = KIND_VIRTUAL;
  h->slabs.resize(nslabs);
  for (int g = 0; g < nslabs; ++g) {
    Slab &s = h->slabs[g];
    s.device = device;
    s.id = g;
    jbplan::decompose(h->n_out, nslabs, g, &s.start, &s.chunk);
    rc = alloc_slab(h, s);
    if (rc) { jacobi_destroy(h); return rc; }
  }
  link_local(h);
  *out = h;
  return JACOBI_OK;
}



int jacobi_run(jacobi_t h, int64_t iters) {
  if (!h || iters < 0) return JACOBI_EINVAL;
  if (!h->peers_ready) return JACOBI_ESTATE;
  if (iters == 0) {
    h->last_ms_max = 0;
    return JACOBI_OK;
  }
  if (h->mode == JACOBI_MODE_CPUFREE) return run_cpufree(h, iters);
  if (h->mode == JACOBI_MODE_BASELINE_MEMCPY) return run_baseline(h, iters, BK_COPY);
  if (h->mode == JACOBI_MODE_BASELINE_NCCL) return run_baseline(h, iters, BK_NCCL);
  if (h->mode == JACOBI_MODE_BASELINE_OVERLAP) return run_baseline(h, iters, BK_OVERLAP);
  if (h->mode == JACOBI_MODE_BASELINE_P2P) return run_baseline(h, iters, BK_P2P);
  if (h->mode == JACOBI_MODE_BASELINE_GRAPH) return run_baseline(h, iters, BK_GRAPH);
  if (h->mode == JACOBI_MODE_BASELINE_NVSHMEM) return run_baseline(h, iters, BK_SHMEM);
  return JACOBI_EINVAL;
}

int jacobi_set_mode(jacobi_t h, int mode, int flags) {
  if (!h) return JACOBI_EINVAL;
  if (mode < JACOBI_MODE_CPUFREE || mode > JACOBI_MODE_BASELINE_NVSHMEM) return JACOBI_EINVAL;
  if (flags & ~(JACOBI_FLAG_NO_COMPUTE | JACOBI_FLAG_DROP_SIGNAL)) return JACOBI_EINVAL;
  h->mode = mode;
  h->plan_gen++;
  h->flags = flags;
  return JACOBI_OK;
}

static int64_t *param_slot(jacobi_t h, const char *name) {
  if (!std::strcmp(name, "tile_x")) return &h->tile_x;
  if (!std::strcmp(name, "tile_y")) return &h->tile_y;
  if (!std::strcmp(name, "stages")) return &h->stages;
  if (!std::strcmp(name, "boundary_ctas")) return &h->boundary_ctas;
  if (!std::strcmp(name, "ctas")) return &h->ctas;
  if (!std::strcmp(name, "schedule")) return &h->schedule;
  if (!std::strcmp(name, "timeout_ms")) return &h->timeout_ms;
  if (!std::strcmp(name, "min_block")) return &h->min_block;
  if (!std::strcmp(name, "dyn_help")) return &h->dyn_help;
  if (!std::strcmp(name, "resident")) return &h->resident;
  if (!std::strcmp(name, "block_sync")) return &h->block_sync;
  if (!std::strcmp(name, "norm_every")) return &h->norm_every;
  if (!std::strcmp(name, "l2hint")) return &h->l2hint;
  if (!std::strcmp(name, "last_resident")) return &h->last_resident;
  if (!std::strcmp(name, "tblock")) return &h->tblock;
  if (!std::strcmp(name, "tb_min_block")) return &h->tb_min_block;
  if (!std::strcmp(name, "tb_ctas")) return &h->tb_ctas;
  if (!std::strcmp(name, "tb_k")) return &h->tb_k;
  if (!std::strcmp(name, "tb_ppt")) return &h->tb_ppt;
  if (!std::strcmp(name, "tb_lag")) return &h->tb_lag;
  if (!std::strcmp(name, "tb_rpw")) return &h->tb_rpw;
  if (!std::strcmp(name, "tb_ws")) return &h->tb_ws;
  if (!std::strcmp(name, "last_tb_ws")) return &h->last_tb_ws;
  if (!std::strcmp(name, "last_tb_k")) return &h->last_tb_k;
  if (!std::strcmp(name, "last_tblock")) return &h->last_tblock;
  if (!std::strcmp(name, "halo_trace")) return &h->halo_trace;
  if (!std::strcmp(name, "barrier")) return &h->barrier;
  if (!std::strcmp(name, "halo_ll")) return &h->halo_ll;
  if (!std::strcmp(name, "flag_scope")) return &h->flag_scope;
  if (!std::strcmp(name, "cluster")) return &h->cluster;
  if (!std::strcmp(name, "last_cluster")) return &h->last_cluster;
  if (!std::strcmp(name, "last_launches")) return &h->last_launches;
  return nullptr;
}

int jacobi_set_param(jacobi_t h, const char *name, int64_t value) {
  if (!h || !name) return JACOBI_EINVAL;
  if (!std::strcmp(name, "last_resident") || !std::strcmp(name, "last_tblock") || !std::strcmp(name, "last_tb_k") ||
      !std::strcmp(name, "last_launches") || !std::strcmp(name, "last_tb_ws") || !std::strcmp(name, "last_cluster"))
    return JACOBI_EINVAL;  // read-only
  int64_t *p = param_slot(h, name);
  if (!p) return JACOBI_EINVAL;
  if (!std::strcmp(name, "timeout_ms")) value = value < 0 ? 20000 : value;
  if (!std::strcmp(name, "tile_x") && value > 4096) return JACOBI_EINVAL;
  if (!std::strcmp(name, "tile_y") && value > 30) return JACOBI_EINVAL;
  if (!std::strcmp(name, "halo_trace") && (value < 0 || value > (1 << 20))) return JACOBI_EINVAL;
  if (!std::strcmp(name, "flag_scope") && value > 0 && h->kind != KIND_VIRTUAL) return JACOBI_EINVAL;  // .gpu needs one device
  *p = value;
  h->plan_gen++;
  return JACOBI_OK;
}

int jacobi_get_param(jacobi_t h, const char *name, int64_t *value) {
  if (!h || !name || !value) return JACOBI_EINVAL;
  int64_t *p = param_slot(h, name);
  if (!p) return JACOBI_EINVAL;
  *value = *p;
  return JACOBI_OK;
}

int jacobi_scatter(jacobi_t h, const double *in) {
  if (!h || !in) return JACOBI_EINVAL;
  const int64_t pe = h->geom.plane_elems, pitch = h->geom.pitch;
  const int64_t rows_per_plane = h->dim == 2 ? 1 : h->ny;
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    const double *src = in + (s.start - 1) * rows_per_plane * h->nx;
    // All copies on the slab's stream, then a stream sync: a device-to-device cudaMemcpy is
    // asynchronous w.r.t. the host and would race with the next launch on this stream.
    CK(cudaMemcpy2DAsync(s.buf[0] + 3, pitch * sizeof(double), src, h->nx * sizeof(double),
                         h->nx * sizeof(double), (s.chunk + 2) * rows_per_plane, cudaMemcpyHostToDevice,
                         s.stream));
    CK(cudaMemcpyAsync(s.buf[1], s.buf[0], (size_t)(s.chunk + 2) * pe * sizeof(double),
                       cudaMemcpyDeviceToDevice, s.stream));
  }
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(cudaStreamSynchronize(s.stream));
  }
  return JACOBI_OK;
}

int jacobi_gather(jacobi_t h, double *out) {
  if (!h || !out) return JACOBI_EINVAL;
  const int64_t pe = h->geom.plane_elems, pitch = h->geom.pitch;
  const int64_t rpp = h->dim == 2 ? 1 : h->ny;
  const int cur = (int)(h->t & 1);
  const size_t w = h->nx * sizeof(double), dp = pitch * sizeof(double);
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(cudaMemcpy2DAsync(out + s.start * rpp * h->nx, w, s.buf[cur] + pe + 3, dp, w, s.chunk * rpp,
                         cudaMemcpyDeviceToHost, s.stream));
    if (s.id == 0)
      CK(cudaMemcpy2DAsync(out, w, s.buf[cur] + 3, dp, w, rpp, cudaMemcpyDeviceToHost, s.stream));
    if (s.id == h->total - 1)
      CK(cudaMemcpy2DAsync(out + (h->n_out - 1) * rpp * h->nx, w, s.buf[cur] + (s.chunk + 1) * pe + 3, dp, w,
                           rpp, cudaMemcpyDeviceToHost, s.stream));
  }
  for (auto &s : h->slabs) {
    CK(cudaSetDevice(s.device));
    CK(cudaStreamSynchronize(s.stream));
  }
  return JACOBI_OK;
}

int jacobi_set_tolerance(jacobi_t h, double tol) {
  if (!h || !(tol >= 0.0)) return JACOBI_EINVAL;
  h->tol = tol;
  return JACOBI_OK;
}

int jacobi_last_norm(jacobi_t h, double *norm) {
  if (!h || !norm) return JACOBI_EINVAL;
  *norm = h->last_norm;
  return JACOBI_OK;
}

int jacobi_read_slab(jacobi_t h, int i, int parity, double *out) {
  if (!h || !out || i < 0 || i >= (int)h->slabs.size() || (parity != 0 && parity != 1)) return JACOBI_EINVAL;
  Slab &s = h->slabs[i];
  CK(cudaSetDevice(s.device));
  CK(cudaMemcpy(out, s.buf[parity], (size_t)slab_elems(h, s) * sizeof(double), cudaMemcpyDeviceToHost));
  return JACOBI_OK;
}

int jacobi_last_time(jacobi_t h, double *ms_max, double *ms_per_slab) {
  if (!h) return JACOBI_EINVAL;
  if (ms_max) *ms_max = h->last_ms_max;
  if (ms_per_slab)
    for (size_t i = 0; i < h->slabs.size(); ++i) ms_per_slab[i] = h->slabs[i].last_ms;
  return JACOBI_OK;
}

int jacobi_halo_trace(jacobi_t h, int slab, uint64_t *out, int64_t n) {
  if (!h || !out || slab < 0 || slab >= (int)h->slabs.size() || n < 0) return JACOBI_EINVAL;
  Slab &s = h->slabs[slab];
  if (n > s.trace_n || !s.trace) return JACOBI_ESTATE;  // no traced run of that length yet
  CK(cudaSetDevice(s.device));
  CK(cudaStreamSynchronize(s.stream));
  // the last run laid the buffer out for trace_n exchanges per side: copy each side's first n
  for (int side = 0; side < 2; ++side)
    CK(cudaMemcpy(out + (size_t)side * n * 3, s.trace + (size_t)side * s.trace_n * 3, (size_t)n * 3 * 8,
                  cudaMemcpyDeviceToHost));
  return JACOBI_OK;
}

int jacobi_iterations(jacobi_t h, int64_t *t) {
  if (!h || !t) return JACOBI_EINVAL;
  *t = h->t;
  return JACOBI_OK;
}

int jacobi_num_slabs(jacobi_t h, int *local, int *total) {
  if (!h) return JACOBI_EINVAL;
  if (local) *local = (int)h->slabs.size();
  if (total) *total = h->total;
  return JACOBI_OK;
}

int jacobi_describe(jacobi_t h, int i, int64_t *o) {
  if (!h || !o || i < 0 || i >= (int)h->slabs.size()) return JACOBI_EINVAL;
  Slab &s = h->slabs[i];
  // Plan the CPU-free launch now so the description is current.
  std::vector<LaunchPlan> plans;
  for (auto &grp : launch_groups(h)) {
    if (std::find(grp.begin(), grp.end(), i) == grp.end()) continue;
    LaunchPlan L;
    int rc = plan_launch(h, grp, LK_PERSIST, h->flags & JACOBI_FLAG_NO_COMPUTE, L);
    if (rc) return rc;
    o[0] = s.start; o[1] = s.chunk; o[2] = L.P.g.pitch; o[3] = L.P.g.plane_elems;
    o[4] = L.P.g.tx; o[5] = L.P.g.ty; o[6] = L.P.g.units_x; o[7] = L.P.g.units_y;
    o[8] = L.P.g.stages; o[9] = s.desc.n_top; o[10] = s.desc.n_bot;
    o[11] = s.desc.cta_count - s.desc.n_top - s.desc.n_bot; o[12] = s.desc.cta_count;
    o[13] = s.desc.k_planes; o[14] = (int64_t)L.smem; o[15] = s.device;
  }
  return JACOBI_OK;
}

int jacobi_destroy(jacobi_t h) {
  if (!h) return JACOBI_OK;
  for (auto &s : h->slabs) {
    if (s.device >= 0) cudaSetDevice(s.device);
    if (s.stream) cudaStreamSynchronize(s.stream);
  }
#ifdef JB_NVSHMEM
  if (h->kind == KIND_SHMEM) nvshmem_barrier_all();  // collective: no PE still reads our heap
#endif
  for (auto &s : h->slabs) free_slab(s, h->alloc);
  if (h->graph_exec) cudaGraphExecDestroy(h->graph_exec);
  delete h;
  return JACOBI_OK;
}
}  // extern "C"
