// runtime_internal.h — host-runtime types shared by runtime.cu (core: slabs, planning, the
// CPU-Free run and the C ABI), baselines.cu (CPU-controlled comparison modes) and multiproc.cu
// (CUDA IPC, NCCL, NVSHMEM, device-memory allocators).  Product code only.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstddef>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/jacobi.h"
#include "jacobi_internal.h"
#ifdef JB_NVSHMEM
#include <nvshmem.h>
#include <nvshmemx.h>
#endif

namespace jbk {
cudaError_t prepare(int dim, bool nocomp, bool persist, size_t smem);
cudaError_t occupancy(int dim, bool nocomp, bool persist, size_t smem, int *blocks_per_sm);
cudaError_t launch_sweep(const JbParams &p, bool nocomp, bool persist, int grid, size_t smem,
                         cudaStream_t st);
cudaError_t launch_init(double *b0, double *b1, int64_t nplanes, const JbGeom &g, int64_t z_first,
                        unsigned long long seed, cudaStream_t st);
cudaError_t launch_flag_max(unsigned long long *flags, int n, unsigned long long v, cudaStream_t st);
cudaError_t prepare_resident(int dim, int cpp, size_t smem, int *blocks_per_sm);
cudaError_t launch_resident(const JbParams &p, int cpp, int grid, size_t smem, cudaStream_t st);
cudaError_t launch_neighbour_wait(const JbParams &p, unsigned long long target, cudaStream_t st);
int cluster_choice(const JbGeom &g, int64_t chunk, int smem_optin, size_t *smem_out);
cudaError_t launch_cluster(const JbParams &p, int nc, size_t smem, cudaStream_t st);
int tblock_ty();
int tblock_ncw(int dim, int k, int ppt, int lag, int per_sm, int ws = 0);
size_t tblock_smem(const JbGeom &g);
cudaError_t prepare_tblock(const JbGeom &g, int k, int ppt, int lag, int per_sm, int ws, size_t smem, int *blocks_per_sm);
cudaError_t launch_tblock(const JbParams &p, int k, int ppt, int lag, int per_sm, int ws, int grid, size_t smem,
                          cudaStream_t st);
}  // namespace jbk

namespace jbrt {

constexpr unsigned long long kSeedBench = 0x5C24ull;
enum Kind { KIND_SINGLE = 0, KIND_VIRTUAL = 1, KIND_DIST = 2, KIND_SHMEM = 3 };

inline int cuda_err(cudaError_t e) {
  if (e == cudaSuccess) return JACOBI_OK;
  if (e == cudaErrorMemoryAllocation) return JACOBI_ENOMEM;
  if (e == cudaErrorCooperativeLaunchTooLarge) return JACOBI_ENOCOOP;
  if (getenv("JACOBI_DEBUG")) fprintf(stderr, "[jacobi] CUDA error: %s\n", cudaGetErrorString(e));
  return JACOBI_ECUDA;
}
#define CK(x)                                  \
  do {                                         \
    int _rc = cuda_err(x);                     \
    if (_rc != JACOBI_OK) return _rc;          \
  } while (0)

// ---------------------------------------------------------------- NCCL (dlopen'ed on demand)
struct NcclApi {
  void *lib = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommInitAll)(ncclComm_t *, int, const int *) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  bool load() {
    if (lib) return true;
    // JACOBI_NCCL_LIB (set by the Python binding to the NCCL that PyTorch ships) first: the
    // process must not end up with two different libnccl.so.2 — a system NCCL loaded here
    // first would be reused by a later `import torch` (same soname) and lack its symbols.
    // Loaded RTLD_LOCAL: the library's symbols are only reached through the pointers below.
    const char *env = getenv("JACOBI_NCCL_LIB");
    const char *names[] = {env ? env : "libnccl.so.2", "libnccl.so.2", "libnccl.so"};
    for (const char *n : names) {
      lib = dlopen(n, RTLD_NOW | RTLD_LOCAL);
      if (lib) break;
    }
    if (!lib) return false;
#define LD(f) f = reinterpret_cast<decltype(f)>(dlsym(lib, "nccl" #f))
    LD(GetUniqueId); LD(CommInitRank); LD(CommInitAll); LD(CommDestroy);
    LD(Send); LD(Recv); LD(GroupStart); LD(GroupEnd);
#undef LD
    return GetUniqueId && CommInitRank && CommInitAll && CommDestroy && Send && Recv && GroupStart && GroupEnd;
  }
};
extern NcclApi g_nccl;

// Device-memory allocator for the slab buffers and control blocks (jacobi_set_allocator):
// cudaMalloc by default, or a caller-supplied one (the Python binding installs PyTorch's caching
// allocator so that PyTorch owns the device memory, as the north star asks).
struct Allocator {
  jacobi_alloc_fn alloc = nullptr;
  jacobi_free_fn free = nullptr;
  void *user = nullptr;
};
extern Allocator g_alloc;

// cuMemGetAddressRange through the runtime's driver entry point (no libcuda link needed): the
// base of the allocation containing `p`, so IPC handles of sub-allocations carry their offset.
size_t alloc_offset(const void *p);

// ---------------------------------------------------------------- IPC blob (dist mode)
struct IpcBlob {
  uint32_t magic;
  int32_t rank;
  int32_t sms;  // SM count of the rank's GPU: the CPU-Free role split must match across ranks
  int32_t pad;
  int64_t chunk;
  int64_t plane_elems;
  cudaIpcMemHandle_t buf[2];
  cudaIpcMemHandle_t ctrl;
  uint64_t off[3];  // offsets of buf[0], buf[1], ctrl inside their allocations (caller allocators)
};
constexpr uint32_t kIpcMagic = 0x4A43424Bu;

typedef int (*PFN_getAddressRange)(unsigned long long *, size_t *, unsigned long long);
}  // namespace jbrt

using namespace jbrt;

struct Slab {
  int device = 0;
  int id = 0;  // global slab index
  int64_t start = 0, chunk = 0;
  double *buf[2] = {nullptr, nullptr};
  JbCtrl *ctrl = nullptr;
  cudaStream_t stream = nullptr;
  cudaStream_t stream2 = nullptr;  // comm stream of the Copy-Overlap baseline
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  cudaEvent_t ev_sync = nullptr, ev_copy = nullptr;  // baseline stream / graph dependencies
  bool has_top = false, has_bot = false;
  double *peer_top[2] = {nullptr, nullptr};
  double *peer_bot[2] = {nullptr, nullptr};
  double *mid_top_out = nullptr, *mid_bot_out = nullptr;  // neighbours' time-blocked edge slots
  unsigned long long *ll_out_top[2] = {nullptr, nullptr};  // neighbours' LL receive areas (halo_ll)
  unsigned long long *ll_out_bot[2] = {nullptr, nullptr};
  unsigned long long *flag_out_top = nullptr, *flag_out_bot = nullptr;
  int peer_top_dev = -1, peer_bot_dev = -1;
  int shm_pe_top = -1, shm_pe_bot = -1;  // NVSHMEM variant: neighbour PEs
  std::vector<void *> ipc_opened;
  ncclComm_t comm = nullptr;
  double last_ms = 0;
  JbSlab desc{};  // last launch descriptor (for jacobi_describe)
  int32_t *dyn_table = nullptr;  // guided-schedule block table of the last plan (device; one of tabs)
  struct DynTab {                // cached tables: the per-iteration and the time-blocked plan alternate
    int32_t *ptr = nullptr;      // within one jacobi_run, so two entries keep both resident
    int64_t cap = 0;             // entries allocated
    int64_t key[4] = {0, 0, 0, 0};
    uint64_t used = 0;           // LRU stamp
  } tabs[2];
  uint64_t tab_clock = 0;
  unsigned long long *blk_flags = nullptr;  // resident kernel: per-block flags (device)
  double *partials = nullptr;               // N4: per-run partial sums (device)
  int64_t partials_cap = 0;
  JbCtrl **norm_peers = nullptr;            // N4: device array of every slab's control block
  unsigned long long *bar_flags = nullptr;  // flag-array grid barrier: one slot per CTA (device)
  unsigned long long *trace = nullptr;  // halo-exchange trace of the last CPU-Free run (device)
  int64_t trace_cap = 0;                // its capacity (exchanges per side)
  int64_t trace_n = 0;                  // exchanges per side recorded by the last run (its stride)
  void *tmap = nullptr;       // time-blocked 3D kernel: two CUtensorMaps (buf[0], buf[1]) in device memory
  int tmap_key[2] = {0, 0};   // their box (columns, rows)
  int grid = 0;
  size_t smem = 0;
};

struct jacobi_ctx {
  int kind = KIND_SINGLE;
  int64_t nx = 0, ny = 0, nz = 0, n_out = 0;
  int stencil = 5, dim = 2;
  int total = 1;  // total slabs P
  int rank = 0;
  std::vector<Slab> slabs;
  int64_t t = 0;
  int mode = JACOBI_MODE_CPUFREE, flags = 0;
  int64_t tile_x = -1, tile_y = -1, stages = -1, boundary_ctas = -1, ctas = -1, schedule = -1;
  int64_t min_block = 8, dyn_help = 1;
  int64_t resident = -1;       // on-chip resident kernel: -1 auto (when the slab fits), 0 off, 1 on
  int64_t block_sync = 0;      // resident kernel: 0 grid barrier, 1 neighbour-block flags
  int64_t l2hint = -1;         // streaming loads with L2 eviction hints (-1 default = off)
  int64_t last_resident = 0;   // read-only: whether the last CPU-Free run used it
  int64_t tblock = -1;         // temporally blocked kernel (K iterations per HBM pass): -1 auto
                               // (2D always, edge zones between slabs; 3D see run_cpufree), 0 never, 1 force
  int64_t tb_min_block = 16;   // smallest dynamic plane block of the temporally blocked kernel
  int64_t tb_ctas = 1;         // CTAs per SM of the temporally blocked kernel (1 or 2; K = 2 only)
  int64_t tb_k = -1;           // iterations per time block: -1 auto (2D: JB_TB_K2D = 5, 3D: JB_TB_K3D = 3); 2, 3, 5
  int64_t tb_ppt = -1;         // 2D cell pairs per thread and level: -1 auto (K = 2, 3: 4; K = 5: JB_TB_PPT5 = 1; 3D: 1)
  int64_t tb_lag = -1;         // 2D odd K: wavefront lag between levels (1 or 2; -1 auto)
  int64_t tb_rpw = -1;         // 3D odd K: rows per warp of the tile (-1 auto)
  int64_t tb_ws = -1;          // warp-specialised register split (12 compute warps; -1 auto = where built, 0 off)
  int64_t last_tb_ws = 0;      // read-only: whether the last time-blocked run used it
  int64_t last_tb_k = 0;       // read-only: K of the last time-blocked run
  int64_t last_tblock = 0;     // read-only: iterations of the last CPU-Free run done time-blocked
  int64_t last_launches = 0;   // read-only: kernels this process launched in the last jacobi_run
  int64_t barrier = 0;         // grid barrier of the CPU-Free kernels: 0 counter, 1 per-CTA flags
  int64_t halo_trace = 0;      // measurement: record the first n halo exchanges of each CPU-Free run
  int64_t cluster = -1;        // one-cluster on-chip kernel for small 2D grids (§5.12): -1 auto, 0 off, 1 force
  int64_t last_cluster = 0;    // read-only: cluster size of the last CPU-Free run (0: not used)
  int64_t flag_scope = -1;     // halo flag scope: -1 auto (.gpu for virtual slabs, .sys otherwise), 0 sys, 1 gpu
  int64_t halo_ll = -1;        // LL halo protocol of the streaming CPU-Free kernel (§5.11): -1 auto, 0 off, 1 on
                               // (%globaltimer wait begin / flag acquired / signal; jacobi_halo_trace)
  int64_t norm_every = 0;      // N4: check the update norm every k iterations (0 = off)
  double tol = 0.0;            // N4: stop once the norm <= tol
  int64_t norm_checks = 0;     // N4: checks performed so far (monotone slot values)
  double last_norm = -1.0;     // N4: norm of the last check
  std::vector<JbCtrl *> all_ctrl;  // dist mode: every rank's control block (opened via IPC)
  int64_t timeout_ms = 20000;
  bool peers_ready = false;
  bool all_peers = true;   // single process: peer access enabled between EVERY pair of GPUs (norm all-reduce)
  bool nccl_ready = false;
  double last_ms_max = 0;
  cudaGraphExec_t graph_exec = nullptr;  // cached GRAPH-baseline executable
  int64_t graph_iters = -1;
  int graph_parity = -1;
  int64_t graph_gen = -1, plan_gen = 0;  // plan_gen bumps on every set_mode / set_param
  JbGeom geom{};  // layout geometry (pitch, plane_elems) fixed at create
  Allocator alloc;  // allocator of buffers / control blocks (captured at create)
};

namespace jbrt {

// What a launch computes (CPU-Free persistent kernel or one of the discrete baseline kernels).
enum LaunchKind {
  LK_PERSIST = 0,  // CPU-Free: roles, peer stores, flags, grid barrier, all iterations
  LK_ALL,          // discrete: every plane 1..chunk, no roles (Copy / NCCL / graph baselines)
  LK_P2P,          // discrete: boundary roles store edge planes straight into the peers' halos
  LK_INNER,        // discrete: planes 2..chunk-1 only (Copy-Overlap compute kernel)
  LK_EDGES,        // discrete: planes 1 and chunk only, no peer stores (Copy-Overlap comm kernel)
};

struct LaunchPlan {
  JbParams P;
  int grid = 0;
  int cpp = 0;  // resident kernel: cell pairs per thread
  size_t smem = 0;
  int device = 0;
  cudaStream_t stream = nullptr;
  std::vector<int> slab_idx;
};

enum BaseKind { BK_COPY, BK_NCCL, BK_OVERLAP, BK_P2P, BK_GRAPH, BK_SHMEM };

int64_t slab_elems(const jacobi_ctx *h, const Slab &s);
int validate(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs);
jacobi_ctx *new_ctx(int64_t nx, int64_t ny, int64_t nz, int stencil, int total);
int alloc_slab(jacobi_ctx *h, Slab &s);
void free_slab(Slab &s, const Allocator &a);
void link_local(jacobi_ctx *h);
int upload_table(Slab &s, int64_t npl, int units, int n, int min_blk, int64_t nb);
int launch_ctas(const jacobi_ctx *h, int sms);
int slab_ctas(const jacobi_ctx *h, int id, int sms);
void split_roles(const jacobi_ctx *h, int count, int64_t inner, bool top, bool bot, int units, int *nt,
                 int *nb, int *ni);
void neighbour_roles(const jacobi_ctx *h, int id, int sms, int units, int *nt_out, int *nb_out);
int plan_launch(jacobi_ctx *h, const std::vector<int> &idx, LaunchKind lk, bool nocomp, LaunchPlan &L,
                int grid_override = 0);
cudaError_t reset_run_counters(Slab &s, cudaStream_t st);
int read_status(Slab &s);
std::vector<std::vector<int>> launch_groups(jacobi_ctx *h);
int plan_resident(jacobi_ctx *h, const std::vector<int> &idx, LaunchPlan &L);
bool resident_fits_all(jacobi_ctx *h);
int setup_norm(jacobi_ctx *h, LaunchPlan &L);
int setup_trace(jacobi_ctx *h, LaunchPlan &L);
int run_cpufree(jacobi_ctx *h, int64_t iters);
int run_cpufree_k1(jacobi_ctx *h, int64_t iters);
int run_tblock(jacobi_ctx *h, int64_t iters, int k, int ppt, int lag, int ws);
// Tensor maps of a slab's two buffers for TMA box loads of `cols` x `rows` elements (one plane).
int slab_tensor_maps(jacobi_ctx *h, Slab &s, int cols, int rows);
// Time-block depth and pairs per thread the runtime would use for this handle (K = 0: none).
void tblock_choice(const jacobi_ctx *h, int *k, int *ppt, int *lag, int *ws);
int ensure_nccl(jacobi_ctx *h);
int time_begin(jacobi_ctx *h);
int time_end(jacobi_ctx *h, int64_t iters);
int copy_edges(jacobi_ctx *h, Slab &s, int nxt, cudaStream_t st, bool capturing = false);
int nccl_edges(jacobi_ctx *h, int nxt);
int run_baseline(jacobi_ctx *h, int64_t iters, BaseKind kind);
int run_graph(jacobi_ctx *h, int64_t iters, bool nocomp, std::vector<LaunchPlan> &plans);
}  // namespace jbrt
