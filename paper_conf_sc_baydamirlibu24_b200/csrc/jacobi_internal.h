// jacobi_internal.h — structures shared by the host runtime (runtime.cu, plan.cpp) and the
// device kernels (sweep.cu, resident.cu, util.cu).  Product code only; nothing here is shared with oracle/.
#pragma once
#include <stdint.h>

#define JB_MAX_SLABS 8          // slabs per launch (virtual mode)
#define JB_NCW 8                // consumer warps per CTA
#define JB_NC (JB_NCW * 32)     // consumer threads per CTA
#define JB_THREADS (JB_NC + 32) // + one producer warp (bulk-copy issue)
#define JB_MAX_STAGES 32
#define JB_RQ 4                 // run-descriptor queue depth (producer -> consumers)
#define JB_MAX_NORM 64          // max slabs in the residual-norm all-reduce (N4)
#define JB_MAXK 32              // max boundary CTAs per side (one inbound flag slot each)
#define JB_RNT 512              // threads per CTA of the resident (on-chip) kernel
#define JB_MAX_BLOCKS 1024      // per-slab block flags of the resident kernel
#define JB_RCPP_MAX 8           // max cell pairs per thread held in registers by the resident kernel
#define JB_SMEM_DEFAULT 232448  // B200 opt-in dynamic shared memory per block (227 KB)
#define JB_TB_KMAX2 5           // deepest time block of the 2D time-blocked kernel (tblock.cu)
#define JB_TB_K2D 5             // its default depth (auto; measured fastest)
#define JB_TB_PPT5 1            // default cell pairs per lane at K = 5 (x 11 consumer warps)
#define JB_TB_LAG 1             // default wavefront lag of the odd-K march
#define JB_TB_KMAX3 3           // deepest time block of the 3D time-blocked kernel
#define JB_TB_K3D 3             // its default depth (auto; slabs without neighbours only)
#define JB_CLUSTER_AUTO 1        // cluster = -1 (auto): one-cluster kernel for small single 2D slabs on/off
#define JB_PFLAG_GPU_SCOPE (1 << 30)  // JbParams::flags (internal): every peer of the launch is on this GPU -> halo
                                      // flags released / acquired at .gpu instead of .sys scope (knob flag_scope)
#define JB_LL_AUTO 0             // halo_ll = -1 (auto): LL halo protocol of the streaming kernel on/off
#define JB_DYN_MIN_CELLS (1 << 17)          // auto schedule: dynamic from this many interior cells per CTA (else static)
#define JB_TB2_NB_MIN_CELLS (1 << 16)       // auto: 2D time-blocked kernel for slabs with neighbours from this many cells per CTA
#define JB_TB3_NB_MIN_CELLS (3 << 16)       // ... and 3D (plus >= 64 CTAs per slab)
#define JB_TB_RPW3 2            // 3D odd K: default rows per warp (x 11 warps)

// Scratch planes after each slab buffer for the time-blocked kernel's edge zones of depth K
// (tblock.cu): K-1 slots for the neighbour's intermediate levels + the side's own level-m planes,
// 2K-m of them for m = 1..K-1.  2D buffers carry enough for JB_TB_KMAX2, 3D ones for JB_TB_KMAX3.
static inline int64_t jb_edge_planes_k(int K) { return (K - 1) + (int64_t)(K - 1) * 2 * K - (int64_t)(K - 1) * K / 2; }
static inline int64_t jb_edge_planes(int dim) { return jb_edge_planes_k(dim == 2 ? JB_TB_KMAX2 : JB_TB_KMAX3); }
// Read slack after each field buffer (doubles): the vectorised edge zones load whole 16-byte cell
// pairs and their x neighbours, which at the grid's last column reach up to two doubles past the
// last row of the last scratch plane (the values are never used).
#define JB_BUF_SLACK 8
// Doubles of ONE field buffer of a slab with `chunk` owned planes.
static inline int64_t jb_buf_doubles(int64_t chunk, int dim, int64_t plane_elems) {
  return (chunk + 2 + jb_edge_planes(dim)) * plane_elems + JB_BUF_SLACK;
}

// LL receive area of a slab buffer (JbSlab::ll_in_*): 2 planes of doubles (one 16-byte LL cell per
// cell of the halo plane) per side — side 0 from the top neighbour, 1 from the bottom one — in the
// last 4 edge-scratch planes (the streaming kernel never uses that scratch otherwise).
static inline unsigned long long *jb_ll_area(double *buf, int64_t chunk, int dim, int64_t plane_elems, int side) {
  return reinterpret_cast<unsigned long long *>(buf + (chunk + 2 + jb_edge_planes(dim) - 4 + 2 * side) * plane_elems);
}

// Grid geometry in HBM and the tile shape of the march.
//   element (x, y, z) of slab plane p lives at  buf + p*plane_elems + y*pitch + (x + 3)
//   (2D: plane p IS row y = start-1+p, so there is no y*pitch term).  The +3 shift makes the
//   first interior cell x = 1 16-byte aligned, so 128-bit loads/stores never straddle.
struct JbGeom {
  int64_t nx, ny, nz;
  int64_t pitch;        // doubles per row: round_up(nx + 3, 4)
  int64_t plane_elems;  // 2D: pitch; 3D: ny * pitch
  int32_t dim;          // 2 or 3
  int32_t tx;           // x tile width (power of two >= 8): cells x0 .. x0+tx-1, x0 = 1 + ux*tx
  int32_t txp_shift;    // log2(tx / 2)
  int32_t ty;           // rows per tile (3D), 1 in 2D
  int32_t rh;           // rows per smem stage: 1 (2D) or ty + 2 (3D, y halo rows)
  int32_t ws;           // smem row stride in doubles: tx + 4
  int32_t units_x, units_y, units;
  int32_t stages;       // ring depth
  int32_t stage_doubles;// rh * ws
  int32_t res_rs;       // resident kernel: smem row stride in doubles (x at column x + 1)
  int32_t l2hint;       // streaming loads: 1 = L2 evict_first for rows read once, evict_last for
                        // 3D y-halo rows (read again by the neighbouring tile)
  int32_t xch_doubles;  // time-blocked 3D kernel with K odd: shared-memory row exchange (doubles)
};

struct JbCtrl;
struct JbSlab {
  double *buf[2];                 // local slab, planes 0..chunk+1 (0 and chunk+1 are halos)
  double *peer_top[2];            // top neighbour's plane chunk_top+1 (its bottom halo), per parity
  double *peer_bot[2];            // bottom neighbour's plane 0 (its top halo), per parity
  // Flags: one u64 slot per boundary CTA of the sending side, in the RECEIVER's memory.
  // Sender CTA j of a side sets slot j to the iteration whose halo it delivered (t+1) with one
  // sys-scope release store; the receiver waits until slots 0..k_in-1 all reach t.
  unsigned long long *flag_in_top;   // local [JB_MAXK]; written by the top neighbour's bottom CTAs
  unsigned long long *flag_in_bot;   // local [JB_MAXK]; written by the bottom neighbour's top CTAs
  unsigned long long *flag_out_top;  // = top neighbour's flag_in_bot
  unsigned long long *flag_out_bot;  // = bottom neighbour's flag_in_top
  int32_t k_in_top, k_in_bot;        // boundary CTA counts of the neighbours facing this slab
  unsigned int *side_ctr;            // local [2]: boundary CTAs done per side (reset each run)
  unsigned long long *barrier;       // local grid-barrier counter (reset each run)
  int64_t chunk;
  int32_t cta_begin, cta_count;
  int32_t n_top, n_bot;              // boundary CTAs per side (0: no neighbour on that side)
  int32_t k_planes;                  // static lockstep plane ranges for the interior (0: linear)
  int32_t slab_id;                   // global slab index g
  // Dynamic (guided self-scheduling) interior work, used when dyn_min_blk > 0: items are
  // (plane block, unit) pairs claimed from work_ctr[t & 1] in block-major order; block k has
  // max(dyn_min_blk, ceil(rem * units / (2 * dyn_n))) planes (rem = planes not yet blocked).
  // Item c -> block b = c / units, unit u = c % units; planes lo + dyn_table[b] ..
  // lo + dyn_table[b+1] - 1 (host-built table).  Interior CTA i starts with item i (no claim);
  // further items are dyn_first + atomicAdd(work_ctr[t & 1], 1).
  unsigned int *work_ctr;            // local [2], one per iteration parity
  const int32_t *dyn_table;          // device, nblocks + 1 entries
  int32_t dyn_min_blk;
  int32_t dyn_n;
  int32_t dyn_help;                  // boundary CTAs join the interior after signalling
  int32_t dyn_first;                 // items handed out statically (one per interior CTA)
  int64_t dyn_items;                 // units * number of blocks
  int32_t excl_top, excl_bot;        // interior excludes plane 1 / chunk although n_top/n_bot == 0
                                     // (the inner kernel of the Copy-Overlap baseline)
  int32_t res_nbz, res_nby;          // resident kernel: the slab's (outer x y) block grid
  int32_t res_relaxed;               // resident kernel: 1 = neighbour-block flags instead of the grid barrier
  int32_t pad2;
  unsigned long long *blk_flags;     // resident kernel: per-block "faces of iteration v are stored" flags
  // Residual norm (N4): per-run partial sums of (u_new - u_old)^2 at fixed indices (dynamic item
  // i -> i; boundary unit u of side s -> dyn_items + s*units + u), summed in index order; then an
  // all-reduce over every slab through the JbCtrl norm slots (device array of P ctrl pointers).
  double *partials;
  struct JbCtrl **norm_peers;
  int32_t n_partials;
  int32_t norm_slabs;                // P
  // NVSHMEM variant (N3, libjacobi_b200_nvshmem.so only): peer_top/peer_bot and flag_out_* are
  // symmetric-heap addresses, written with nvshmemx_putmem(_signal)_nbi_warp to these PEs.
  int32_t use_shm;
  int32_t shm_pe_top, shm_pe_bot;
  int32_t pad3;
  // Temporally blocked kernel (tblock.cu): interior level-K planes tb_lo..tb_hi (dynamic items),
  // and the neighbours' intermediate-level slots this slab writes: the top neighbour's bottom
  // scratch (its E_bot) and the bottom neighbour's top scratch (its E_top); slot m-1 holds level m.
  // A slab's own edge scratch: E_top = buf[0] + (chunk+2)*plane_elems, E_bot = buf[1] +
  // (chunk+2)*plane_elems, jb_edge_planes(dim) planes each.
  int64_t tb_lo, tb_hi;
  double *mid_top_out;
  double *mid_bot_out;
  const void *tmap;                  // 3D odd-K time-blocked kernel: CUtensorMap[2] (buf[0], buf[1]) or null
  // Halo-exchange trace (measurement, param halo_trace = n > 0): for the first n exchanges of a run
  // the first boundary CTA of each side records %globaltimer at wait begin / flag acquired /
  // signal released: halo_trace[(side * n + e) * 3 + {0, 1, 2}], side 0 = top, 1 = bottom.
  unsigned long long *halo_trace;
  // Grid barrier with per-CTA arrival flags (knob "barrier" = 1; null: the counter barrier): CTA c
  // stores the barrier's epoch (the global iteration count after it) into bar_flags[c] and warp 0
  // of every CTA polls all cta_count flags — no atomic serialised on one address.
  unsigned long long *bar_flags;
  // LL halo protocol (knob "halo_ll", streaming CPU-Free kernel): every halo cell
  // travels as a 16-byte LL cell {tag:lo32, tag:hi32} (two single-copy-atomic 8-byte words), so
  // the receiver polls the data itself and neither side issues a sys-scope fence per iteration.
  // ll_out_*[p]: the neighbour's receive area for iteration parity p; ll_in_*[p]: this slab's own
  // (from the top / bottom neighbour).  Null: the flag protocol above.  Areas live in the last 4
  // edge-scratch planes of buf[p] (jb_ll_area).
  unsigned long long *ll_out_top[2];
  unsigned long long *ll_out_bot[2];
  const unsigned long long *ll_in_top[2];
  const unsigned long long *ll_in_bot[2];
};

struct JbParams {
  JbGeom g;
  JbSlab s[JB_MAX_SLABS];
  int32_t nslabs;
  int32_t flags;
  int64_t t0;       // global iteration counter at launch
  int64_t iters;
  unsigned long long timeout_ns;
  int *status;      // [0] error code (0 ok), [1] abort flag
  unsigned long long *trace;  // debug (JACOBI_TRACE): per-iteration CTA work-end timestamps, or null
  int32_t norm_every;         // N4: check the update norm after every norm_every-th iteration (0: off)
  int32_t halo_trace_n;       // exchanges recorded per side in JbSlab::halo_trace (0: off)
  double tol;                 // stop after the first check with norm <= tol
  int64_t k0;                 // global number of norm checks before this launch (monotone slots)
};

// Per-slab control block in device memory (one allocation, IPC-exportable).
struct JbCtrl {
  unsigned long long flag_in[2][JB_MAXK];  // [0] from the top neighbour, [1] from the bottom one
  unsigned long long barrier;
  unsigned int side_ctr[2];
  int status[2];
  unsigned int work[2];            // dynamic-schedule claim counters per iteration parity
  long long done_iters;            // N4: iterations the last run performed (written by CTA 0)
  double norm_out;                 // N4: last norm (written by CTA 0 of every slab)
  double norm_val[2][JB_MAX_NORM]; // N4: slab sums of check k, slot [k & 1][slab], written by each slab
  unsigned long long norm_flag[JB_MAX_NORM];  // N4: check count delivered by each slab (monotone)
  unsigned long long pad[26];
};

// ---- host-side planning (plan.cpp) -----------------------------------------------------
namespace jbplan {
int64_t pow2ceil(int64_t v);
void decompose(int64_t n_out, int nslabs, int slab, int64_t *start, int64_t *chunk);
// Fill geometry for tile sizes (tile_x/tile_y <= 0: defaults); returns 0 or -1.
int geometry(int64_t nx, int64_t ny, int64_t nz, int dim, int tile_x, int tile_y, int smem_bytes,
             int stages_req, JbGeom *g);
void tb_split(int ctas, int64_t inner_planes, int has_top, int has_bot, int64_t units,
              int override_per_side, int *n_top, int *n_bot, int *n_int);
// Choose ty (3D) maximising the lockstep utilisation of `n_int` interior CTAs.
int choose_ty(int64_t ny, int units_x, int n_int, int smem_bytes, int ws);
int tallest_ty(int64_t ny, int smem_bytes, int ws);
int lockstep_k(int units, int n_int, int64_t inner_planes);
// Auto policies of DESIGN.md §5.14 (global inputs only: identical on every rank).
int64_t cells_per_cta(int64_t nx, int64_t ny, int64_t nz, int dim, int64_t job_ctas);
bool schedule_dynamic_auto(int64_t cells_per_cta);
bool tblock_neighbours_auto(int dim, int64_t cells_per_cta, int min_slab_ctas);
// Number of plane blocks of the guided dynamic schedule (see JbSlab::dyn_min_blk).
int64_t dyn_blocks(int64_t npl, int units, int n, int min_blk, int32_t *table = nullptr);
// Resident (on-chip) tiling of a slab of `chunk` planes over at most `count` CTAs: nbz x nby
// blocks whose rows (+ halo ring) fit in `smem` bytes and whose cell pairs fit in JB_RNT threads x
// JB_RCPP_MAX registers.  Returns 0 and fills the outputs, or -1 if the slab does not fit.
int resident_tiling(int64_t nx, int64_t ny, int dim, int64_t chunk, int count, int smem, int *nbz, int *nby,
                    int *cpp, size_t *smem_used);
// Even split of n items into k parts: part i has n/k (+1 for the first n%k) items starting at start.
void even_split(int64_t n, int k, int i, int64_t *start, int64_t *len);
size_t smem_bytes(const JbGeom &g);
}  // namespace jbplan
