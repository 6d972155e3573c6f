/*
 * jacobi.h — C ABI of the B200-native CPU-Free Jacobi library (libjacobi_b200.so).
 *
 * What the library computes (PAPER.md = /root/reference/PAPER.md):
 *   The Jacobi method for the Laplace equation with Dirichlet data on the domain boundary
 *   (§2.1), on a 2D 5-point ("2D5pt", Fig. 4.1) or 3D 7-point ("3D7pt",
 *   P:535 §6.1.1) grid, for a fixed number of iterations (Listing 4.1), every
 *   iteration reading only the previous time step (§4.1.1).  The grid is divided
 *   equally into slabs along its outermost axis (y in 2D, z in 3D) with one halo plane on
 *   each side, one slab per GPU.
 *   In the CPU-Free mode (Ch.3-4) every iteration runs inside ONE persistent kernel per GPU
 *   (§3.1.1): boundary thread blocks wait on a flag from their neighbour, compute
 *   the edge plane, store it straight into the neighbour GPU's halo over NVLink and raise the
 *   neighbour's flag (Listing 4.1), interior thread blocks stream
 *   the bulk, and a device-side grid barrier ends the iteration.
 *   The CPU-controlled comparison modes launch kernels every iteration and move halos with
 *   cudaMemcpyPeerAsync, NCCL send/recv or in-kernel peer stores, with a host synchronisation
 *   per iteration (Listing 2.1a), or replay the loop as a CUDA graph.
 *
 * Numerics (readings R1-R4): IEEE fp64, per interior cell
 *   2D: new = 0.25 * (((u[x+1] + u[x-1]) + u[y+1]) + u[y-1])
 *   3D: new = fl(1/6) * (((((u[x+1] + u[x-1]) + u[y+1]) + u[y-1]) + u[z+1]) + u[z-1])
 *   no FMA contraction, no flush-to-zero: results are bitwise identical to the CPU oracle and
 *   independent of the number of GPUs, the mode and the tiling.
 *
 * Field layout seen by the caller (scatter/gather): C-contiguous fp64 array of nx*ny*nz
 * doubles, x fastest, idx = (z*ny + y)*nx + x; 2D has nz == 1.  Extents INCLUDE the one-cell
 * Dirichlet layer on every face; only interior cells (1..n-2 on every axis) are ever updated.
 *
 * Error behaviour: every int-returning call returns JACOBI_OK (0) or a negative JACOBI_E*
 * code; after any error the handle remains valid for jacobi_destroy.  A handle is used by one
 * host thread at a time (not re-entrant).  Calls block until their GPU work is complete.
 * Ownership: the library owns all device memory and peer mappings it creates; the caller owns
 * every host array it passes (pageable or pinned; copies are synchronous).
 */
#ifndef JACOBI_B200_H
#define JACOBI_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- error codes --------------------------------------------------------------------- */
#define JACOBI_OK        0
#define JACOBI_EINVAL   -1  /* bad argument (extents < 3, stencil/nz mismatch, slab < 2 planes when P > 1, ...) */
#define JACOBI_ENODEV   -2  /* requested more GPUs than visible / bad device index */
#define JACOBI_ENOPEER  -3  /* cudaDeviceCanAccessPeer failed for a neighbour pair */
#define JACOBI_ENOCOOP  -4  /* no cooperative launch, or the persistent grid is not co-resident */
#define JACOBI_ENOMEM   -5  /* device or host allocation failed */
#define JACOBI_ECUDA    -6  /* any other CUDA runtime error */
#define JACOBI_ETIMEOUT -7  /* device watchdog fired: a neighbour never signalled (state undefined) */
#define JACOBI_ENCCL    -8  /* NCCL unavailable or failed */
#define JACOBI_ESTATE   -9  /* call not valid in this handle's state (e.g. peers not attached) */

/* ---- modes for jacobi_set_mode --------------------------------------------------------- */
#define JACOBI_MODE_CPUFREE          0  /* persistent TB-specialised kernel, device-side flags (default) */
#define JACOBI_MODE_BASELINE_MEMCPY  1  /* per-iteration kernel + cudaMemcpyPeerAsync + host sync */
#define JACOBI_MODE_BASELINE_NCCL    2  /* per-iteration kernel + ncclSend/ncclRecv + host sync */
#define JACOBI_MODE_BASELINE_OVERLAP 3  /* boundary kernel + copies on a comm stream, interior kernel
                                           on the compute stream, host sync ("Overlap") */
#define JACOBI_MODE_BASELINE_P2P     4  /* per-iteration kernel whose boundary blocks store into the
                                           peers' halos (GPU-initiated data, host sync) */
#define JACOBI_MODE_BASELINE_GRAPH   5  /* the MEMCPY loop captured once into a CUDA graph with
                                           cross-GPU event edges, one host launch per run */
#define JACOBI_MODE_BASELINE_NVSHMEM 6  /* NVSHMEM variant only: per iteration a discrete kernel whose
                                           boundary blocks put halos with NVSHMEM, then a dedicated
                                           neighbour-sync kernel; no host barrier */

/* ---- flags for jacobi_set_mode --------------------------------------------------------- */
#define JACOBI_FLAG_NO_COMPUTE   1  /* measurement only: skip the stencil
                                       arithmetic and interior sweep, keep halo copies, flags and
                                       barriers.  The field is NOT a Jacobi result afterwards. */
#define JACOBI_FLAG_DROP_SIGNAL  2  /* debug: slab 0 never raises its neighbours' flags (tests the
                                       watchdog; the run must return JACOBI_ETIMEOUT) */

typedef struct jacobi_ctx *jacobi_t; /* opaque, library-owned */

/* ---- creation ---------------------------------------------------------------------------
 * All creators validate: nx, ny >= 3; stencil == 5 with nz == 1, or stencil == 7 with nz >= 3;
 * nslabs >= 1; if nslabs > 1 every slab owns >= 2 outer planes (chunk sizes follow
 * jacobi_decompose).  The field is initialised on the device with the U12 generator
 * (seed 0x5C24), so create -> run -> gather needs no host upload. */

/* Single process, one slab per GPU on devices 0..ngpus-1, peer access enabled between
 * neighbours (P:321-323 UVA load/store).  ngpus == 1 is the 1-GPU path. */
int jacobi_create(int64_t nx, int64_t ny, int64_t nz, int stencil, int ngpus, jacobi_t *out);

/* Single process, `nslabs` slabs on ONE device, all driven by one cooperative launch in which
 * each slab gets its own group of thread blocks, grid barrier, flags and "peer" pointers into
 * the other slabs' buffers.  Exercises the complete multi-GPU protocol on one GPU (the
 * SURVEY.md §4.2 "virtual PE" backend).  1 <= nslabs <= 8. */
int jacobi_create_virtual(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs,
                          int device, jacobi_t *out);

/* One process per GPU (torchrun): this process owns slab `rank` of `world_size` on `device`.
 * Before the first run, exchange jacobi_get_ipc_handle() blobs with the neighbours (any
 * transport; the Python binding uses torch.distributed) and call jacobi_open_peers().
 * All dist-mode calls that touch the protocol (run, set_mode) are collective over ranks. */
int jacobi_create_rank(int64_t nx, int64_t ny, int64_t nz, int stencil, int world_size,
                       int rank, int device, jacobi_t *out);
int jacobi_ipc_handle_bytes(void);                     /* size of the blob below */
int jacobi_get_ipc_handle(jacobi_t h, void *out);      /* CUDA IPC handles of this rank's buffers + flags */
int jacobi_open_peers(jacobi_t h, const void *top_blob, const void *bottom_blob); /* NULL = no neighbour */
/* Like jacobi_open_peers, given the blobs of ALL ranks (world * jacobi_ipc_handle_bytes(), in rank
 * order): also opens every rank's control block, which the residual-norm all-reduce needs. */
int jacobi_open_ranks(jacobi_t h, const void *blobs, int world);
/* NCCL baseline in dist mode: rank 0 creates a 128-byte ncclUniqueId, every rank passes it to
 * jacobi_nccl_init (collective).  libnccl.so.2 is loaded with dlopen (RTLD_LOCAL) on first use —
 * the file named by the environment variable JACOBI_NCCL_LIB if set (the Python binding sets it
 * to the NCCL PyTorch ships, so the process never holds two different libnccl.so.2), else the
 * default search path. */
int jacobi_nccl_unique_id(void *out128);
int jacobi_nccl_init(jacobi_t h, const void *id128);

/* ---- device memory ------------------------------------------------------------------------
 * The two field buffers and the control block of every slab are obtained from an allocator:
 * cudaMalloc/cudaFree by default, or the caller's (e.g. PyTorch's caching allocator, installed by
 * the Python binding's use_torch_allocator(); the north star's "PyTorch used for device memory").
 * alloc(bytes, device, user) must return device memory on `device`, 16-byte aligned, or NULL;
 * free(ptr, device, user) releases it.  Captured by each handle at creation; pass NULL, NULL to
 * restore cudaMalloc.  Returns JACOBI_EINVAL if exactly one of the two is NULL. */
typedef void *(*jacobi_alloc_fn)(size_t bytes, int device, void *user);
typedef void (*jacobi_free_fn)(void *ptr, int device, void *user);
int jacobi_set_allocator(jacobi_alloc_fn alloc, jacobi_free_fn free_fn, void *user);
/* Bytes of ONE field buffer of slab `slab` (of `nslabs`) for this grid (host-only helper):
 * (chunk + 2) planes (owned + halos) + the time-blocked kernel's edge-zone scratch
 * (DESIGN.md §5.7-5.9): 34 planes in 2D (time blocks up to K = 5), 11 in 3D (K <= 3), + 8 doubles
 * of read slack (the edge zones' 16-byte pair loads at the last grid column). */
int jacobi_slab_bytes(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs, int slab, int64_t *bytes);

/* ---- NVSHMEM variant — exported ONLY by libjacobi_b200_nvshmem.so --------
 * Same library built with -DJB_NVSHMEM: one PE per process; the slab buffers and control blocks
 * live on the NVSHMEM symmetric heap and the CPU-Free kernel's boundary blocks deliver halos with
 * nvshmemx_putmem_signal_nbi_warp / nvshmem signals (the paper's own layer) instead
 * of raw peer stores.  Rank 0 calls jacobi_nvshmem_uid(); every rank passes that id (any
 * transport) to jacobi_create_nvshmem (collective, once per process; NVSHMEM_SYMMETRIC_SIZE is
 * set from the grid if unset).  jacobi_destroy is collective for these handles; call
 * jacobi_nvshmem_finalize() before process exit.  Baseline modes are not available here. */
int jacobi_nvshmem_uid_bytes(void);
int jacobi_nvshmem_uid(void *out);
int jacobi_create_nvshmem(int64_t nx, int64_t ny, int64_t nz, int stencil, const void *uid, int world_size,
                          int rank, int device, jacobi_t *out);
int jacobi_nvshmem_finalize(void);

/* ---- running ----------------------------------------------------------------------------- */
/* Advance the field by `iters` Jacobi iterations in the current mode (the fixed iteration count
 * of P:355, Listing 4.1 "for (iter = 0; iter < iter_max; ...)").  CPU-Free mode: ONE persistent
 * cooperative launch per GPU for all `iters` (§3.1.1, §4.1.1) — the only host
 * action of the run; baseline modes: one host-driven launch + halo copy +
 * host sync per iteration (Listing 2.1a).  Continues from the current state:
 * run(a); run(b) == run(a+b) bitwise (every iteration reads only the previous time step).
 * run(0) is a no-op.  iters < 0: JACOBI_EINVAL; peers not attached (dist mode): JACOBI_ESTATE;
 * a neighbour that never signals: JACOBI_ETIMEOUT (watchdog, field undefined).  Blocks until done. */
int jacobi_run(jacobi_t h, int64_t iters);
/* Select how later runs are orchestrated (JACOBI_MODE_*, the paper's CPU-Free model vs the
 * CPU-controlled baselines of P:528-531) and measurement flags (JACOBI_FLAG_*, the no-compute
 * runs of P:550-552).  Unknown mode / flag bits: JACOBI_EINVAL.  Collective in dist mode. */
int jacobi_set_mode(jacobi_t h, int mode, int flags);
/* Tuning knobs (none changes results): "tile_x", "tile_y", "stages", "boundary_ctas",
 * "ctas" (persistent grid size per slab group, 0 = all co-resident), "schedule" (interior
 * work distribution: -1 auto = 2 for grids of >= 2^17 interior cells per CTA of the job, else 0;
 * 0 static linear, 1 static lockstep, 2 dynamic guided self-scheduling), "min_block" (smallest dynamic block, planes, default 8), "dyn_help"
 * (1: boundary blocks join the dynamic interior after signalling), "resident" (CPU-Free runs
 * with compute keep each slab on chip — PERKS-style, P:335-337, P:406-408 — when it fits in the
 * shared memory/registers of its CTAs: -1 auto (default), 0 never, 1 always (EINVAL if it does
 * not fit)), "block_sync" (resident kernel: 0 = default, device-wide grid barrier per iteration
 * as in P:372; 1 = each block waits only for its face-sharing neighbour blocks' flags),
 * "l2hint" (streaming loads with L2 evict_first / evict_last policies; default off — measured
 * 2-3 % slower on B200), "timeout_ms" (watchdog, default 20000), "tblock" (CPU-Free runs with
 * compute advance K iterations per pass over HBM — temporal blocking; slabs
 * with neighbours keep the per-iteration halo exchange through edge zones, which need 2K planes
 * per slab — for every whole multiple of K iterations (2K for K = 2), the rest per iteration:
 * -1 auto (default: a single slab — except 2D slabs that fit on chip, which use the resident
 * kernel, unless of >= 2^18 interior cells; slabs with neighbours when the grid has >= 2^16 (2D) /
 * 3 x 2^16 (3D, and >= 64 CTAs per slab) interior cells per CTA of the job), 0 never, 1 always (EINVAL when a slab has < 2K planes with P > 1,
 * with the norm, in no-compute mode or in the NVSHMEM variant)), "tb_k" (iterations per time block: -1 auto = 5 in
 * 2D, 3 in 3D; 2D accepts 2, 3, 5, 3D 2, 3 — a deeper K than the slabs fit falls back to 3, then 2),
 * "tb_ppt" (2D cell pairs per lane and level: K = 2: from tile_x; K = 3: 2 or 4; K = 5: 1 (default,
 * 11 consumer warps) or 2 (7 warps); 3D K = 3: 1 (default) or 2), "tb_rpw" (3D K = 3: rows per
 * warp, 2 (default, 11 warps) or 3 (7 warps)),
 * "tb_ws" (warp-specialised register split of the time-blocked kernel — 12 compute warps at 160
 * registers via setmaxnreg, built for 2D K = 5 / 1 pair per lane and 3D K = 3 / 2 rows per warp:
 * -1 auto (default: where built), 0 off), "tb_lag" (odd K: wavefront skew between levels, 1 default or 2), "tb_min_block" (smallest
 * dynamic plane block of that kernel, default 16), "tb_ctas" (its CTAs per SM, 1 or 2; 2 only
 * for K = 2 and P = 1).  Read-only: "last_resident" (1 if the last CPU-Free run used the resident
 * kernel), "last_tblock" (iterations of the last CPU-Free run done time-blocked), "last_tb_k"
 * (its K, 0 if none), "last_tb_ws" (1 if it used the register split), "last_launches" (kernels this process launched in the last jacobi_run, all
 * GPUs).  Measurement: "halo_trace" (see jacobi_halo_trace; 0 = off, <= 2^20).
 * "barrier" (the CPU-Free kernels' device-side grid barrier: 0 = one counter per slab with
 * red.release + acquire spin (default), 1 = per-CTA arrival flags polled in parallel by every CTA).
 * "cluster" (CPU-Free runs of ONE 2D slab that fits in the shared memory of one thread-block
 * cluster of <= 16 CTAs, both time levels: the whole grid stays on chip, halo rows between the
 * cluster's CTAs are read through DSMEM and the iteration barrier of P:372 is the hardware cluster
 * barrier; with compute, no norm: -1 auto (default: used while "resident" and "tblock" are auto
 * too — C1 2D 256^2 1.29 vs 2.33 us/iteration), 0 never, 1 always (EINVAL where it does not
 * apply)); read-only "last_cluster" (its cluster size in the last CPU-Free run, 0 if not used).
 * "halo_ll" (streaming CPU-Free kernel, not with the norm: halo cells travel as tagged 16-byte LL
 * cells {tag:lo32, tag:hi32} that the receiving boundary CTAs poll and unpack into their halo
 * plane, instead of plain peer stores + one sys-scope release flag per boundary CTA and
 * iteration (P:394's signal); the first / last halo of every run keep the flags, so runs of every
 * kind mix.  -1 auto (default: off), 0 off, 1 on.  DESIGN.md §5.11: removes the 1.5-3.9 us
 * MEMBAR.SYS of each release but doubles the halo bytes — measured equal or slower except 2D
 * no-compute / latency runs at 4-8 slabs).
 * "flag_scope" (memory scope of the halo flags' release store and acquire poll, P:364-365 /
 * P:394's signal and wait: -1 auto (default: .gpu for virtual slabs — every neighbour is a thread
 * block group of the same launch on the same GPU — and .sys otherwise, which a neighbour on another
 * GPU or in another process needs), 0 .sys always, 1 .gpu (EINVAL unless the handle was made by
 * jacobi_create_virtual).  DESIGN.md §5.13: a .sys release costs 1.5-3.9 us, a .gpu one 0.4 us.
 * Unknown names return JACOBI_EINVAL. */
int jacobi_set_param(jacobi_t h, const char *name, int64_t value);
int jacobi_get_param(jacobi_t h, const char *name, int64_t *value);

/* Residual norm and convergence (not in the paper, which runs a fixed count):
 * with the knob "norm_every" = k > 0, CPU-Free runs with compute check the update norm
 * sqrt(sum over interior cells of (u_new - u_old)^2) after every k-th iteration of the run — an
 * all-reduce over every GPU done on the devices (each slab writes its sum into every slab's
 * control block and raises a flag) — and stop after the first check with norm <= tol.  The sum
 * order is fixed, so the norm and the stop decision are identical on every GPU and reproducible.
 * jacobi_iterations() then tells how many iterations ran; jacobi_last_norm() the last norm
 * (-1 before any check).  Uses the dynamic schedule and the streaming kernel; <= 32 slabs. */
int jacobi_set_tolerance(jacobi_t h, double tol);
int jacobi_last_norm(jacobi_t h, double *norm);

/* ---- data movement -------------------------------------------------------------------- */
/* Set the whole field (boundary included: the Dirichlet data of P:197 is whatever the caller's
 * boundary cells hold) from a caller-owned host array `in` of nx*ny*nz doubles (layout above);
 * both device buffers are written (R10), each slab receives its owned planes plus one
 * halo plane per side.  In dist mode only this rank's slab (+ its halos) is read.
 * `in` NULL: JACOBI_EINVAL.  Synchronous (returns after the copies completed). */
int jacobi_scatter(jacobi_t h, const double *in);
/* Write the current field (buf[t & 1], the result of the last completed iteration) into a
 * caller-owned host array `out` of nx*ny*nz doubles (layout above): every slab's owned planes, and
 * the global boundary planes from the first / last slab.  In dist mode only this rank's owned
 * planes (and the global boundary planes it holds) are written; the rest of `out` is untouched.
 * `out` NULL: JACOBI_EINVAL.  Synchronous. */
int jacobi_gather(jacobi_t h, double *out);

/* ---- introspection ---------------------------------------------------------------------- */
/* Device time of the last jacobi_run (the quantity behind the paper's timing method, "minimum
 * of 5 runs", and SURVEY §8(d)): max over this process's GPUs into *ms_max and, if
 * ms_per_slab != NULL (caller array of one double per LOCAL slab), one entry per slab.  CUDA
 * events on each GPU's launch stream around the launch(es) — the persistent kernel in CPU-Free
 * mode, the whole host loop in the baseline modes (host overhead shows as GPU idle time).
 * Multi-process: the caller takes the max over ranks.  h NULL: JACOBI_EINVAL. */
int jacobi_last_time(jacobi_t h, double *ms_max, double *ms_per_slab);
/* Halo-exchange trace of the last CPU-Free run (measurement of P:394's wait -> compute + put ->
 * signal sequence and of the per-iteration halo latency): with the knob "halo_trace"
 * = n > 0, the first boundary thread block of each side of every slab records %globaltimer (ns,
 * per-GPU clock) for the first n exchanges of a run (one exchange = one iteration; the
 * time-blocked kernel's K phases per block are K exchanges): [0] the wait for the neighbour's
 * flag begins, [1] the flag was acquired, [2] this block's own signal was released.  Copies 2 x n
 * x 3 uint64 into `out` (caller-owned): side 0 (top) exchanges 0..n-1, then side 1 (bottom); zero
 * where nothing was recorded (no neighbour on that side, or the event did not happen — e.g. no
 * wait before iteration 0 of the resident kernel).  n larger than the last traced run recorded:
 * JACOBI_ESTATE; bad slab index / NULL: JACOBI_EINVAL. */
int jacobi_halo_trace(jacobi_t h, int slab, uint64_t *out, int64_t n);
int jacobi_iterations(jacobi_t h, int64_t *t);          /* global iteration counter */
int jacobi_num_slabs(jacobi_t h, int *local, int *total);
/* Plan of local slab `i`: out[0..15] = start, chunk, pitch, plane_elems, tile_x, tile_y,
 * units_x, units_y, stages, n_top, n_bot, n_interior, ctas, k_planes, smem_bytes, device. */
int jacobi_describe(jacobi_t h, int i, int64_t *out16);
/* Raw copy of local slab i's buffer `parity` (0/1) in its HBM layout ((chunk+2)
 * planes of plane_elems doubles, halos included) into a caller array of
 * (chunk+2)*plane_elems doubles — for tests of the halo protocol. */
int jacobi_read_slab(jacobi_t h, int i, int parity, double *out);
/* Static English text of a JACOBI_* code ("unknown error" otherwise); never NULL. */
const char *jacobi_strerror(int code);
/* Release everything the handle owns: waits for its streams, frees the slab buffers, control
 * blocks, peer / IPC mappings, NCCL communicators and cached graphs (the halos and
 * flags of P:394 live in those buffers).  NULL-safe (returns JACOBI_OK); valid after any error.
 * NVSHMEM handles: collective.  The handle must not be used afterwards. */
int jacobi_destroy(jacobi_t h);

/* ---- host-only helpers (no GPU needed) ---------------------------------------------------- */
/* Slab decomposition of the interior outer indices 1..n_out-2 into nslabs chunks: with
 * q = (n_out-2) / nslabs, r = (n_out-2) % nslabs, slab g owns q + (g < r) planes starting at
 * global outer index 1 + g*q + min(g, r)  ("divided equally among GPUs"). */
int jacobi_decompose(int64_t n_out, int nslabs, int slab, int64_t *start, int64_t *chunk);
/* The thread-block split of P:398-404 (§4.1.2, garbled formula reconstructed in DESIGN.md
 * reading R11): boundary_TB = TB_total * w_b / (inner + sides * w_b) per side, rounded up,
 * >= 1 per side with a neighbour, >= 1 interior block if there is interior work.
 * out[0..2] = n_top, n_bot, n_interior. */
int jacobi_tb_split(int ctas, int64_t chunk, int has_top, int has_bottom, int64_t units,
                    int override_per_side, int *out3);
/* Geometry chosen for a grid: out[0..7] = pitch, plane_elems, tile_x, tile_y, units_x,
 * units_y, stage_rows, stage_row_doubles.  tile_x/tile_y <= 0 pick defaults. */
/* Host-only (no GPU needed): the auto policies of DESIGN.md §5.14 for a grid split into `nslabs`
 * slabs — one GPU each with `sms` SMs (virtual_slabs = 0), or all on one GPU (virtual_slabs = 1).
 * out4[0] = interior cells per CTA of the whole job, out4[1] = 1 if the per-iteration kernel's
 * interior schedule is dynamic (knob schedule = -1), out4[2] = 1 if CPU-Free runs with compute
 * take the time-blocked kernel (knob tblock = -1; always 1 for one slab), out4[3] = CTAs of the
 * smallest slab.  Functions of the global problem only, so every rank decides the same.
 * Bad extents / stencil, nslabs < 1, sms < 1, out4 NULL: JACOBI_EINVAL. */
int jacobi_auto_policy(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs, int virtual_slabs, int sms,
                       int64_t *out4);
int jacobi_geometry(int64_t nx, int64_t ny, int64_t nz, int stencil, int tile_x, int tile_y,
                    int64_t *out8);
int jacobi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* JACOBI_B200_H */
