// resident.cu — the PERKS-style on-chip CPU-Free kernel; see DESIGN.md §5.3.
#include "device_common.cuh"

namespace {

// ---------------------------------------------------------------- resident (on-chip) kernel
// SURVEY §8(f) N2, after PERKS: for slabs small enough to live in
// the shared memory of their CTAs, each CTA keeps one (outer-plane x row) block of the slab — plus
// a one-row halo ring — in shared memory for the whole run.  Per iteration it (1) refreshes only
// the halo ring from L2 (its neighbour blocks' faces; the slab's outer halo after the neighbour
// GPU's flag), (2) computes every owned cell into registers, (3) writes them back to shared memory
// and stores only its faces to the next global buffer — plus, for blocks on the slab's edge
// plane, into the neighbour GPU's halo followed by one sys-scope release of its flag slot
// — and (4) joins the slab's grid barrier.  The full block is written to
// global memory in the last iteration, so buffers are consistent between runs and modes.
// Same fp64 operation order as the oracle.
template <int DIM, int CPP>
__global__ void __launch_bounds__(JB_RNT, 1) jb_resident(const __grid_constant__ JbParams P) {
  extern __shared__ __align__(16) double tile[];
  __shared__ int s_abort, s_abort_pw;
  const JbGeom &g = P.g;
  int si = 0;
  while (si + 1 < P.nslabs && (int)blockIdx.x >= P.s[si + 1].cta_begin) ++si;
  const JbSlab &SL = P.s[si];
  const int c = (int)blockIdx.x - SL.cta_begin;
  const int nby = SL.res_nby;
  const int bz = c / nby, by = c - bz * nby;
  int pz0, zb, y0 = 0, yb = 1;  // 32-bit: resident slabs are < 2^31 elements (host-checked)
  {
    int64_t a, b;
    jbplan_even_split(SL.chunk, SL.res_nbz, bz, &a, &b);
    pz0 = (int)a + 1;  // owned planes pz0 .. pz0+zb-1 (slab planes are 1-based)
    zb = (int)b;
    if (DIM == 3) {
      jbplan_even_split(g.ny - 2, nby, by, &a, &b);
      y0 = (int)a + 1;
      yb = (int)b;
    }
  }
  const int rs = g.res_rs;
  const int YR = DIM == 3 ? yb + 2 : 1;  // smem rows per plane (incl. y halo rows)
  const int pe = (int)g.plane_elems, pitch = (int)g.pitch;
  const int nx = (int)g.nx;
  const int ppr = (nx - 1) / 2;               // pairs per row: x = 1+2j, 2+2j
  const int tid = threadIdx.x;
  const bool has_top = SL.flag_out_top != nullptr, has_bot = SL.flag_out_bot != nullptr;
  const bool top_blk = has_top && bz == 0, bot_blk = has_bot && bz == SL.res_nbz - 1;
  // smem row of (lz, ly), lz in [-1, zb], ly in [-1, yb] (ly ignored in 2D)
  auto srow = [&](int lz, int ly) { return ((lz + 1) * YR + (DIM == 3 ? ly + 1 : 0)) * rs; };
  // global element offset of (plane pz0+lz, row y0+ly, x) in a slab buffer
  auto goff = [&](int lz, int ly, int x) {
    return (pz0 + lz) * pe + (DIM == 3 ? (y0 + ly) * pitch : 0) + 3 + x;
  };

  // ---- this thread's cell pairs (fixed for the run)
  int soff[CPP];
  int gofs[CPP];  // element offsets inside the slab buffer (host checks the slab is < 2^31 elements)
  unsigned valid = 0, full = 0, face = 0, top_face = 0, bot_face = 0;
  const int nrows = zb * yb;
#pragma unroll
  for (int i = 0; i < CPP; ++i) {
    const int k = tid + i * JB_RNT;
    const int r = k / ppr, j = k - r * ppr;
    const int lz = DIM == 3 ? r / yb : r, ly = DIM == 3 ? r - lz * yb : 0;
    const int x = 1 + 2 * j;
    soff[i] = srow(lz, ly) + x + 1;
    gofs[i] = (int)goff(lz, ly, x);
    if (r < nrows) {
      valid |= 1u << i;
      if (x + 1 <= nx - 2) full |= 1u << i;
      const bool f = lz == 0 || lz == zb - 1 || (DIM == 3 && (ly == 0 || ly == yb - 1));
      if (f) face |= 1u << i;
      if (top_blk && lz == 0) top_face |= 1u << i;
      if (bot_blk && lz == zb - 1) bot_face |= 1u << i;
    }
  }
  if (tid == 0) s_abort = s_abort_pw = 0;
  // neighbour blocks (face-sharing) for the relaxed synchronisation
  const bool relaxed = SL.res_relaxed != 0;
  int nbr[4], n_nbr = 0;
  if (bz > 0) nbr[n_nbr++] = c - nby;
  if (bz < SL.res_nbz - 1) nbr[n_nbr++] = c + nby;
  if (DIM == 3 && by > 0) nbr[n_nbr++] = c - 1;
  if (DIM == 3 && by < nby - 1) nbr[n_nbr++] = c + 1;

  // ---- whole block + ring (incl. the x boundary cells) at run start: flattened over all threads
  auto load_all = [&](const double *src) {
    const int nrow = (zb + 2) * YR;
    for (int k = tid; k < nrow * nx; k += JB_RNT) {
      const int rr = k / nx, x = k - rr * nx;
      const int lz = rr / YR - 1, ly = DIM == 3 ? rr % YR - 1 : 0;
      tile[srow(lz, ly) + 1 + x] = __ldcg(src + goff(lz, ly, x));
    }
  };
  // ---- halo ring only (interior x), one 16-byte pair per thread per step: ring row rr is
  //      2D: lz = -1, zb;  3D: (lz = -1 | zb, ly = 0..yb-1) then (ly = -1 | yb, lz = 0..zb-1)
  const int ring_rows = DIM == 3 ? 2 * yb + 2 * zb : 2;
  auto load_ring = [&](const double *src) {
    for (int k = tid; k < ring_rows * ppr; k += JB_RNT) {
      const int rr = k / ppr, q = k - rr * ppr;
      int lz, ly;
      if (DIM == 2) {
        lz = rr == 0 ? -1 : zb;
        ly = 0;
      } else if (rr < 2 * yb) {
        lz = rr < yb ? -1 : zb;
        ly = rr < yb ? rr : rr - yb;
      } else {
        const int r2 = rr - 2 * yb;
        ly = r2 < zb ? -1 : yb;
        lz = r2 < zb ? r2 : r2 - zb;
      }
      const int x = 1 + 2 * q;
      const double *gp = src + goff(lz, ly, x);
      double *sp = tile + srow(lz, ly) + 1 + x;
      if (x + 1 <= nx - 2) *reinterpret_cast<double2 *>(sp) = __ldcg(reinterpret_cast<const double2 *>(gp));
      else *sp = __ldcg(gp);
    }
  };

  for (int64_t t = 0; t < P.iters; ++t) {
    const int64_t tg = P.t0 + t;
    const double *cur = SL.buf[tg & 1];
    double *nxt = SL.buf[(tg + 1) & 1];
    // (1) halo: wait for the neighbour GPU's edge plane (and, with relaxed sync, for the
    //     neighbour blocks' faces of the previous iteration), then refresh the ring from L2
    // (with the grid barrier, boundary blocks acquired the neighbour's flag during the last
    //  barrier: the pre-wait below)
    if (t > 0 && relaxed) {
      if (tid == 0 && by == 0) {
        if (top_blk) halo_mark(SL, P, 0, t, 0);
        if (bot_blk) halo_mark(SL, P, 1, t, 0);
      }
      if (tid < 32) {
        bool ok = true;
        if (top_blk) ok &= wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)tg, P, tid);
        if (bot_blk) ok &= wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)tg, P, tid);
        if (relaxed) ok &= wait_slots_idx(SL.blk_flags, nbr, n_nbr, (unsigned long long)tg, P, tid);
        if (tid == 0 && !ok) s_abort = 1;
        if (tid == 0 && by == 0) {
          if (top_blk) halo_mark(SL, P, 0, t, 1);
          if (bot_blk) halo_mark(SL, P, 1, t, 1);
        }
      }
      __syncthreads();
      if (s_abort) return;
    }
    if (t == 0) load_all(cur);
    else load_ring(cur);
    __syncthreads();
    // (2) compute every owned pair into registers (oracle order)
    double2 v[CPP];
#pragma unroll
    for (int i = 0; i < CPP; ++i) {
      if (valid >> i & 1u) {
        const double *cc = tile + soff[i];
        const double2 C = lds2(cc);
        const double w = cc[-1], e = cc[2];
        if (DIM == 2) {
          const double2 N = lds2(cc + rs), S = lds2(cc - rs);  // y+1 / y-1 = next / previous plane
          v[i].x = 0.25 * (((C.y + w) + N.x) + S.x);
          v[i].y = 0.25 * (((e + C.x) + N.y) + S.y);
        } else {
          const double2 N = lds2(cc + rs), S = lds2(cc - rs);            // y+1, y-1
          const double2 U = lds2(cc + YR * rs), D = lds2(cc - YR * rs);  // z+1, z-1
          v[i].x = kC6 * (((((C.y + w) + N.x) + S.x) + U.x) + D.x);
          v[i].y = kC6 * (((((e + C.x) + N.y) + S.y) + U.y) + D.y);
        }
      }
    }
    __syncthreads();
    // (3) write back; faces (all cells in the last iteration) to the next buffer; edge-plane
    //     cells also into the neighbour GPU's halo
    const bool last = t == P.iters - 1;
    double *rt = top_blk ? SL.peer_top[(tg + 1) & 1] : nullptr;
    double *rb = bot_blk ? SL.peer_bot[(tg + 1) & 1] : nullptr;
#pragma unroll
    for (int i = 0; i < CPP; ++i) {
      if (valid >> i & 1u) {
        const bool fl = full >> i & 1u;
        double *sp = tile + soff[i];
        if (fl) *reinterpret_cast<double2 *>(sp) = v[i];
        else sp[0] = v[i].x;
        if (last || (face >> i & 1u)) {
          double *gp = nxt + gofs[i];
          if (fl) __stcg(reinterpret_cast<double2 *>(gp), v[i]);
          else __stcg(gp, v[i].x);
        }
        // the peer halo plane has the same in-plane layout: drop this block's plane offset
        if (top_face >> i & 1u) store_pair(rt + (gofs[i] - pz0 * pe), v[i].x, v[i].y, fl);
        if (bot_face >> i & 1u) store_pair(rb + (gofs[i] - (pz0 + zb - 1) * pe), v[i].x, v[i].y, fl);
      }
    }
    // Signal: with the grid barrier the block's next action is its arrival, so the
    // flag(s) share the arrival's release fence (slab_barrier; one fence instead of two
    // serialised ones); with relaxed sync a release store of its own.
    unsigned long long *sig_top = nullptr, *sig_bot = nullptr;
    if (top_blk || bot_blk) {
      if (relaxed) __syncthreads();  // every thread's peer stores precede thread 0's release (CTA scope)
      if (tid == 0 && !((P.flags & JACOBI_FLAG_DROP_SIGNAL) && SL.slab_id == 0)) {
        if (relaxed) {
          if (top_blk) st_release_flag(P, SL.flag_out_top + by, (unsigned long long)(tg + 1));
          if (bot_blk) st_release_flag(P, SL.flag_out_bot + by, (unsigned long long)(tg + 1));
        } else {
          if (top_blk) sig_top = SL.flag_out_top + by;
          if (bot_blk) sig_bot = SL.flag_out_bot + by;
        }
        if (by == 0) {
          if (top_blk) halo_mark(SL, P, 0, t, 2);
          if (bot_blk) halo_mark(SL, P, 1, t, 2);
        }
      }
    }
    // (4) grid barrier of the slab, or with relaxed sync only a release of this block's
    //     flag: its neighbours wait for it before reading its faces (and nobody else needs to)
    __syncthreads();
    if (relaxed) {
      if (tid == 0) st_release_gpu(SL.blk_flags + c, (unsigned long long)(tg + 1));
      continue;
    }
    if (tid < 32) {
      const bool ok = slab_barrier(SL, P, c, (unsigned long long)(t + 1), (unsigned long long)(tg + 1), tid,
                                   sig_top ? sig_top : sig_bot, (unsigned long long)(tg + 1),
                                   sig_top ? sig_bot : nullptr);
      if (tid == 0) s_abort = ok ? 0 : 1;  // (slab_barrier also reports an abort flag)
    } else if (tid < 64 && (top_blk || bot_blk) && t + 1 < P.iters) {
      // Pre-wait (P:394's wait, off the critical path): the neighbour raises the next
      // iteration's flag in its own iteration t, independent of this slab's barrier, so warp 1
      // polls it while warp 0 spins on the barrier instead of paying an L2 round trip after it.
      const int ln = tid - 32;
      if (ln == 0 && by == 0) {
        if (top_blk) halo_mark(SL, P, 0, t + 1, 0);
        if (bot_blk) halo_mark(SL, P, 1, t + 1, 0);
      }
      bool ok = true;
      if (top_blk) ok &= wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(tg + 1), P, ln);
      if (bot_blk) ok &= wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(tg + 1), P, ln);
      if (ln == 0 && !ok) s_abort_pw = 1;
      if (ln == 0 && by == 0) {
        if (top_blk) halo_mark(SL, P, 0, t + 1, 1);
        if (bot_blk) halo_mark(SL, P, 1, t + 1, 1);
      }
    }
    __syncthreads();
    if (s_abort || s_abort_pw) return;
  }
  // End of run: the neighbours' last halo planes have landed before the kernel completes.
  if (tid < 32 && P.iters > 0) {
    if (top_blk) wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(P.t0 + P.iters), P, tid);
    if (bot_blk) wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(P.t0 + P.iters), P, tid);
  }
}

}  // namespace

namespace jbk {

const void *resident_fn(int dim, int cpp) {
#define JB_RES(D, C) reinterpret_cast<const void *>(&jb_resident<D, C>)
  if (dim == 2) {
    switch (cpp) { case 1: return JB_RES(2, 1); case 2: return JB_RES(2, 2); case 4: return JB_RES(2, 4);
                   default: return JB_RES(2, 8); }
  }
  switch (cpp) { case 1: return JB_RES(3, 1); case 2: return JB_RES(3, 2); case 4: return JB_RES(3, 4);
                 default: return JB_RES(3, 8); }
#undef JB_RES
}

cudaError_t prepare_resident(int dim, int cpp, size_t smem, int *blocks_per_sm) {
  const void *fn = resident_fn(dim, cpp);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, fn, JB_RNT, smem);
}

cudaError_t launch_resident(const JbParams &p, int cpp, int grid, size_t smem, cudaStream_t st) {
  void *args[] = {const_cast<JbParams *>(&p)};
  return cudaLaunchCooperativeKernel(resident_fn(p.g.dim, cpp), dim3(grid), dim3(JB_RNT), args, smem, st);
}

}  // namespace jbk
