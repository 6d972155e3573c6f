// sweep.cu — the streaming CPU-Free kernel and the discrete baseline kernels (sm_100a).
//
// jb_sweep<DIM, NOCOMP, PERSIST> is the whole hot path:
//   PERSIST = true : the CPU-Free persistent kernel of PAPER.md Listing 4.1.  The time
//                    loop runs on the device (§3.1.1); thread blocks are specialised
//                    (§3.1.3): TOP/BOTTOM boundary CTAs wait on a flag from
//                    their neighbour ("signal_wait_until ... compared to the
//                    current iteration"), compute the edge plane, store it into the local next
//                    buffer AND straight into the neighbour GPU's halo through a peer pointer
//                    (§3.1.4), then set the neighbour's flag to the next
//                    iteration; INTERIOR CTAs stream the bulk;
//                    a device-side grid barrier closes the iteration.
//   PERSIST = false: the discrete one-iteration kernel of the CPU-controlled baseline
//                    (Listing 2.1a) — same tile code, launched once per iteration.
//
// B200 design: one CTA per SM; inside it one producer warp streams planes of a
// tile from HBM into a shared-memory ring with 1D bulk copies (cp.async.bulk, the TMA engine)
// completing on mbarriers, and 8 consumer warps march the tile along the outer axis (2.5D), so
// every cell is read from HBM once and written once per iteration (16 B/cell).  Arithmetic is
// fp64 in the oracle's order, compiled with -fmad=false (no contraction).
#include "device_common.cuh"

namespace {

// ---------------------------------------------------------------- work schedule
struct Run {
  int32_t unit;
  int64_t p0, p1;  // planes computed: p0..p1 (inclusive), marched in order
};

// Deterministic run list of one CTA for one iteration; producer and consumers enumerate it
// identically.  kind: 0 none, 1 linear range over (unit, plane) pairs in unit-major order,
// 2 lockstep (one unit, one plane range), 3 boundary (units ub..ue-1, one plane each).
struct Sched {
  int kind;
  int32_t units;
  int64_t w, we, npl, lo;
  int32_t ub, ue;
  int64_t plane;
  __device__ bool next(Run &r) {
    if (kind == 1) {
      if (w >= we) return false;
      const int64_t u = w / npl;
      const int64_t e = min(we, (u + 1) * npl);
      r.unit = (int32_t)u;
      r.p0 = lo + (w - u * npl);
      r.p1 = lo + (e - 1 - u * npl);
      w = e;
      return true;
    }
    if (kind == 2) {
      kind = 0;
      r.unit = ub;
      r.p0 = w;
      r.p1 = we;
      return true;
    }
    if (kind == 3) {
      if (ub >= ue) return false;
      r.unit = ub++;
      r.p0 = r.p1 = plane;
      return true;
    }
    return false;
  }
};

__device__ Sched make_sched(const JbGeom &g, const JbSlab &S, int role, int ridx, int rcount) {
  Sched s;
  s.kind = 0;
  s.units = g.units;
  s.w = s.we = s.npl = s.lo = 0;
  s.ub = s.ue = 0;
  s.plane = 0;
  if (role == ROLE_TOP || role == ROLE_BOT) {
    s.kind = 3;
    s.ub = (int32_t)((int64_t)g.units * ridx / rcount);
    s.ue = (int32_t)((int64_t)g.units * (ridx + 1) / rcount);
    s.plane = role == ROLE_TOP ? 1 : S.chunk;
    return s;
  }
  const int64_t lo = (S.n_top || S.excl_top) ? 2 : 1;
  const int64_t hi = (S.n_bot || S.excl_bot) ? S.chunk - 1 : S.chunk;
  const int64_t npl = hi - lo + 1;
  if (npl <= 0 || rcount <= 0) return s;
  if (S.k_planes > 0) {
    const int K = S.k_planes;
    if (ridx >= g.units * K) return s;
    const int u = ridx % g.units, kr = ridx / g.units;
    const int64_t a = lo + npl * kr / K, b = lo + npl * (kr + 1) / K - 1;
    if (b < a) return s;
    s.kind = 2;
    s.ub = u;
    s.w = a;
    s.we = b;
    return s;
  }
  const int64_t W = (int64_t)g.units * npl;
  s.kind = 1;
  s.npl = npl;
  s.lo = lo;
  s.w = W * ridx / rcount;
  s.we = W * (ridx + 1) / rcount;
  return s;
}

// ---------------------------------------------------------------- LL halo protocol
// The flag protocol pays one sys-scope release (MEMBAR.SYS: 1.5 us alone, 3.9 us with every CTA
// issuing one, profiles/r02_ubench_fence.txt) per boundary CTA and iteration.  LL cells carry
// the iteration in each 8-byte word, so a cell is valid exactly when both of its words show the
// tag of the awaited iteration — no fence, no flag.  Tags are a bijective mix of the global
// iteration, odd (never 0, so untouched memory never matches; iterations only grow, so stale
// cells of earlier runs never match either).
__device__ __forceinline__ uint32_t ll_tag(int64_t tg) { return ((uint32_t)tg * 2654435761u ^ 0x6a09e667u) | 1u; }
__device__ __forceinline__ void ll_store(unsigned long long *p, double v, uint32_t tag) {
  const unsigned long long t = (unsigned long long)tag << 32;
  const unsigned long long w0 = t | (uint32_t)__double2loint(v), w1 = t | (uint32_t)__double2hiint(v);
  asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(w0), "l"(w1) : "memory");
}
__device__ __forceinline__ void ll_store_pair(unsigned long long *p, double o0, double o1, bool pair, uint32_t tag) {
  ll_store(p, o0, tag);
  if (pair) ll_store(p + 2, o1, tag);
}
__device__ __forceinline__ ulonglong2 ll_load(const unsigned long long *p) {
  ulonglong2 v;
  asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "l"(p) : "memory");
  return v;
}

// Receiver side: every thread of a boundary CTA polls the LL cells of the halo-plane cells its
// units' edge tiles read (the cells straight above / below the tile: the edge plane's y-1 / y+1
// (2D) or z-1 / z+1 (3D) neighbours) and writes them into the halo plane of the current buffer,
// in batches of 4 independent cells per thread.  False: watchdog / abort.
__device__ bool ll_unpack(const JbGeom &g, const Sched &sc, double *halo, const unsigned long long *ll, uint32_t tag,
                          const JbParams &P) {
  constexpr int B = 4;
  const int nth = blockDim.x;
  const unsigned long long t_start = globaltimer();
  volatile int *abort_flag = P.status + 1;
  for (int u = sc.ub; u < sc.ue; ++u) {
    const int ux = u % g.units_x, uy = u / g.units_x;
    const int64_t x0 = 1 + (int64_t)ux * g.tx;
    const int vx = (int)min((int64_t)g.tx, g.nx - 1 - x0);
    const int64_t y0 = g.dim == 3 ? 1 + (int64_t)uy * g.ty : 0;
    const int vy = g.dim == 3 ? (int)min((int64_t)g.ty, g.ny - 1 - y0) : 1;
    const int n = vx * vy;
    for (int i0 = (int)threadIdx.x; i0 < n; i0 += B * nth) {
      int64_t idx[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int i = i0 + b * nth;
        const int r = i / vx;
        idx[b] = i < n ? (y0 + r) * g.pitch + 3 + x0 + (i - r * vx) : -1;
      }
      ulonglong2 v[B];
      uint32_t cnt = 0;
      while (true) {
        bool ok = true;
#pragma unroll
        for (int b = 0; b < B; ++b)
          if (idx[b] >= 0) {
            v[b] = ll_load(ll + 2 * idx[b]);
            ok &= (uint32_t)(v[b].x >> 32) == tag && (uint32_t)(v[b].y >> 32) == tag;
          }
        if (ok) break;
        if ((++cnt & 63u) == 0) {
          if (*abort_flag) return false;
          if (globaltimer() - t_start > P.timeout_ns) {
            atomicCAS(P.status, 0, JACOBI_ETIMEOUT);
            atomicExch(P.status + 1, 1);
            return false;
          }
        }
      }
#pragma unroll
      for (int b = 0; b < B; ++b)
        if (idx[b] >= 0) halo[idx[b]] = __hiloint2double((int)(uint32_t)v[b].y, (int)(uint32_t)v[b].x);
    }
  }
  return true;
}

// ---------------------------------------------------------------- producer
// Where one tile's stage comes from: the rows of tile `unit` (1 in 2D; ty + 2 in 3D incl. the y
// halo rows), each row the x window [x0-2, x0+tx+2) of 16-byte aligned doubles, one
// cp.async.bulk per row (one row per producer lane).
struct TileSrc {
  const double *base;  // cur + xs + ya*pitch + lane*pitch (plane 0)
  uint32_t row_bytes;
  int nrows;
  __device__ __forceinline__ TileSrc(const JbGeom &g, const double *cur, int32_t unit, int lane) {
    const int ux = unit % g.units_x, uy = unit / g.units_x;
    const int64_t xs = 2 + (int64_t)ux * g.tx;
    const int64_t xe = min(xs + g.tx + 4, g.pitch);
    row_bytes = (uint32_t)((xe - xs) * 8);
    int64_t ya = 0;
    nrows = 1;
    if (g.dim == 3) {
      ya = (int64_t)uy * g.ty;  // = y0 - 1
      const int64_t yb = min(ya + 1 + g.ty, g.ny - 1);
      nrows = (int)(yb - ya + 1);
    }
    base = cur + xs + ya * g.pitch + (int64_t)lane * g.pitch;
  }
};

// Load plane p of a tile into ring position `at` (acquire the stage, arm its full barrier, copy).
__device__ __forceinline__ void produce_stage(const JbGeom &g, const TileSrc &T, int64_t p, const RingPos &at,
                                              const Ring &R, int lane) {
  if (lane == 0) {
    // First pass: waiting on the parity of the (virtual) preceding phase returns at once.
    mbar_wait(&R.empty[at.slot], at.phase ^ 1u);
    mbar_expect_tx(&R.full[at.slot], T.row_bytes * (uint32_t)T.nrows);
  }
  __syncwarp();
  if (lane < T.nrows) {
    double *dst = R.stage(at) + (size_t)lane * g.ws;
    const double *src = T.base + p * g.plane_elems;
    if (g.l2hint)  // y-halo rows (first/last of a 3D stage) are read again by the neighbour tile
      bulk_g2s_hint(dst, src, T.row_bytes, &R.full[at.slot],
                    l2_policy(g.dim == 3 && (lane == 0 || lane == T.nrows - 1)));
    else
      bulk_g2s(dst, src, T.row_bytes, &R.full[at.slot]);
  }
}

// Load planes pf..pl of tile `unit` from `cur` into consecutive ring stages starting at q.
__device__ __forceinline__ void produce_planes(const JbGeom &g, const double *cur, int32_t unit,
                                               int64_t pf, int64_t pl, RingPos &q, const Ring &R,
                                               int lane) {
  const TileSrc T(g, cur, unit, lane);
  for (int64_t p = pf; p <= pl; ++p) {
    produce_stage(g, T, p, q, R, lane);
    q.advance(R.S);
  }
}

// ---------------------------------------------------------------- consumers

// 2D: march one x strip of tx cells over planes (= rows) p0..p1.  Thread ctid owns the
// cell pairs kk = ctid + i*NC (i < PPT), contiguous across lanes (conflict-free 16-byte LDS,
// coalesced 16-byte STG).  Rows y-1 / y are carried in registers along the march, so each
// plane costs one 16-byte LDS + two 8-byte LDS (x-1, x+2) per pair.
template <int PPT, bool NOCOMP, bool NORM>
__device__ __forceinline__ void consume_run_2d(const JbGeom &g, const Ring &R, RingPos &q, const Run &run,
                                               const double *cur, double *nxt, double *remote,
                                               unsigned long long *rll, uint32_t tag, int ctid, int lane,
                                               double &acc) {
  const int64_t x0 = 1 + (int64_t)run.unit * g.tx;
  const int vx = (int)min((int64_t)g.tx, g.nx - 1 - x0);
  const int txp = g.tx >> 1;
  // pair i of this thread: kk = ctid + i*NC, smem column j0 + 2*i*NC, global column col + 2*i*NC
  const int j0 = 2 + 2 * ctid;
  unsigned in_tile = 0, ok = 0, full = 0;
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const int kk = ctid + i * JB_NC;
    in_tile |= (kk < txp ? 1u : 0u) << i;
    ok |= (kk < txp && 2 * kk < vx ? 1u : 0u) << i;
    full |= (2 * kk + 1 < vx ? 1u : 0u) << i;
  }
  const int64_t col = 3 + x0 + 2 * ctid;
  const int64_t L = run.p1 - run.p0 + 1;
  if (NOCOMP) {  // no-compute: the owned edge plane goes to the neighbour as-is,
                 // 16-byte loads straight from the current buffer (L2), no ring stages
    for (int64_t p = 0; p < L; ++p) {
      const double *src = cur + (run.p0 + p) * g.plane_elems + col;
      double2 v[PPT];  // every pair's load issued before the stores (one L2 round trip)
#pragma unroll
      for (int i = 0; i < PPT; ++i)
        if ((ok >> i & 1u) && (remote || rll)) v[i] = __ldcg(reinterpret_cast<const double2 *>(src + 2 * i * JB_NC));
#pragma unroll
      for (int i = 0; i < PPT; ++i)
        if ((ok >> i & 1u) && (remote || rll)) {
          if (rll) ll_store_pair(rll + 2 * (col + 2 * i * JB_NC), v[i].x, v[i].y, full >> i & 1u, tag);
          else store_pair(remote + col + 2 * i * JB_NC, v[i].x, v[i].y, full >> i & 1u);
        }
    }
    return;
  }
  RingPos pm = q, pc = q;
  pc.advance(R.S);
  RingPos pp = pc;
  pp.advance(R.S);
  R.wait_full(pm);
  R.wait_full(pc);
  double2 S[PPT], C[PPT];
#pragma unroll
  for (int i = 0; i < PPT; ++i)
    if (in_tile >> i & 1u) {
      S[i] = lds2(R.stage(pm) + j0 + 2 * i * JB_NC);
      C[i] = lds2(R.stage(pc) + j0 + 2 * i * JB_NC);
    }
  double *dst = nxt + run.p0 * g.plane_elems + col;
  double *rem = remote ? remote + col : nullptr;
  unsigned long long *rl = rll ? rll + 2 * col : nullptr;
  const int64_t pe = g.plane_elems;
  for (int64_t p = 0; p < L; ++p) {
    R.wait_full(pp);
    const double *sc = R.stage(pc) + j0, *sn = R.stage(pp) + j0;
#pragma unroll
    for (int i = 0; i < PPT; ++i)
      if (in_tile >> i & 1u) {
        const double2 N = lds2(sn + 2 * i * JB_NC);
        const double W = sc[2 * i * JB_NC - 1], E = sc[2 * i * JB_NC + 2];
        // oracle order: ((x+1) + (x-1)) + (y+1) + (y-1), then * 0.25
        const double o0 = 0.25 * (((C[i].y + W) + N.x) + S[i].x);
        const double o1 = 0.25 * (((E + C[i].x) + N.y) + S[i].y);
        if (ok >> i & 1u) {
          store_pair(dst + 2 * i * JB_NC, o0, o1, full >> i & 1u);
          if (rl) ll_store_pair(rl + 4 * i * JB_NC, o0, o1, full >> i & 1u, tag);
          else if (rem) store_pair(rem + 2 * i * JB_NC, o0, o1, full >> i & 1u);
          if (NORM) {  // update norm (N4): fixed per-thread order
            const double d0 = o0 - C[i].x;
            acc = acc + d0 * d0;
            if (full >> i & 1u) {
              const double d1 = o1 - C[i].y;
              acc = acc + d1 * d1;
            }
          }
        }
        S[i] = C[i];
        C[i] = N;
      }
    R.release(pm, lane);
    pm = pc;
    pc = pp;
    pp.advance(R.S);
    dst += pe;
  }
  R.release(pm, lane);
  R.release(pc, lane);
  q = pp;
}

// 3D: march one (ty rows x tx cells) tile over z planes p0..p1.  Thread ctid owns the x pair
// kk = ctid % (tx/2) in a contiguous block of rows; along y it carries rows y-1 / y in
// registers, so each cell row costs LDS: 16 B (y+1) + 8 B + 8 B (x-1, x+2) + 16 B (z+1) +
// 16 B (z-1) per pair.
template <bool NOCOMP, bool NORM>
__device__ __forceinline__ void consume_run_3d(const JbGeom &g, const Ring &R, RingPos &q, const Run &run,
                                               const double *cur, double *nxt, double *remote,
                                               unsigned long long *rll, uint32_t tag, int ctid, int lane,
                                               double &acc) {
  const int ux = run.unit % g.units_x, uy = run.unit / g.units_x;
  const int64_t x0 = 1 + (int64_t)ux * g.tx;
  const int vx = (int)min((int64_t)g.tx, g.nx - 1 - x0);
  const int64_t y0 = 1 + (int64_t)uy * g.ty;
  const int vy = (int)min((int64_t)g.ty, g.ny - 1 - y0);
  const int txp = g.tx >> 1;
  const int G = JB_NC / txp;  // row groups
  const int kk = ctid & (txp - 1), rg = ctid / txp;
  const int rpt = (g.ty + G - 1) / G;
  const int rb = rg * rpt, re = min(rb + rpt, vy);
  const int j = 2 + 2 * kk;
  const bool ok = 2 * kk < vx, full = 2 * kk + 1 < vx;
  const int ws = g.ws;
  const int64_t col = (y0 + rb) * g.pitch + 3 + x0 + 2 * kk;
  const int64_t L = run.p1 - run.p0 + 1;
  const int srow = (rb + 1) * ws + j;  // stage offset of (row rb, pair kk) center
  if (NOCOMP) {  // no-compute: the owned edge plane to the neighbour as-is, straight from L2
    for (int64_t p = 0; p < L; ++p) {
      if ((remote || rll) && ok) {
        const double *c = cur + (run.p0 + p) * g.plane_elems + col;
        if (rll) {
          unsigned long long *o = rll + 2 * col;
          for (int r = rb; r < re; ++r, c += g.pitch, o += 2 * g.pitch) {
            const double2 v = __ldcg(reinterpret_cast<const double2 *>(c));
            ll_store_pair(o, v.x, v.y, full, tag);
          }
        } else {
          // loads of up to 4 rows issued before their stores: one L2 round trip per 4 rows on the
          // halo's critical path instead of one per row
          double *o = remote + col;
          for (int r = rb; r < re; r += 4, c += 4 * g.pitch, o += 4 * g.pitch) {
            double2 v[4];
#pragma unroll
            for (int u = 0; u < 4; ++u)
              if (r + u < re) v[u] = __ldcg(reinterpret_cast<const double2 *>(c + u * g.pitch));
#pragma unroll
            for (int u = 0; u < 4; ++u)
              if (r + u < re) store_pair(o + u * g.pitch, v[u].x, v[u].y, full);
          }
        }
      }
    }
    return;
  }
  RingPos pm = q, pc = q;
  pc.advance(R.S);
  RingPos pp = pc;
  pp.advance(R.S);
  R.wait_full(pm);
  R.wait_full(pc);
  double *dst = nxt + run.p0 * g.plane_elems + col;
  double *rem = remote ? remote + col : nullptr;
  unsigned long long *rlb = rll ? rll + 2 * col : nullptr;
  for (int64_t p = 0; p < L; ++p) {
    R.wait_full(pp);
    if (rb < re) {
      const double *c = R.stage(pc) + srow;
      const double *u = R.stage(pp) + srow;
      const double *d = R.stage(pm) + srow;
      double2 S = lds2(c - ws), C = lds2(c);
      double *o = dst, *ro = rem;
      unsigned long long *rl = rlb;
#pragma unroll 2
      for (int r = rb; r < re; ++r) {
        const double2 N = lds2(c + ws);
        const double w = c[-1], e = c[2];
        const double2 U = lds2(u), D = lds2(d);
        // oracle order: x+1, x-1, y+1, y-1, z+1, z-1, then * fl(1/6)
        const double o0 = kC6 * (((((C.y + w) + N.x) + S.x) + U.x) + D.x);
        const double o1 = kC6 * (((((e + C.x) + N.y) + S.y) + U.y) + D.y);
        if (ok) {
          store_pair(o, o0, o1, full);
          if (rl) ll_store_pair(rl, o0, o1, full, tag);
          else if (ro) store_pair(ro, o0, o1, full);
          if (NORM) {  // update norm (N4): fixed per-thread order
            const double d0 = o0 - C.x;
            acc = acc + d0 * d0;
            if (full) {
              const double d1 = o1 - C.y;
              acc = acc + d1 * d1;
            }
          }
        }
        S = C;
        C = N;
        c += ws;
        u += ws;
        d += ws;
        o += g.pitch;
        if (ro) ro += g.pitch;
        if (rl) rl += 2 * g.pitch;
      }
    }
    R.release(pm, lane);
    pm = pc;
    pc = pp;
    pp.advance(R.S);
    dst += g.plane_elems;
  }
  R.release(pm, lane);
  R.release(pc, lane);
  q = pp;
}

template <int DIM, bool NOCOMP, bool NORM>
__device__ __forceinline__ void consume_run(const JbGeom &g, const Ring &R, RingPos &q, const Run &run,
                                            const double *cur, double *nxt, double *remote,
                                            unsigned long long *rll, uint32_t tag, int ctid, int lane,
                                            double &acc) {
  if (DIM == 3) {
    consume_run_3d<NOCOMP, NORM>(g, R, q, run, cur, nxt, remote, rll, tag, ctid, lane, acc);
    return;
  }
  const int ppt = g.tx / (2 * JB_NC);
  if (ppt >= 4) consume_run_2d<4, NOCOMP, NORM>(g, R, q, run, cur, nxt, remote, rll, tag, ctid, lane, acc);
  else if (ppt == 2) consume_run_2d<2, NOCOMP, NORM>(g, R, q, run, cur, nxt, remote, rll, tag, ctid, lane, acc);
  else consume_run_2d<1, NOCOMP, NORM>(g, R, q, run, cur, nxt, remote, rll, tag, ctid, lane, acc);
}

// ---------------------------------------------------------------- run-descriptor queue
// The producer warp decides the work (static runs, then dynamically claimed interior items) and
// hands each run to the consumer warps through a JB_RQ-deep queue of descriptors in shared
// memory, guarded by its own full/empty mbarriers.
enum { RUN_WORK = 0, RUN_SIGNAL = 1, RUN_END = 2 };
struct RunDesc {
  int32_t kind;
  int32_t unit;
  int32_t item;  // N4: partial-sum index of this run
  int32_t pad;
  int64_t p0, p1;
};
struct Queue {
  uint64_t *full, *empty;
  RunDesc *desc;
};

__device__ __forceinline__ void publish(const Queue &Q, RingPos &qp, int kind, const Run &r, int lane,
                                        int item = 0) {
  if (lane == 0) {
    mbar_wait(&Q.empty[qp.slot], qp.phase ^ 1u);
    RunDesc d;
    d.kind = kind;
    d.unit = r.unit;
    d.item = item;
    d.pad = 0;
    d.p0 = r.p0;
    d.p1 = r.p1;
    Q.desc[qp.slot] = d;
    mbar_arrive(&Q.full[qp.slot]);  // release: the descriptor is visible to the waiters
  }
  qp.advance(JB_RQ);
}

__device__ __forceinline__ RunDesc fetch(const Queue &Q, RingPos &qc, int lane) {
  mbar_wait(&Q.full[qc.slot], qc.phase);
  const RunDesc d = Q.desc[qc.slot];
  __syncwarp();
  if (lane == 0) mbar_arrive(&Q.empty[qc.slot]);
  qc.advance(JB_RQ);
  return d;
}

#ifdef JB_NVSHMEM
// N3 — the paper's own communication layer: after a boundary CTA computed its edge
// tiles, one warp sends them into the neighbour PE's halo with nvshmemx_putmem_nbi_warp, row by
// row, and the last row with nvshmemx_putmem_signal_nbi_warp, which sets this CTA's flag slot on
// the neighbour to t+1 once the data is there (nvshmem_fence orders the earlier rows before it).
// (NO_COMPUTE: the owned edge plane of the current buffer is sent as-is.)
template <int DIM, bool NOCOMP>
__device__ void shm_put_boundary(const JbGeom &g, const JbSlab &SL, int role, int ridx, int rcount,
                                 const double *cur, double *nxt, int64_t tg, bool drop_signal) {
  const Sched sc = make_sched(g, SL, role, ridx, rcount);
  const int pe = role == ROLE_TOP ? SL.shm_pe_top : SL.shm_pe_bot;
  double *dst_plane = role == ROLE_TOP ? SL.peer_top[(tg + 1) & 1] : SL.peer_bot[(tg + 1) & 1];
  uint64_t *sig = reinterpret_cast<uint64_t *>((role == ROLE_TOP ? SL.flag_out_top : SL.flag_out_bot) + ridx);
  const double *src_plane = (NOCOMP ? cur : nxt) + sc.plane * g.plane_elems;
  int rows_left = 0;
  for (int u = sc.ub; u < sc.ue; ++u) {
    const int uy = u / g.units_x;
    const int64_t y0 = 1 + (int64_t)uy * g.ty;
    rows_left += DIM == 3 ? (int)min((int64_t)g.ty, g.ny - 1 - y0) : 1;
  }
  bool signalled = false;
  for (int u = sc.ub; u < sc.ue; ++u) {
    const int ux = u % g.units_x, uy = u / g.units_x;
    const int64_t x0 = 1 + (int64_t)ux * g.tx;
    const int64_t vx = min((int64_t)g.tx, g.nx - 1 - x0);
    const int64_t y0 = DIM == 3 ? 1 + (int64_t)uy * g.ty : 0;
    const int vy = DIM == 3 ? (int)min((int64_t)g.ty, g.ny - 1 - y0) : 1;
    for (int r = 0; r < vy; ++r) {
      const int64_t off = (DIM == 3 ? (y0 + r) * g.pitch : 0) + 3 + x0;
      if (--rows_left > 0 || drop_signal) {
        nvshmemx_putmem_nbi_warp(dst_plane + off, src_plane + off, vx * sizeof(double), pe);
      } else {
        nvshmem_fence();
        nvshmemx_putmem_signal_nbi_warp(dst_plane + off, src_plane + off, vx * sizeof(double), sig,
                                        (uint64_t)(tg + 1), NVSHMEM_SIGNAL_SET, pe);
        signalled = true;
      }
    }
  }
  if (!signalled && !drop_signal && (threadIdx.x & 31) == 0)
    nvshmemx_signal_op(sig, (uint64_t)(tg + 1), NVSHMEM_SIGNAL_SET, pe);
  nvshmem_quiet();  // the source planes may be overwritten two iterations later
}
#endif

// ---------------------------------------------------------------- the kernel
template <int DIM, bool NOCOMP, bool PERSIST, bool NORM>
__global__ void __launch_bounds__(JB_THREADS, 1) jb_sweep(const __grid_constant__ JbParams P) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int s_abort;
  __shared__ double s_red[JB_NCW];  // N4: per-warp partial sums
  const JbGeom &g = P.g;
  Ring R;
  R.S = (uint32_t)g.stages;
  R.stage_doubles = g.stage_doubles;
  R.full = reinterpret_cast<uint64_t *>(smem);
  R.empty = R.full + R.S;
  Queue Q;
  Q.full = R.empty + R.S;
  Q.empty = Q.full + JB_RQ;
  Q.desc = reinterpret_cast<RunDesc *>(Q.empty + JB_RQ);
  const uint32_t hdr = 2 * R.S * 8 + 2 * JB_RQ * 8 + JB_RQ * 32;
  R.stages = reinterpret_cast<double *>(smem + ((hdr + 127) & ~127u));

  int si = 0;
  while (si + 1 < P.nslabs && (int)blockIdx.x >= P.s[si + 1].cta_begin) ++si;
  const JbSlab &SL = P.s[si];
  const int c = (int)blockIdx.x - SL.cta_begin;
  int role, ridx, rcount;
  if (c < SL.n_top) {
    role = ROLE_TOP; ridx = c; rcount = SL.n_top;
  } else if (c < SL.n_top + SL.n_bot) {
    role = ROLE_BOT; ridx = c - SL.n_top; rcount = SL.n_bot;
  } else {
    role = ROLE_INT; ridx = c - SL.n_top - SL.n_bot; rcount = SL.cta_count - SL.n_top - SL.n_bot;
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const bool producer = warp == JB_NCW;
  const int ctid = threadIdx.x;  // consumer thread id (valid when !producer)

  if (threadIdx.x == 0) {
    for (uint32_t i = 0; i < R.S; ++i) {
      mbar_init(&R.full[i], 1);
      mbar_init(&R.empty[i], JB_NC);  // one arrival per consumer thread (Ring::release)
    }
    for (int i = 0; i < JB_RQ; ++i) {
      mbar_init(&Q.full[i], 1);
      mbar_init(&Q.empty[i], JB_NCW);
    }
    fence_mbar_init();
    s_abort = 0;
  }
  __syncthreads();

  const bool dyn = !NOCOMP && SL.dyn_min_blk > 0 && SL.dyn_items > 0 &&
                   (role == ROLE_INT || SL.dyn_help);
  // With the dynamic schedule the interior has no static runs.
  const Sched sched0 = (role == ROLE_INT && SL.dyn_min_blk > 0 && !NOCOMP)
                           ? Sched{0, 0, 0, 0, 0, 0, 0, 0, 0}
                           : make_sched(g, SL, role, ridx, rcount);
  const bool drop_signal = (P.flags & JACOBI_FLAG_DROP_SIGNAL) && SL.slab_id == 0;
  const int64_t lo = (SL.n_top || SL.excl_top) ? 2 : 1;
  RingPos q = {0u, 0u};   // data ring: producer and consumers advance identical copies
  RingPos rq = {0u, 0u};  // run queue

  __shared__ int s_stop, s_abort_pw;
  if (threadIdx.x == 0) s_stop = s_abort_pw = 0;
  int64_t done = P.iters;
  bool prewaited = false;  // producer of a boundary CTA: this iteration's halo flag was acquired during the last barrier
  for (int64_t t = 0; t < P.iters; ++t) {
    const int64_t tg = P.t0 + t;
    const bool pw = prewaited;
    prewaited = false;
    unsigned long long *sig_pending = nullptr;  // thread 0 (NOCOMP): flag to raise at the barrier
    const bool check = NORM && P.norm_every > 0 && (t + 1) % P.norm_every == 0;
    const double *cur = SL.buf[tg & 1];
    double *nxt = SL.buf[(tg + 1) & 1];
    double *remote = nullptr;  // peer stores (UVA / IPC); the NVSHMEM variant puts after the run
    if (role == ROLE_TOP && !SL.use_shm) remote = SL.peer_top[(tg + 1) & 1];
    if (role == ROLE_BOT && !SL.use_shm) remote = SL.peer_bot[(tg + 1) & 1];
    const bool active = !(NOCOMP && role == ROLE_INT);
    // LL halo protocol (§5.11): iterations after the run's first receive LL cells, iterations
    // before its last send them; the first / last halo of a run keep the flag protocol, so flags
    // and halo planes are valid between runs of any kind.
    const unsigned long long *llin = nullptr;
    unsigned long long *llout = nullptr, *rll = nullptr;
    if (PERSIST && !NORM && role != ROLE_INT) {
      if (t > 0) llin = role == ROLE_TOP ? SL.ll_in_top[tg & 1] : SL.ll_in_bot[tg & 1];
      if (t + 1 < P.iters) llout = role == ROLE_TOP ? SL.ll_out_top[(tg + 1) & 1] : SL.ll_out_bot[(tg + 1) & 1];
      if (llout && !drop_signal) {  // (a dropped signal: plain halo stores, no LL cells)
        rll = llout;
        remote = nullptr;
      }
    }
    const uint32_t tag_out = ll_tag(tg + 1);
    if (llin) {
      // receive this iteration's halo: every thread of the boundary CTA unpacks LL cells into the
      // halo plane of cur, then the producer's bulk copies read it (generic -> async proxy fence)
      const bool mark = threadIdx.x == JB_NC && ridx == 0;
      if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 0);
      double *halo = SL.buf[tg & 1] + (role == ROLE_TOP ? 0 : SL.chunk + 1) * g.plane_elems;
      ll_unpack(g, sched0, halo, llin, ll_tag(tg), P);  // (false: abort flag up, the barrier ends the run)
      fence_proxy_async_global();
      __syncthreads();
      if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 1);
    }

    // (no-compute: interior CTAs have no runs — they only join the barrier — and no CTA issues
    //  bulk copies, so the queue hand-off and the generic -> async proxy fences are skipped)
    // No-compute boundary CTA with the flag protocol: the consumer warps copy their runs directly
    // (the schedule is static), without the producer's run queue — three hand-offs fewer on the
    // halo's critical path.  The neighbour's flag was acquired during the last barrier (pre-wait;
    // t = 0: consumer warp 0 waits here first).
    bool nc_direct = false;
#ifdef JB_NVSHMEM
    const bool shm_nc = SL.use_shm;
#else
    const bool shm_nc = false;
#endif
    if (NOCOMP && PERSIST && role != ROLE_INT && !llin && !llout && !shm_nc) nc_direct = true;
    if (NOCOMP && role == ROLE_INT) {
    } else if (nc_direct) {
      if (!producer) {
        if (t == 0) {
          if (warp == 0) {
            const bool mark = lane == 0 && ridx == 0;
            if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 0);
            const bool okw = role == ROLE_TOP ? wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)tg, P, lane)
                                              : wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)tg, P, lane);
            if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 1);
            if (lane == 0 && !okw) s_abort_pw = 1;
          }
          named_bar_consumers();
        }
        if (!s_abort_pw) {
          Sched sched = sched0;
          Run run;
          double acc = 0.0;
          while (sched.next(run))
            consume_run<DIM, NOCOMP, false>(g, R, q, run, cur, nxt, remote, nullptr, tag_out, ctid, lane, acc);
        }
        // (the CTA barrier before the grid barrier orders every consumer's peer stores before
        //  thread 0's release of the flag)
        if (ctid == 0 && !drop_signal) {
          sig_pending = (role == ROLE_TOP ? SL.flag_out_top : SL.flag_out_bot) + ridx;
          if (ridx == 0) halo_mark(SL, P, role == ROLE_BOT, t, 2);
        }
      }
    } else if (producer) {
      // Every lane that issues bulk copies orders them after the grid barrier's acquire (and the
      // generic-proxy stores it covers) with its own proxy fence.
      if (!NOCOMP) fence_proxy_async_global();
      // The claim counter of the next iteration is idle now (last used in iteration t-1).
      if (!NOCOMP && lane == 0 && c == 0 && SL.work_ctr) SL.work_ctr[(tg + 1) & 1] = 0u;
      // boundary blocks wait until the neighbour committed the halo of the previous time
      // step.  With compute, the two owned planes of the first boundary tile are already in
      // flight while we wait; only the halo plane's load waits for the flag.
      bool waited = !(PERSIST && role != ROLE_INT) || llin != nullptr || pw;
      auto wait_flag = [&]() {
        if (!waited) {
          const bool mark = PERSIST && lane == 0 && ridx == 0;
          if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 0);
          if (role == ROLE_TOP) wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)tg, P, lane);
          else wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)tg, P, lane);
          if (mark) halo_mark(SL, P, role == ROLE_BOT, t, 1);
          __syncwarp();
          if (!NOCOMP) fence_proxy_async_global();  // every copying lane: halo rows written by the neighbour
          waited = true;
        }
      };
      Sched sched = sched0;
      Run run;
      if (active) {
        while (sched.next(run)) {
          if (NOCOMP) {
            wait_flag();  // remote stores of this run must follow the neighbour's signal
            publish(Q, rq, RUN_WORK, run, lane);  // (the consumers copy from L2: no stages)
          } else if (role != ROLE_INT) {
            // boundary tile (one plane): halo is p-1 (top) or p+1 (bottom)
            publish(Q, rq, RUN_WORK, run, lane,
                    (int)(SL.dyn_items + (role == ROLE_TOP ? 0 : g.units) + run.unit));
            const TileSrc T(g, cur, run.unit, lane);
            RingPos q1 = q, q2 = q;
            q1.advance(R.S);
            q2 = q1;
            q2.advance(R.S);
            const int64_t p = run.p0;
            if (role == ROLE_TOP) {
              produce_stage(g, T, p, q1, R, lane);
              produce_stage(g, T, p + 1, q2, R, lane);
              wait_flag();
              produce_stage(g, T, p - 1, q, R, lane);
            } else {
              produce_stage(g, T, p - 1, q, R, lane);
              produce_stage(g, T, p, q1, R, lane);
              wait_flag();
              produce_stage(g, T, p + 1, q2, R, lane);
            }
            q = q2;
            q.advance(R.S);
          } else {
            publish(Q, rq, RUN_WORK, run, lane);
            produce_planes(g, cur, run.unit, run.p0 - 1, run.p1 + 1, q, R, lane);
          }
        }
      }
      wait_flag();  // (boundary CTA without units this iteration still keeps the protocol)
      // Boundary runs done: signal (CPU-Free) and, in every mode, stop peer stores.
      if (role != ROLE_INT) publish(Q, rq, RUN_SIGNAL, run, lane);
      if (dyn) {
        // Guided self-scheduling (block-major items, host-built block table).  Interior CTA
        // i's first item is item i; every further item is claimed with one atomicAdd, issued
        // before the previous item's loads so its latency overlaps them.
        unsigned int *ctr = SL.work_ctr + (tg & 1);
        int64_t item = (role == ROLE_INT && ridx < SL.dyn_first) ? ridx : -1;
        unsigned int claim = 0;
        if (item < 0) {
          if (lane == 0) claim = atomicAdd(ctr, 1u);
          item = SL.dyn_first + (int64_t)__shfl_sync(0xffffffffu, claim, 0);
        }
        while (item < SL.dyn_items) {
          const int64_t b = item / g.units;
          run.unit = (int32_t)(item - b * g.units);
          run.p0 = lo + SL.dyn_table[b];
          run.p1 = lo + SL.dyn_table[b + 1] - 1;
          // Claim the next item now if this one fits in the ring (its loads are issued at once,
          // so the atomic's latency hides behind them); for a long item claim only after its
          // loads are issued, or the claim would reserve work long before it is needed.
          const bool early = run.p1 - run.p0 + 3 <= (int64_t)R.S;
          if (early && lane == 0) claim = atomicAdd(ctr, 1u);
          publish(Q, rq, RUN_WORK, run, lane, (int)item);
          produce_planes(g, cur, run.unit, run.p0 - 1, run.p1 + 1, q, R, lane);
          if (!early && lane == 0) claim = atomicAdd(ctr, 1u);
          item = SL.dyn_first + (int64_t)__shfl_sync(0xffffffffu, claim, 0);
        }
      }
      publish(Q, rq, RUN_END, run, lane);
    } else {
      while (true) {
        const RunDesc d = fetch(Q, rq, lane);
        if (d.kind == RUN_END) break;
        if (d.kind == RUN_SIGNAL) {
          // P:364-365 / P:394: signal the neighbour that the halo of iteration tg+1 is in place.
          if (PERSIST || SL.use_shm) named_bar_consumers();
          // bar.sync makes every consumer thread's peer stores precede thread 0 (CTA scope);
          // its sys-scope release store into this CTA's slot publishes them to the neighbour.
#ifdef JB_NVSHMEM
          if (SL.use_shm) {  // CPU-Free (persistent) and the "Baseline NVSHMEM" discrete kernel
            if (warp == 0) shm_put_boundary<DIM, NOCOMP>(g, SL, role, ridx, rcount, cur, nxt, tg, drop_signal);
            remote = nullptr;
            continue;
          }
#endif
          if (PERSIST && ctid == 0 && !drop_signal) {
            if (!llout) {
              unsigned long long *fo = role == ROLE_TOP ? SL.flag_out_top : SL.flag_out_bot;
              // no-compute: the CTA's next action is the grid barrier, so the signal shares the
              // arrival's release fence (slab_barrier): one fence instead of two serialised ones
              if (NOCOMP) sig_pending = fo + ridx;
              else st_release_flag(P, fo + ridx, (unsigned long long)(tg + 1));
            }  // (LL: the cells carry their iteration, nothing to signal)
            if (ridx == 0) halo_mark(SL, P, role == ROLE_BOT, t, 2);
          }
          remote = nullptr;  // later (interior) runs stay local
          rll = nullptr;
          continue;
        }
        Run run;
        run.unit = d.unit;
        run.p0 = d.p0;
        run.p1 = d.p1;
        double acc = 0.0;
        if (NORM && check) {
          consume_run<DIM, NOCOMP, NORM>(g, R, q, run, cur, nxt, remote, rll, tag_out, ctid, lane, acc);
          // deterministic per-run sum: xor tree in each warp, then warps in order
          for (int o = 16; o > 0; o >>= 1) acc = acc + __shfl_xor_sync(0xffffffffu, acc, o);
          if (lane == 0) s_red[warp] = acc;
          named_bar_consumers();
          if (ctid == 0) {
            double v = s_red[0];
            for (int w = 1; w < JB_NCW; ++w) v = v + s_red[w];
            __stcg(SL.partials + d.item, v);
          }
          named_bar_consumers();
        } else {
          consume_run<DIM, NOCOMP, false>(g, R, q, run, cur, nxt, remote, rll, tag_out, ctid, lane, acc);
        }
      }
      // Our generic-proxy stores must be ordered before later bulk (async-proxy) reads.
      if (!NOCOMP) fence_proxy_async_global();
    }
    if (!PERSIST) break;
    if (P.trace && t < 8 && threadIdx.x == 0) P.trace[t * gridDim.x + blockIdx.x] = globaltimer();

    // Device-side grid barrier of this slab's CTAs (P:372 grid.sync()).
    __syncthreads();
    if (warp == 0) {
      const bool ok = slab_barrier(SL, P, c, (unsigned long long)(t + 1), (unsigned long long)(tg + 1), lane,
                                   sig_pending, (unsigned long long)(tg + 1));
      if (lane == 0) s_abort = ok ? 0 : 1;  // (slab_barrier also reports an abort flag)
    } else if (PERSIST && producer && role != ROLE_INT && t + 1 < P.iters &&
               (NORM || (role == ROLE_TOP ? SL.ll_in_top[(tg + 1) & 1] : SL.ll_in_bot[(tg + 1) & 1]) == nullptr)) {
      // Pre-wait (P:394's wait, moved off the critical path): the neighbour's flag for the next
      // iteration does not depend on this slab's barrier (the neighbour raises it in its own
      // iteration t), so the boundary CTA's producer polls it while warp 0 spins on the barrier,
      // instead of paying another L2 round trip after it.
      const bool mark = lane == 0 && ridx == 0;
      if (mark) halo_mark(SL, P, role == ROLE_BOT, t + 1, 0);
      const bool ok = role == ROLE_TOP ? wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(tg + 1), P, lane)
                                       : wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(tg + 1), P, lane);
      if (mark) halo_mark(SL, P, role == ROLE_BOT, t + 1, 1);
      __syncwarp();
      if (!NOCOMP) fence_proxy_async_global();  // every copying lane: halo rows written by the neighbour
      prewaited = ok;
      if (!ok && lane == 0) s_abort_pw = 1;
    }
    __syncthreads();
    if (s_abort || s_abort_pw) return;
    if (NORM && check) {
      // N4: all-reduce of the update norm over every slab (device-side, through the JbCtrl
      // norm slots of each slab), identical on every CTA of every GPU, then the stop decision.
      const int64_t k = P.k0 + (t + 1) / P.norm_every - 1;  // global check index
      JbCtrl *mine = SL.norm_peers[SL.slab_id];
      if (warp == 0) {
        if (c == 0) {
          double v = 0.0;
          for (int i = lane; i < SL.n_partials; i += 32) v = v + __ldcg(SL.partials + i);
          for (int o = 16; o > 0; o >>= 1) v = v + __shfl_xor_sync(0xffffffffu, v, o);
          if (lane < SL.norm_slabs) {  // lane g delivers this slab's sum to slab g
            JbCtrl *dst = SL.norm_peers[lane];
            dst->norm_val[k & 1][SL.slab_id] = v;
            st_release_flag(P, &dst->norm_flag[SL.slab_id], (unsigned long long)(k + 1));
          }
        }
        const bool ok = wait_slots(mine->norm_flag, SL.norm_slabs, (unsigned long long)(k + 1), P, lane);
        if (lane == 0) {
          double tot = 0.0;
          for (int g2 = 0; g2 < SL.norm_slabs; ++g2) tot = tot + __ldcv(&mine->norm_val[k & 1][g2]);
          const double r = sqrt(tot);
          if (c == 0) mine->norm_out = r;
          s_stop = (!ok) ? 2 : (r <= P.tol ? 1 : 0);
        }
      }
      __syncthreads();
      if (s_stop == 2) return;
      if (s_stop) {
        done = t + 1;
        break;
      }
    }
  }
  if (NORM && c == 0 && threadIdx.x == 0) SL.norm_peers[SL.slab_id]->done_iters = done;

  // End of run: wait for the neighbour's last halo so no remote store is still in flight into
  // this GPU's buffers when the kernel (and the host's view of the run) completes.
  if (PERSIST && producer && role != ROLE_INT && done > 0) {
    if (role == ROLE_TOP) wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(P.t0 + done), P, lane);
    else wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(P.t0 + done), P, lane);
  }
}

// "Baseline NVSHMEM": the dedicated kernel, launched by the host every iteration after
// the compute kernel, that waits until both neighbours delivered this iteration's halos.
__global__ void jb_neighbour_wait(const __grid_constant__ JbParams P, unsigned long long target) {
  const JbSlab &S = P.s[0];
  const int lane = threadIdx.x & 31;
  if (S.k_in_top > 0) wait_slots(S.flag_in_top, S.k_in_top, target, P, lane);
  if (S.k_in_bot > 0) wait_slots(S.flag_in_bot, S.k_in_bot, target, P, lane);
}

template <int DIM, bool NOCOMP, bool PERSIST>
const void *kfn() {
  return reinterpret_cast<const void *>(&jb_sweep<DIM, NOCOMP, PERSIST, false>);
}

const void *sweep_fn(int dim, bool nocomp, bool persist, bool norm = false) {
  if (norm) {  // residual-norm variant: CPU-Free persistent with compute only
    return dim == 2 ? reinterpret_cast<const void *>(&jb_sweep<2, false, true, true>)
                    : reinterpret_cast<const void *>(&jb_sweep<3, false, true, true>);
  }
  if (dim == 2) {
    if (persist) return nocomp ? kfn<2, true, true>() : kfn<2, false, true>();
    return nocomp ? kfn<2, true, false>() : kfn<2, false, false>();
  }
  if (persist) return nocomp ? kfn<3, true, true>() : kfn<3, false, true>();
  return nocomp ? kfn<3, true, false>() : kfn<3, false, false>();
}

}  // namespace

// ---------------------------------------------------------------- host-side launchers
namespace jbk {

cudaError_t prepare(int dim, bool nocomp, bool persist, size_t smem) {
  cudaError_t e = cudaFuncSetAttribute(sweep_fn(dim, nocomp, persist), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)smem);
  if (e != cudaSuccess || nocomp || !persist) return e;
  return cudaFuncSetAttribute(sweep_fn(dim, false, true, true), cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)smem);
}

cudaError_t occupancy(int dim, bool nocomp, bool persist, size_t smem, int *blocks_per_sm) {
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, sweep_fn(dim, nocomp, persist),
                                                       JB_THREADS, smem);
}

cudaError_t launch_sweep(const JbParams &p, bool nocomp, bool persist, int grid, size_t smem,
                         cudaStream_t st) {
  void *args[] = {const_cast<JbParams *>(&p)};
  const void *fn = sweep_fn(p.g.dim, nocomp, persist, persist && !nocomp && p.norm_every > 0);
  if (persist) return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(JB_THREADS), args, smem, st);
  return cudaLaunchKernel(fn, dim3(grid), dim3(JB_THREADS), args, smem, st);
}

cudaError_t launch_neighbour_wait(const JbParams &p, unsigned long long target, cudaStream_t st) {
  jb_neighbour_wait<<<1, 32, 0, st>>>(p, target);
  return cudaGetLastError();
}

}  // namespace jbk
