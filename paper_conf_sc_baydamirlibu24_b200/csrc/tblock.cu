// tblock.cu — temporally blocked CPU-Free sweep: K Jacobi iterations per
// pass over HBM — 2D: K = 2 (extra-cell scheme, §5.7), K = 3 / 5 (overlapped warp segments,
// §5.8; default K = 5); 3D: K = 2 (§5.7), K = 3 (x/y-overlapped tiles with a shared-memory row
// exchange and TMA box loads, §5.9; the default for slabs without neighbours).
//
// The method is unchanged — every cell is updated every iteration with the oracle's fp64 order
// (-fmad=false), each iteration reads only the previous time step, Dirichlet cells are
// never written — only the schedule of the updates differs: a work item (plane block
// [a, b] x strip / tile) streams the time-t planes a-K .. b+K of its strip from HBM through the
// same TMA ring as jb_sweep, computes the intermediate levels t+1 .. t+K-1 in registers (x
// neighbours by warp shuffles) and level t+K for planes a .. b, which it stores into the other
// buffer.  The intermediate levels never touch HBM, so the algorithmic traffic per cell-update
// is 16 B / K instead of 16 B (overlapped tiling: the values near a strip's / tile's edges are
// recomputed by its neighbours).  Slabs with neighbours keep the paper's per-iteration halo
// exchange through edge zones (K phases per time block, tb_edge).  The persistent structure of
// the paper is kept: one cooperative launch for the whole run, a device-side grid barrier
// between time blocks, no host involvement.
//
// Buffers: time block j of a launch reads buf[(t0 + j) & 1] and writes buf[(t0 + j + 1) & 1]
// (out of place — neighbouring strips still read the time-t columns of this strip); for K = 2
// the host runs an even number of blocks, for odd K any number, so the result lands in
// buf[(t0 + K nb) & 1] as in every other path (R10).
#include <type_traits>

#include "device_common.cuh"

namespace {

enum { TB_WORK = 0, TB_END = 1 };
struct TbDesc {
  int32_t kind;
  int32_t unit;
  int64_t a, b;  // output planes a..b of this item (time t+2)
  int64_t pad;
};

// TMA box copy (tensor map in global memory) of one plane window into shared memory.
__device__ __forceinline__ void tma_box3(void *dst, const void *tmap, int c0, int c1, int c2, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
      "[%5];" ::"r"(sptr(dst)),
      "l"(tmap), "r"(c0), "r"(c1), "r"(c2), "r"(sptr(bar))
      : "memory");
}

// The odd-K marches run towards row / plane 0 (shorter fp64 dependency chain, see tbk_march).
constexpr bool TB_REV = true;
#ifndef TB2_HOIST
#define TB2_HOIST 1  // 2D odd-K march: shuffle every level's centre-row x neighbours at the step start
#endif
#ifndef TB3_PF
#define TB3_PF 1  // 3D odd-K march: level-0 planes of the steady state kept in registers (tb3k_march)
#endif

// Position `off` stages after p in the ring.
__device__ __forceinline__ RingPos ring_add(RingPos p, uint32_t off, uint32_t S) {
  const uint32_t s = p.slot + off;
  const uint32_t wraps = s / S;
  return RingPos{s - wraps * S, p.phase ^ (wraps & 1u)};
}

// Per-warp geometry of one item.
struct TbSeg {
  int j0;                // stage index of pair i = 0 (stage s <-> column x0 - 2 + s)
  unsigned in_tile, ok, full, first, last;
  int sx;                // stage index of this lane's extra level-1 cell (segment ends)
  bool ex_in;            // that extra cell is an interior column
  bool fast;             // every pair of the segment is interior: no per-pair masks
};

// Level 1 (t+1) of this lane's pairs and extra cell on the row whose level-0 stages are
// sm (row-1), sc (row), sn (row+1); rows outside 1..C keep level 0 (rowin = false).
template <int PPT, bool FAST, bool ROWIN>
__device__ __forceinline__ void tb_level1(const TbSeg &L, const double *sm, const double *sc, const double *sn,
                                          bool rowin_rt, double2 *V, double &ex) {
  const bool rowin = ROWIN || rowin_rt;
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const int j = L.j0 + 64 * i;
    if (FAST || (L.in_tile >> i & 1u)) {
      const double2 S0 = lds2(sm + j), C0 = lds2(sc + j), N0 = lds2(sn + j);
      const double W = sc[j - 1], E = sc[j + 2];
      // oracle order: ((x+1) + (x-1)) + (y+1) + (y-1), then * 0.25
      const double l0 = 0.25 * (((C0.y + W) + N0.x) + S0.x);
      const double l1 = 0.25 * (((E + C0.x) + N0.y) + S0.y);
      V[i].x = (rowin && (FAST || (L.ok >> i & 1u))) ? l0 : C0.x;  // Dirichlet cells keep level 0
      V[i].y = (rowin && (FAST || (L.full >> i & 1u))) ? l1 : C0.y;
    }
  }
  const int x = L.sx;
  const double e = 0.25 * (((sc[x + 1] + sc[x - 1]) + sn[x]) + sm[x]);
  ex = (rowin && L.ex_in) ? e : sc[x];
}

// Level 2 (t+2) of the middle level-1 row C1 (rows S1, C1, N1), stored at o.  x neighbours by
// rotations: lane l gets lane l-1's .y (W) and lane l+1's .x (E); lane 0 / lane 31 take the
// wrapped value of the previous / next pair, the segment's end pairs the extra cells.
template <int PPT, bool FAST>
__device__ __forceinline__ void tb_level2(const TbSeg &L, const double2 *S1, const double2 *C1, const double2 *N1,
                                          double exl, double exr, int lane, double *o) {
  double rw_prev = 0.0;
  double re_next = __shfl_sync(0xffffffffu, C1[0].x, (lane + 1) & 31);
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const double rw = __shfl_sync(0xffffffffu, C1[i].y, (lane + 31) & 31);
    const double re = re_next;
    if (i + 1 < PPT) re_next = __shfl_sync(0xffffffffu, C1[i + 1].x, (lane + 1) & 31);
    const double W = (L.first >> i & 1u) ? exl : (lane == 0 ? rw_prev : rw);
    const double E = (L.last >> i & 1u) ? exr : (lane == 31 ? re_next : re);
    const double o0 = 0.25 * (((C1[i].y + W) + N1[i].x) + S1[i].x);
    const double o1 = 0.25 * (((E + C1[i].x) + N1[i].y) + S1[i].y);
    if (FAST) *reinterpret_cast<double2 *>(o + 64 * i) = make_double2(o0, o1);
    else if (L.ok >> i & 1u) store_pair(o + 64 * i, o0, o1, L.full >> i & 1u);
    rw_prev = rw;
  }
}

// One item: level-0 rows r0..r1 of strip `unit` sit in consecutive ring stages from q.
//   level 1 (t+1): rows q1 = a-1 .. b+1 (Dirichlet rows / columns keep level 0)
//   level 2 (t+2): rows a .. b, columns x0 .. x0+tx-1  -> out
// Warp w owns the contiguous cell pairs kk = w*32*PPT + i*32 + lane (i < PPT): conflict-free
// 16-byte stage loads, coalesced 16-byte stores.  Level-1 x neighbours inside the segment come
// from neighbouring lanes by shuffles; at the segment's ends the warp computes one extra
// level-1 cell from the level-0 stage (overlapped by one cell per side), so warps never wait
// for each other: no CTA barrier, each warp marches at its own pace.
template <int PPT, bool FAST>
__device__ __forceinline__ void tb2_march(const TbSeg &L, const Ring &R, RingPos q, int64_t a, int64_t b,
                                          int64_t C, int64_t r0, int64_t r1, double *dst, int64_t pe, int lane) {
  // Level-1 rows live in three register sets X0, X1, X2 whose roles (y-1, y, y+1) rotate with
  // the march; the loop is unrolled by three so the rotation is static (no register moves).
  // Extras: lane 0 holds the left one, lane 1 the right one, one slot per set.
  double2 X0[PPT], X1[PPT], X2[PPT];
  double e0, e1, e2;
  // Level-1 row q1 reads level-0 rows max(q1-1, r0), q1, min(q1+1, r1): ring positions pm, pc,
  // pn, advanced by one stage per row (row a-2 exists iff r0 = a-2).
  RingPos pc = ring_add(q, (uint32_t)(a - 1 - r0), R.S);
  RingPos pm = a - 2 >= r0 ? q : pc;
  R.wait_full(pm);
  R.wait_full(pc);
  // rows 1..C are interior (compile-time in the steady state); 0 and C+1 keep level 0
  auto row = [&](auto rowin_ct, int64_t q1, double2 *out, double &e) {
    RingPos pn = pc;
    if (q1 + 1 <= r1) pn.advance(R.S);
    R.wait_full(pn);
    double ex;
    tb_level1<PPT, FAST, decltype(rowin_ct)::value>(L, R.stage(pm), R.stage(pc), R.stage(pn),
                                                    q1 >= 1 && q1 <= C, out, ex);
    e = ex;
    if (q1 - 1 >= r0) R.release(pm, lane);  // row q1-1 is no longer needed
    pm = pc;
    pc = pn;
  };
  using RT = std::integral_constant<bool, true>;
  using RF = std::integral_constant<bool, false>;
  double *o = dst + a * pe;
  // level 2 of the middle row from (S, C, N); extras of the middle row: shuffles from lanes 0/1
  auto lvl2 = [&](const double2 *S, const double2 *Cm, const double2 *N, double em) {
    const double exl = __shfl_sync(0xffffffffu, em, 0), exr = __shfl_sync(0xffffffffu, em, 1);
    tb_level2<PPT, FAST>(L, S, Cm, N, exl, exr, lane, o);
    o += pe;
  };
  row(RF{}, a - 1, X0, e0);  // may be the Dirichlet row 0
  row(RT{}, a, X1, e1);      // a >= 1
  const int64_t qe = min(b + 1, C);  // last interior level-1 row of the march
  int64_t q1 = a + 1;
  for (; q1 + 2 <= qe; q1 += 3) {
    row(RT{}, q1, X2, e2);
    lvl2(X0, X1, X2, e1);
    row(RT{}, q1 + 1, X0, e0);
    lvl2(X1, X2, X0, e2);
    row(RT{}, q1 + 2, X1, e1);
    lvl2(X2, X0, X1, e0);
  }
  // 0-2 interior rows left, then (b == C) the Dirichlet row C+1; the set roles continue the cycle
  // (left <= 3)
  const int64_t left = qe - q1 + 1 + (b + 1 > C ? 1 : 0);
  if (left >= 1) {
    if (q1 <= C) row(RT{}, q1, X2, e2); else row(RF{}, q1, X2, e2);
    lvl2(X0, X1, X2, e1);
  }
  if (left >= 2) {
    if (q1 + 1 <= C) row(RT{}, q1 + 1, X0, e0); else row(RF{}, q1 + 1, X0, e0);
    lvl2(X1, X2, X0, e2);
  }
  if (left >= 3) {  // two interior rows + the Dirichlet row C+1
    row(RF{}, q1 + 2, X1, e1);
    lvl2(X2, X0, X1, e0);
  }
  // rows b+1 .. r1 were not released by the march
  RingPos pr = ring_add(q, (uint32_t)(b + 1 - r0), R.S);
  for (int64_t p = b + 1; p <= r1; ++p) {
    R.release(pr, lane);
    pr.advance(R.S);
  }
}

template <int PPT>
__device__ __forceinline__ void tb2_item(const JbGeom &g, const Ring &R, RingPos &q, int unit, int64_t a,
                                         int64_t b, int64_t C, double *out, int warp, int lane) {
  const int64_t x0 = 1 + (int64_t)unit * g.tx;
  const int vx = (int)min((int64_t)g.tx, g.nx - 1 - x0);  // interior columns of this strip
  const int txp = g.tx >> 1;
  const int seg_b = warp * 32 * PPT;             // first pair of this warp's segment
  const int seg_e = min(seg_b + 32 * PPT, txp);  // one past its last pair
  const int64_t r0 = max(a - 2, (int64_t)0), r1 = min(b + 2, C + 1);
  const RingPos q0 = q;
  q = ring_add(q, (uint32_t)(r1 - r0 + 1), R.S);
  if (seg_b >= seg_e) {  // no pairs in this strip for this warp: only return the stages
    for (int64_t p = r0; p <= r1; ++p) {
      const RingPos pp = ring_add(q0, (uint32_t)(p - r0), R.S);
      R.wait_full(pp);
      R.release(pp, lane);
    }
    return;
  }
  TbSeg L;
  L.j0 = 2 + 2 * (seg_b + lane);
  L.in_tile = L.ok = L.full = L.first = L.last = 0;
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const int kk = seg_b + i * 32 + lane;
    L.in_tile |= (kk < seg_e ? 1u : 0u) << i;
    L.ok |= (kk < seg_e && 2 * kk < vx ? 1u : 0u) << i;
    L.full |= (kk < seg_e && 2 * kk + 1 < vx ? 1u : 0u) << i;
    L.first |= (kk == seg_b ? 1u : 0u) << i;
    L.last |= (kk == seg_e - 1 ? 1u : 0u) << i;
  }
  // extra level-1 cells: lane 1 computes the right one (column x0 + 2 seg_e), every other lane
  // the left one (x0 + 2 seg_b - 1); level 2 takes them from lanes 0 and 1.
  L.sx = lane == 1 ? 2 * seg_e + 2 : 2 * seg_b + 1;
  const int64_t cx = x0 - 2 + L.sx;
  L.ex_in = cx >= 1 && cx <= g.nx - 2;
  const bool fast = seg_e - seg_b == 32 * PPT && 2 * seg_e <= vx;
  double *dst = out + 3 + x0 + 2 * (seg_b + lane);
  if (fast) tb2_march<PPT, true>(L, R, q0, a, b, C, r0, r1, dst, g.plane_elems, lane);
  else tb2_march<PPT, false>(L, R, q0, a, b, C, r0, r1, dst, g.plane_elems, lane);
}

// ---------------------------------------------------------------- 2D, deeper time blocks (K odd)
// K = 3, 5: levels 1 .. K of one item, no extra cells.  Warp w computes every level over the same
// 64 PPT columns s_w .. s_w + 64 PPT - 1 (s_w = x0 + w WO - (K-1), WO = 64 PPT - 2 (K-1)); lane l
// owns the PPT contiguous cell pairs kk = l PPT + i.  Level 1 comes from the level-0 stage,
// level k >= 2 from level k-1 in registers: x neighbours inside a lane are its own registers,
// across lanes one shuffle per side and level.  At the two ends of the segment a level loses one
// valid column per side (the shuffle wraps around), so level K is valid on the middle WO columns,
// which are this warp's outputs; neighbouring warps overlap by 2(K-1) columns and never
// communicate.  With K odd both the level-1 loads (stage index 2 + 2 kk) and the level-K
// stores (column s_w + K-1, odd x) stay 16-byte aligned.  Rows: the march takes one level-0 row
// per step and advances every level by one row (a wavefront, see tbk_march).
// Cells outside the interior (Dirichlet rows / columns, the garbage columns past the grid)
// keep their previous level — the definition's untouched boundary — and never reach an
// interior output.
struct TbkLane {
  int j0;                  // stage index of pair 0 of this lane
  unsigned ok, full, st;   // per pair: cell x / x+1 interior; pair stored at level K
};

template <int PPT, bool FAST, bool STEADY>
__device__ __forceinline__ void tbk_level1(const TbkLane &L, const double *sm, const double *sc, const double *sn,
                                           bool rowin, double2 *V) {
  double2 S0[PPT], C0[PPT], N0[PPT];
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    S0[i] = lds2(sm + L.j0 + 2 * i);
    C0[i] = lds2(sc + L.j0 + 2 * i);
    N0[i] = lds2(sn + L.j0 + 2 * i);
  }
  const double Wl = sc[L.j0 - 1], Er = sc[L.j0 + 2 * PPT];
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const double W = i == 0 ? Wl : C0[i - 1].y;
    const double E = i == PPT - 1 ? Er : C0[i + 1].x;
    // oracle order: ((x+1) + (x-1)) + (y+1) + (y-1), then * 0.25
    const double l0 = 0.25 * (((C0[i].y + W) + N0[i].x) + S0[i].x);
    const double l1 = 0.25 * (((E + C0[i].x) + N0[i].y) + S0[i].y);
    if (FAST && STEADY) {
      V[i] = make_double2(l0, l1);
    } else {
      const bool r = STEADY || rowin;
      V[i].x = (r && (FAST || (L.ok >> i & 1u))) ? l0 : C0[i].x;
      V[i].y = (r && (FAST || (L.full >> i & 1u))) ? l1 : C0[i].y;
    }
  }
}

// Level 1 from level-0 pairs already in registers (S, Cm, N rows; W / E: the centre row's cells
// left of pair 0 and right of the last pair) — the software-pipelined steady state of tbk_march.
template <int PPT, bool FAST>
__device__ __forceinline__ void tbk_level1_regs(const TbkLane &L, const double2 *S0, const double2 *C0,
                                                const double2 *N0, double Wl, double Er, double2 *V) {
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const double W = i == 0 ? Wl : C0[i - 1].y;
    const double E = i == PPT - 1 ? Er : C0[i + 1].x;
    // oracle order: ((x+1) + (x-1)) + (y+1) + (y-1), then * 0.25
    const double l0 = 0.25 * (((C0[i].y + W) + N0[i].x) + S0[i].x);
    const double l1 = 0.25 * (((E + C0[i].x) + N0[i].y) + S0[i].y);
    if (FAST) {
      V[i] = make_double2(l0, l1);
    } else {
      V[i].x = (L.ok >> i & 1u) ? l0 : C0[i].x;  // (steady rows are interior; columns may not be)
      V[i].y = (L.full >> i & 1u) ? l1 : C0[i].y;
    }
  }
}

// A double from lane src (two 32-bit shuffles, halves kept in place).
// A double from lane l-1 (up) / l+1 (down): constant deltas, no lane index (whose S2R read the
// compiler re-issues inside the 2D march and whose latency the shuffles then wait for: C2 +3-4 %;
// the 3D march keeps the indexed form, measured equal-or-better there).  Lane 0 / 31
// keep their own value — like the wrapped value before, it only reaches cells outside the valid
// span (each level loses one column per segment end).
__device__ __forceinline__ double shfl_up_d(double v) {
  double r;
  asm("{\n .reg .b32 lo, hi;\n mov.b64 {lo, hi}, %1;\n shfl.sync.up.b32 lo, lo, 1, 0x0, -1;\n"
      " shfl.sync.up.b32 hi, hi, 1, 0x0, -1;\n mov.b64 %0, {lo, hi};\n}"
      : "=d"(r)
      : "d"(v));
  return r;
}
__device__ __forceinline__ double shfl_down_d(double v) {
  double r;
  asm("{\n .reg .b32 lo, hi;\n mov.b64 {lo, hi}, %1;\n shfl.sync.down.b32 lo, lo, 1, 0x1f, -1;\n"
      " shfl.sync.down.b32 hi, hi, 1, 0x1f, -1;\n mov.b64 %0, {lo, hi};\n}"
      : "=d"(r)
      : "d"(v));
  return r;
}
__device__ __forceinline__ double shfl_d(double v, int src) {
  double r;
  asm("{\n .reg .b32 lo, hi;\n mov.b64 {lo, hi}, %1;\n shfl.sync.idx.b32 lo, lo, %2, 0x1f, -1;\n"
      " shfl.sync.idx.b32 hi, hi, %2, 0x1f, -1;\n mov.b64 %0, {lo, hi};\n}"
      : "=d"(r)
      : "d"(v), "r"(src));
  return r;
}

// Level k >= 2 of the middle row of (S, Cm, N) (level k-1): W of pair 0 from lane l-1's last
// pair, E of the last pair from lane l+1's first (lane 0 / 31: wrapped, outside the valid span).
// STORE: level K, written to o (this lane's pair 0 in the output row) instead of V.
template <int PPT, bool FAST, bool STEADY, bool STORE>
__device__ __forceinline__ void tbk_levelk(const TbkLane &L, const double2 *S, const double2 *Cm, const double2 *N,
                                           bool rowin, int lane, double2 *V, double *o, const double *WE = nullptr) {
  // WE: this level's x neighbours of the centre row, already shuffled (TB2_HOIST)
  const double Wl = WE ? WE[0] : shfl_up_d(Cm[PPT - 1].y);
  const double Er = WE ? WE[1] : shfl_down_d(Cm[0].x);
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const double W = i == 0 ? Wl : Cm[i - 1].y;
    const double E = i == PPT - 1 ? Er : Cm[i + 1].x;
    const double o0 = 0.25 * (((Cm[i].y + W) + N[i].x) + S[i].x);
    const double o1 = 0.25 * (((E + Cm[i].x) + N[i].y) + S[i].y);
    if (STORE) {
      if (L.st >> i & 1u) {
        if (FAST) *reinterpret_cast<double2 *>(o + 2 * i) = make_double2(o0, o1);
        else store_pair(o + 2 * i, o0, o1, L.full >> i & 1u);
      }
    } else if (FAST && STEADY) {
      V[i] = make_double2(o0, o1);
    } else {
      const bool r = STEADY || rowin;
      V[i].x = (r && (FAST || (L.ok >> i & 1u))) ? o0 : Cm[i].x;
      V[i].y = (r && (FAST || (L.full >> i & 1u))) ? o1 : Cm[i].y;
    }
  }
}

// The wavefront: at step R (level-0 row R enters) level k computes row R - 1 - LAG (k-1), which
// needs level k-1 rows up to R - LAG (k-1): computed LAG-1 steps earlier.  LAG = 1: the levels of
// a step form one dependency chain, three rows per level in registers; LAG = 2: the K levels of a
// step are independent (more instruction-level parallelism, four rows per level).  Set m % NS
// of a level holds its row computed at step m (static rotation, the loop unrolled by NS).
// REV: the march runs towards row 0 (the producer streams the rows in decreasing order; a, b,
// r0, r1 are then mirrored row indices r' = C+1-r).  In the oracle order ((x+1 + x-1) + y+1) +
// y-1, the row a level just computed is the NEWEST row of the march: marching up it is y+1
// (three dependent fp64 operations after it: + y+1, + y-1, * 1/4), marching down it is y-1
// (two: + y-1, * 1/4), so the dependency chain through the K levels of a step is ~25 % shorter
// — same operations, same order, bit-identical results.
// SD: the stage stride in doubles when it is a compile-time constant of the kernel variant (0:
// runtime R.stage_doubles) — the steady-state preloads then address shared memory with one 32-bit
// register and a constant stride.
template <int K, int PPT, int LAG, bool FAST, bool REV, int SD = 0>
__device__ __forceinline__ void tbk_march(const TbkLane &L, const Ring &R, RingPos q, int a, int b, int C, int r0,
                                          int r1, double *dst, int64_t pe, int lane) {
  constexpr int NS = LAG + 2;
  double2 X[K - 1][NS][PPT];  // X[k-1][m % NS]: level k of the row computed at step m
  const int Rs = a - K >= 0 ? r0 + 2 : r0 + 1;  // first step (r0 = 0 when a - K < 0)
  const int Re = b + 1 + LAG * (K - 1);         // last step: level K of row b
  // steady window: every level's row is needed and interior, level K is stored
  const int Ws = a + 1 + LAG * (K - 1), We = min(b + K, C + 1);
  // output row of step Rs (advanced per step; REV: actual row C+1-r', moving down)
  const int ro0 = Rs - 1 - LAG * (K - 1);
  double *o = dst + (int64_t)(REV ? C + 1 - ro0 : ro0) * pe;
  const int64_t ostep = REV ? -pe : pe;
  // stage positions of level-0 rows R-2, R-1, R, clamped to r0 .. r1
  RingPos pm = q, pc = Rs == r0 + 2 ? ring_add(q, 1u, R.S) : q, pn = pc;
  if (Rs <= r1) pn = ring_add(q, (uint32_t)(Rs - r0), R.S);
  R.wait_full(pm);
  R.wait_full(pc);
  // Software pipelining of the steady state (LAG = 1): the level-0 pairs of the three rows a
  // step reads live in registers Z[m % 3] (newest row of step m), and right after level 1 the
  // step already waits for and loads the NEXT step's new row (one 16-byte LDS) and its centre
  // row's two x neighbours, so their shared-memory latency overlaps levels 2 .. K instead of
  // heading the next step's dependency chain (and 3 instead of 5 LDS per step).
  constexpr bool PF = NS == 3;
  double2 Z[3][PPT];
  double zW = 0.0, zE = 0.0;
  RingPos pnn = pn;  // steady steps: the next step's newest row
  // shared-window addresses fixed for the march, kept in registers (not re-derived from S2R
  // reads inside the loop, whose latency the dependent instructions would wait for)
  const uint32_t sbase = opaque_u32(sptr(R.stages) + 8u * (uint32_t)L.j0);
  const uint32_t fbase = opaque_u32(sptr(R.full)), ebase = opaque_u32(sptr(R.empty));
  auto wait_full_s = [&](const RingPos &p) { mbar_wait_s(fbase + 8u * p.slot, p.phase); };
  auto release_s = [&](const RingPos &p) { mbar_arrive_s(ebase + 8u * p.slot); };
  const uint32_t sstride = 8u * (uint32_t)(SD > 0 ? SD : R.stage_doubles);
  auto zload = [&](double2 *z, const RingPos &p) {
    const uint32_t st = sbase + p.slot * sstride;
#pragma unroll
    for (int i = 0; i < PPT; ++i) z[i] = lds2_s(st + 16u * i);
  };
  auto weload = [&](const RingPos &p) {
    const uint32_t st = sbase + p.slot * sstride;
    zW = lds_s(st - 8u);
    zE = lds_s(st + 16u * PPT);
  };
  auto step = [&](auto u_ct, auto steady_ct, int Rr) {
    constexpr int U = decltype(u_ct)::value;
    constexpr bool ST = decltype(steady_ct)::value;
    // level k-1 rows r+1, r, r-1 were computed at steps m-(LAG-1), m-LAG, m-LAG-1
    constexpr int SN = (U + NS - (LAG - 1)) % NS, SC = (U + NS - LAG) % NS, SS = (U + 2 * NS - LAG - 1) % NS;
    // level k computes row Rr-1-LAG(k-1) if it lies in its range [a-(K-k), b+(K-k)] ∩ [0, C+1]
    auto need = [&](int k, int r) { return r >= max(a - (K - k), 0) && r <= min(b + (K - k), C + 1); };
    // TB2_HOIST: the x neighbours of every level's centre row (computed in the previous step) are
    // shuffled at the start of the step, off the chain through this step's newest rows
    double WE[K - 1][2];
    if (TB2_HOIST && ST) {
#pragma unroll
      for (int k = 2; k <= K; ++k) {
        WE[k - 2][0] = shfl_up_d(X[k - 2][SC][PPT - 1].y);
        WE[k - 2][1] = shfl_down_d(X[k - 2][SC][0].x);
      }
    }
    if (ST && PF) {
      // level-0 rows Rr (newest, Z[U]), Rr-1 (centre, Z[U+2]), Rr-2 (Z[U+1]), preloaded
      constexpr int ZN = U % 3, ZC = (U + 2) % 3, ZO = (U + 1) % 3;
      tbk_level1_regs<PPT, FAST>(L, Z[REV ? ZN : ZO], Z[ZC], Z[REV ? ZO : ZN], zW, zE, X[0][U]);
      release_s(pm);  // row Rr-2: its last reads were the preloads
      // next step (steady steps end before r1): its newest row into Z[U+1] (row Rr-2's, now
      // dead), W / E of its centre row Rr
      pnn = pn;
      pnn.advance(R.S);
      wait_full_s(pnn);
      zload(Z[ZO], pnn);
      weload(pn);
    } else {
      if (ST || Rr <= r1) R.wait_full(pn);
      // (y-1, centre, y+1) rows: the march's older / newer neighbours, swapped when it runs down
      if (ST || need(1, Rr - 1))
        tbk_level1<PPT, FAST, ST>(L, R.stage(REV ? pn : pm), R.stage(pc), R.stage(REV ? pm : pn),
                                  Rr - 1 >= 1 && Rr - 1 <= C, X[0][U]);
      if (ST || (Rr - 2 >= r0 && Rr - 2 <= r1)) R.release(pm, lane);  // row Rr-2 is no longer needed
    }
#pragma unroll
    for (int k = 2; k < K; ++k) {
      const int r = Rr - 1 - LAG * (k - 1);
      if (ST || need(k, r))
        tbk_levelk<PPT, FAST, ST, false>(L, X[k - 2][REV ? SN : SS], X[k - 2][SC], X[k - 2][REV ? SS : SN],
                                         r >= 1 && r <= C, lane, X[k - 1][U], nullptr,
                                         (TB2_HOIST && ST) ? WE[k - 2] : nullptr);
    }
    const int ro = Rr - 1 - LAG * (K - 1);
    if (ST || (ro >= a && ro <= b))
      tbk_levelk<PPT, FAST, ST, true>(L, X[K - 2][REV ? SN : SS], X[K - 2][SC], X[K - 2][REV ? SS : SN], true, lane,
                                      nullptr, o, (TB2_HOIST && ST) ? WE[K - 2] : nullptr);
    o += ostep;
    pm = pc;
    pc = pn;
    if (ST && PF) {
      pn = pnn;
    } else if (Rr + 1 <= r1) {  // branch-free ring advance
      const uint32_t sl = pn.slot + 1u;
      const bool wrap = sl == R.S;
      pn.slot = wrap ? 0u : sl;
      pn.phase ^= wrap ? 1u : 0u;
    }
  };
  using TT = std::integral_constant<bool, true>;
  using TF = std::integral_constant<bool, false>;
  auto group = [&](auto steady_ct, int Rr) {
    constexpr bool ST = decltype(steady_ct)::value;
    step(std::integral_constant<int, 0>{}, steady_ct, Rr);
    if (ST || Rr + 1 <= Re) step(std::integral_constant<int, 1>{}, steady_ct, Rr + 1);
    if (ST || Rr + 2 <= Re) step(std::integral_constant<int, 2>{}, steady_ct, Rr + 2);
    if constexpr (NS == 4)
      if (ST || Rr + 3 <= Re) step(std::integral_constant<int, 3 % NS>{}, steady_ct, Rr + 3);
  };
  // groups of NS steps: a masked prefix, the steady middle, a masked suffix
  const int nsteady = Ws <= We ? (We - max(Ws, Rs) + 1) / NS : 0;  // whole steady groups
  int Rr = Rs;
  if (nsteady > 0) {
    for (; Rr < Ws; Rr += NS) group(TF{}, Rr);  // the prefix keeps the group phase (set rotation)
    // (with the preloads the steady steps end at We - 1: every one has a next row in the ring)
    const int Wend = PF ? We - 1 : We;
    if (Rr + NS - 1 <= Wend) {
      const int Rend = Rr + ((Wend - Rr + 1) / NS) * NS;
      if constexpr (PF) {  // preload the first steady step's rows (Rr, Rr-1, Rr-2 -> Z[0], Z[2], Z[1])
        R.wait_full(pn);
        zload(Z[0], pn);
        zload(Z[2], pc);
        zload(Z[1], pm);
        weload(pc);
      }
      for (; Rr < Rend; Rr += NS) group(TT{}, Rr);
    }
  }
  for (; Rr <= Re; Rr += NS) group(TF{}, Rr);
  // rows Re-1, Re (if they exist) were not released by the march: pm, pc after the last step
  if (Re - 1 <= r1) R.release(pm, lane);
  if (Re <= r1) R.release(pc, lane);
}

template <int K, int PPT, int LAG, int SD = 0>
__device__ __forceinline__ void tbk_item(const JbGeom &g, const Ring &R, RingPos &q, int unit, int64_t a, int64_t b,
                                         int64_t C, double *out, int warp, int lane) {
  constexpr int WO = 64 * PPT - 2 * (K - 1);
  const int64_t x0 = 1 + (int64_t)unit * g.tx;
  const int64_t r0 = max(a - K, (int64_t)0), r1 = min(b + K, C + 1);
  const RingPos q0 = q;
  q = ring_add(q, (uint32_t)(r1 - r0 + 1), R.S);
  const int64_t ow = x0 + (int64_t)warp * WO;  // first output column of this warp
  if (ow > g.nx - 2) {  // no outputs in this strip for this warp: only return the stages
    for (int64_t p = r0; p <= r1; ++p) {
      const RingPos pp = ring_add(q0, (uint32_t)(p - r0), R.S);
      R.wait_full(pp);
      R.release(pp, lane);
    }
    return;
  }
  const int64_t sw = ow - (K - 1);
  TbkLane L;
  L.j0 = warp * WO + 2 + 2 * PPT * lane;
  L.ok = L.full = L.st = 0;
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const int kk = PPT * lane + i;
    const int64_t c = sw + 2 * kk;
    const bool ok = c >= 1 && c <= g.nx - 2;
    L.ok |= (ok ? 1u : 0u) << i;
    L.full |= (ok && c + 1 <= g.nx - 2 ? 1u : 0u) << i;
    L.st |= (ok && kk >= (K - 1) / 2 && kk < 32 * PPT - (K - 1) / 2 ? 1u : 0u) << i;
  }
  const bool fast = sw >= 1 && sw + 64 * PPT - 1 <= g.nx - 2;
  double *dst = out + 3 + sw + 2 * PPT * lane;
  // march downwards (TB_REV): rows in mirrored coordinates r' = C+1-r
  const int ma = TB_REV ? (int)(C + 1 - b) : (int)a, mb = TB_REV ? (int)(C + 1 - a) : (int)b;
  const int m0 = TB_REV ? (int)(C + 1 - r1) : (int)r0, m1 = TB_REV ? (int)(C + 1 - r0) : (int)r1;
  if (fast) tbk_march<K, PPT, LAG, true, TB_REV, SD>(L, R, q0, ma, mb, (int)C, m0, m1, dst, g.plane_elems, lane);
  else tbk_march<K, PPT, LAG, false, TB_REV, SD>(L, R, q0, ma, mb, (int)C, m0, m1, dst, g.plane_elems, lane);
}

// ---------------------------------------------------------------- 3D (7-point)
// Tile = TY rows x tx columns (tx = 64 x warps), marched along z.  Lane `lane` of warp w owns the
// x pair kk = w*32 + lane for EVERY row of the tile, so level-1 y neighbours are its own
// registers; x neighbours come by shuffles (+ the two extra cells per warp segment and row, as
// in 2D).  Stage = level-0 rows y0-2 .. y0+TY+1 (stage row s <-> y0-2+s) of one plane.
//   level 1 (t+1): planes a-1 .. b+1, rows y0-1 .. y0+TY (Dirichlet rows/columns/planes keep level 0)
//   level 2 (t+2): planes a .. b, rows y0 .. y0+TY-1                            -> out
struct TbSeg3 {
  int j0;         // stage column index of this lane's pair
  bool ok, full;  // columns x0+2kk / x0+2kk+1 interior
  bool first, last;
  int sx;         // stage column of this lane's extra cell (lane 1: right end, others: left)
  bool ex_in;
  int y0, vy;     // first row of the tile, interior rows in it (<= TY)
};

// Level 1 of rows y0-1 .. y0+TY of one plane (stages sm / sc / sn = planes q1-1, q1, q1+1).
template <int TY, bool FAST>
__device__ __forceinline__ void tb3_level1(const TbSeg3 &L, const JbGeom &g, const double *sm, const double *sc,
                                           const double *sn, bool planein, double2 *V, double *ex) {
  const int ws = g.ws;
  const double *c = sc + L.j0, *u = sn + L.j0, *d = sm + L.j0;
  double2 Sy = lds2(c);       // stage row 0 = y0-2
  double2 Cy = lds2(c + ws);  // stage row 1 = y0-1
#pragma unroll
  for (int ry = 0; ry < TY + 2; ++ry) {  // level-1 row y0-1+ry = stage row ry+1
    const int o = (ry + 1) * ws;
    const double2 Ny = lds2(c + o + ws), U = lds2(u + o), D = lds2(d + o);
    const double W = c[o - 1], E = c[o + 2];
    // oracle order: x+1, x-1, y+1, y-1, z+1, z-1, then * fl(1/6)
    const double l0 = kC6 * (((((Cy.y + W) + Ny.x) + Sy.x) + U.x) + D.x);
    const double l1 = kC6 * (((((E + Cy.x) + Ny.y) + Sy.y) + U.y) + D.y);
    const int y = L.y0 - 1 + ry;
    const bool rowin = planein && y >= 1 && y <= (int)g.ny - 2;
    V[ry].x = (rowin && (FAST || L.ok)) ? l0 : Cy.x;
    V[ry].y = (rowin && (FAST || L.full)) ? l1 : Cy.y;
    Sy = Cy;
    Cy = Ny;
  }
  // extra cells of the output rows (ry = 1 .. TY)
  const double *ce = sc + L.sx, *ue = sn + L.sx, *de = sm + L.sx;
#pragma unroll
  for (int ry = 1; ry <= TY; ++ry) {
    const int o = (ry + 1) * ws;
    const double e = kC6 * (((((ce[o + 1] + ce[o - 1]) + ce[o + ws]) + ce[o - ws]) + ue[o]) + de[o]);
    const int y = L.y0 - 1 + ry;
    ex[ry - 1] = (planein && L.ex_in && y <= (int)g.ny - 2) ? e : ce[o];
  }
}

// Level 2 of the middle plane (level-1 planes Pm, Pc, Pn), rows y0 .. y0+TY-1, stored at o.
template <int TY, bool FAST>
__device__ __forceinline__ void tb3_level2(const TbSeg3 &L, const double2 *Pm, const double2 *Pc, const double2 *Pn,
                                           const double *exl, const double *exr, int lane, double *o,
                                           int64_t pitch) {
#pragma unroll
  for (int ry = 1; ry <= TY; ++ry) {
    const double rw = __shfl_sync(0xffffffffu, Pc[ry].y, (lane + 31) & 31);
    const double re = __shfl_sync(0xffffffffu, Pc[ry].x, (lane + 1) & 31);
    const double W = L.first ? exl[ry - 1] : rw;
    const double E = L.last ? exr[ry - 1] : re;
    const double o0 = kC6 * (((((Pc[ry].y + W) + Pc[ry + 1].x) + Pc[ry - 1].x) + Pn[ry].x) + Pm[ry].x);
    const double o1 = kC6 * (((((E + Pc[ry].x) + Pc[ry + 1].y) + Pc[ry - 1].y) + Pn[ry].y) + Pm[ry].y);
    double *p = o + (ry - 1) * pitch;
    if (FAST) *reinterpret_cast<double2 *>(p) = make_double2(o0, o1);
    else if (L.ok && ry - 1 < L.vy) store_pair(p, o0, o1, L.full);
  }
}

template <int TY, bool FAST>
__device__ __forceinline__ void tb3_march(const TbSeg3 &L, const JbGeom &g, const Ring &R, RingPos q, int64_t a,
                                          int64_t b, int64_t C, int64_t r0, int64_t r1, double *dst, int lane) {
  double2 Pm[TY + 2], Pc[TY + 2], Pn[TY + 2];
  double ex[TY], exl_c[TY], exr_c[TY], exl_n[TY], exr_n[TY];
  RingPos pc = ring_add(q, (uint32_t)(a - 1 - r0), R.S);
  RingPos pm = a - 2 >= r0 ? q : pc;
  R.wait_full(pm);
  R.wait_full(pc);
  auto plane = [&](int64_t q1, double2 *out) {
    RingPos pn = pc;
    if (q1 + 1 <= r1) pn.advance(R.S);
    R.wait_full(pn);
    tb3_level1<TY, FAST>(L, g, R.stage(pm), R.stage(pc), R.stage(pn), q1 >= 1 && q1 <= C, out, ex);
    if (q1 - 1 >= r0) R.release(pm, lane);
    pm = pc;
    pc = pn;
  };
  auto take_ex = [&](double *xl, double *xr) {
#pragma unroll
    for (int i = 0; i < TY; ++i) {
      xl[i] = __shfl_sync(0xffffffffu, ex[i], 0);
      xr[i] = __shfl_sync(0xffffffffu, ex[i], 1);
    }
  };
  plane(a - 1, Pc);
  plane(a, Pn);
  take_ex(exl_n, exr_n);
  double *o = dst + a * g.plane_elems;
  for (int64_t q1 = a + 1; q1 <= b + 1; ++q1) {
#pragma unroll
    for (int i = 0; i < TY + 2; ++i) {
      Pm[i] = Pc[i];
      Pc[i] = Pn[i];
    }
#pragma unroll
    for (int i = 0; i < TY; ++i) {
      exl_c[i] = exl_n[i];
      exr_c[i] = exr_n[i];
    }
    plane(q1, Pn);
    take_ex(exl_n, exr_n);
    tb3_level2<TY, FAST>(L, Pm, Pc, Pn, exl_c, exr_c, lane, o, g.pitch);
    o += g.plane_elems;
  }
  RingPos pr = ring_add(q, (uint32_t)(b + 1 - r0), R.S);
  for (int64_t p = b + 1; p <= r1; ++p) {
    R.release(pr, lane);
    pr.advance(R.S);
  }
}

template <int TY>
__device__ __forceinline__ void tb3_item(const JbGeom &g, const Ring &R, RingPos &q, int unit, int64_t a,
                                         int64_t b, int64_t C, double *out, int warp, int lane) {
  const int ux = unit % g.units_x, uy = unit / g.units_x;
  const int64_t x0 = 1 + (int64_t)ux * g.tx;
  const int vx = (int)min((int64_t)g.tx, g.nx - 1 - x0);
  const int txp = g.tx >> 1;
  const int seg_b = warp * 32, seg_e = min(seg_b + 32, txp);
  const int64_t r0 = max(a - 2, (int64_t)0), r1 = min(b + 2, C + 1);
  const RingPos q0 = q;
  q = ring_add(q, (uint32_t)(r1 - r0 + 1), R.S);
  const int kk = seg_b + lane;
  if (seg_b >= seg_e) {
    for (int64_t p = r0; p <= r1; ++p) {
      const RingPos pp = ring_add(q0, (uint32_t)(p - r0), R.S);
      R.wait_full(pp);
      R.release(pp, lane);
    }
    return;
  }
  TbSeg3 L;
  L.j0 = 2 + 2 * min(kk, seg_e - 1);  // lanes past the tile read (and discard) the last pair
  L.ok = kk < seg_e && 2 * kk < vx;
  L.full = kk < seg_e && 2 * kk + 1 < vx;
  L.first = kk == seg_b;
  L.last = kk == seg_e - 1;
  L.sx = lane == 1 ? 2 * seg_e + 2 : 2 * seg_b + 1;
  const int64_t cx = x0 - 2 + L.sx;
  L.ex_in = cx >= 1 && cx <= g.nx - 2;
  L.y0 = 1 + uy * TY;
  L.vy = (int)min((int64_t)TY, g.ny - 1 - L.y0);
  const bool fast = seg_e - seg_b == 32 && 2 * seg_e <= vx && L.vy == TY;
  double *dst = out + (int64_t)L.y0 * g.pitch + 3 + x0 + 2 * kk;
  if (fast) tb3_march<TY, true>(L, g, R, q0, a, b, C, r0, r1, dst, lane);
  else tb3_march<TY, false>(L, g, R, q0, a, b, C, r0, r1, dst, lane);
}

// ---------------------------------------------------------------- 3D, deeper time blocks (K odd)
// Tile = TY = NCW·RPW rows x TX = 64·PPT columns, computed at every level and marched along z.
// Warp w owns the tile rows w·RPW .. w·RPW+RPW-1, lane l the contiguous pairs kk = l·PPT + i.
// Neighbours of a level-(k-1) cell: x — own registers / one shuffle per side (as 2D); y — own
// registers, except above the warp's first and below its last row: the neighbouring warps'
// boundary rows, exchanged through shared memory (double-buffered by step parity, so ONE
// consumer barrier per step orders them); z — the level's previous / next plane, in registers
// (z wavefront with LAG = 1, three planes per level).  Every level loses one valid column and
// row per side at the tile's edges (the tile's outermost warps / lanes have no neighbour data),
// so level K is valid on the middle WO = TX - 2(K-1) columns and HO = TY - 2(K-1) rows: the
// tile's outputs (g.tx = WO, g.ty = HO).  Level 1 reads the level-0 stage, which holds the
// tile's rows plus one on each side, so it is valid everywhere.  K odd keeps 16-byte alignment.
struct Tb3kLane {
  int j0;                // stage column index of pair 0 of this lane (stage col 0 <-> s - 2)
  unsigned ok, full, st; // per pair: x / x+1 interior, stored at level K
  unsigned rok, rst;     // per row of the warp: interior row, stored at level K
};

template <int NCW>
__device__ __forceinline__ void bar_consumers() {
  asm volatile("bar.sync 1, %0;" ::"r"(NCW * 32) : "memory");
}

// Level 1 of the warp's RPW rows of the plane whose level-0 stages are zm (z-1), zc, zp (z+1).
template <int PPT, int RPW, bool FAST, bool STEADY>
__device__ __forceinline__ void tb3k_level1(const Tb3kLane &L, int sr0, int ws, const double *zm, const double *zc,
                                            const double *zp, bool planein, double2 (*V)[PPT]) {
  double2 Cr[RPW + 2][PPT];  // rows sr0-1 .. sr0+RPW of the centre plane
#pragma unroll
  for (int j = 0; j < RPW + 2; ++j)
#pragma unroll
    for (int i = 0; i < PPT; ++i) Cr[j][i] = lds2(zc + (sr0 - 1 + j) * ws + L.j0 + 2 * i);
#pragma unroll
  for (int j = 0; j < RPW; ++j) {
    const int o = (sr0 + j) * ws + L.j0;
    const double Wl = zc[o - 1], Er = zc[o + 2 * PPT];
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      const double2 Up = lds2(zp + o + 2 * i), Dn = lds2(zm + o + 2 * i);
      const double2 C = Cr[j + 1][i], N = Cr[j + 2][i], S = Cr[j][i];
      const double W = i == 0 ? Wl : Cr[j + 1][i - 1].y;
      const double E = i == PPT - 1 ? Er : Cr[j + 1][i + 1].x;
      // oracle order: x+1, x-1, y+1, y-1, z+1, z-1, then * fl(1/6)
      const double l0 = kC6 * (((((C.y + W) + N.x) + S.x) + Up.x) + Dn.x);
      const double l1 = kC6 * (((((E + C.x) + N.y) + S.y) + Up.y) + Dn.y);
      if (FAST && STEADY) {
        V[j][i] = make_double2(l0, l1);
      } else {
        const bool r = (STEADY || planein) && (FAST || (L.rok >> j & 1u));
        V[j][i].x = (r && (FAST || (L.ok >> i & 1u))) ? l0 : C.x;
        V[j][i].y = (r && (FAST || (L.full >> i & 1u))) ? l1 : C.y;
      }
    }
  }
}

// Level 1 as tb3k_level1 (steady state: every row and plane interior), with the warp's own
// level-0 rows of the three planes already in registers (Dn: z-1, Cc: z, Up: z+1); only the
// centre plane's rows just above / below the warp and the x neighbours at the lane pair's ends
// come from the centre plane's stage zc.
template <int PPT, int RPW, bool FAST>
__device__ __forceinline__ void tb3k_level1_regs(const Tb3kLane &L, int sr0, int ws, const double *zc,
                                                 const double2 (*Dn)[PPT], const double2 (*Cc)[PPT],
                                                 const double2 (*Up)[PPT], double2 (*V)[PPT]) {
  double2 T[PPT], B[PPT];  // centre-plane rows sr0-1 and sr0+RPW
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    T[i] = lds2(zc + (sr0 - 1) * ws + L.j0 + 2 * i);
    B[i] = lds2(zc + (sr0 + RPW) * ws + L.j0 + 2 * i);
  }
#pragma unroll
  for (int j = 0; j < RPW; ++j) {
    const int o = (sr0 + j) * ws + L.j0;
    const double Wl = zc[o - 1], Er = zc[o + 2 * PPT];
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      const double2 C = Cc[j][i];
      const double2 N = j + 1 < RPW ? Cc[j + 1 < RPW ? j + 1 : j][i] : B[i];
      const double2 S = j > 0 ? Cc[j > 0 ? j - 1 : j][i] : T[i];
      const double W = i == 0 ? Wl : Cc[j][i > 0 ? i - 1 : 0].y;
      const double E = i == PPT - 1 ? Er : Cc[j][i + 1 < PPT ? i + 1 : i].x;
      // oracle order: x+1, x-1, y+1, y-1, z+1, z-1, then * fl(1/6)
      const double l0 = kC6 * (((((C.y + W) + N.x) + S.x) + Up[j][i].x) + Dn[j][i].x);
      const double l1 = kC6 * (((((E + C.x) + N.y) + S.y) + Up[j][i].y) + Dn[j][i].y);
      if (FAST) {
        V[j][i] = make_double2(l0, l1);
      } else {
        V[j][i].x = (L.rok >> j & 1u) && (L.ok >> i & 1u) ? l0 : C.x;
        V[j][i].y = (L.rok >> j & 1u) && (L.full >> i & 1u) ? l1 : C.y;
      }
    }
  }
}

// Level k >= 2 of the warp's rows of the centre plane Zc (level k-1 planes Zm, Zc, Zp); yT / yB:
// the level-(k-1) rows just above / below the warp (other warps' boundary rows).  STORE: level
// K, pair i of row j stored at o + j·pitch + 2i.
template <int PPT, int RPW, bool FAST, bool STEADY, bool STORE>
__device__ __forceinline__ void tb3k_levelk(const Tb3kLane &L, const double2 (*Zm)[PPT], const double2 (*Zc)[PPT],
                                            const double2 (*Zp)[PPT], const double2 *yT, const double2 *yB,
                                            bool planein, int lane, double2 (*V)[PPT], double *o, int64_t pitch) {
#pragma unroll
  for (int j = 0; j < RPW; ++j) {
    const double Wl = shfl_d(Zc[j][PPT - 1].y, (lane + 31) & 31);
    const double Er = shfl_d(Zc[j][0].x, (lane + 1) & 31);
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      const double2 C = Zc[j][i];
      const double2 N = j + 1 < RPW ? Zc[j + 1 < RPW ? j + 1 : j][i] : yB[i];
      const double2 S = j > 0 ? Zc[j > 0 ? j - 1 : j][i] : yT[i];
      const double W = i == 0 ? Wl : Zc[j][i > 0 ? i - 1 : 0].y;
      const double E = i == PPT - 1 ? Er : Zc[j][i + 1 < PPT ? i + 1 : i].x;
      const double2 Up = Zp[j][i], Dn = Zm[j][i];
      const double o0 = kC6 * (((((C.y + W) + N.x) + S.x) + Up.x) + Dn.x);
      const double o1 = kC6 * (((((E + C.x) + N.y) + S.y) + Up.y) + Dn.y);
      if (STORE) {
        if ((L.rst >> j & 1u) && (L.st >> i & 1u)) {
          double *po = o + j * pitch + 2 * i;
          if (FAST) *reinterpret_cast<double2 *>(po) = make_double2(o0, o1);
          else store_pair(po, o0, o1, L.full >> i & 1u);
        }
      } else if (FAST && STEADY) {
        V[j][i] = make_double2(o0, o1);
      } else {
        const bool r = (STEADY || planein) && (FAST || (L.rok >> j & 1u));
        V[j][i].x = (r && (FAST || (L.ok >> i & 1u))) ? o0 : C.x;
        V[j][i].y = (r && (FAST || (L.full >> i & 1u))) ? o1 : C.y;
      }
    }
  }
}

// REV (TB_REV): the z march runs towards plane 0 (a, b, r0, r1 in mirrored plane indices
// p' = C+1-p), so the newest level plane is z-1, the last term of the oracle order: two instead
// of three dependent fp64 operations per level on the step's critical path (see tbk_march).
template <int K, int PPT, int RPW, int NCW, bool FAST, bool REV>
__device__ __forceinline__ void tb3k_march(const Tb3kLane &L, const JbGeom &g, const Ring &R, RingPos q, int a,
                                           int b, int C, int r0, int r1, double *dst, double *xch, int warp,
                                           int lane) {
  constexpr int NS = 3;
  constexpr int TX = 64 * PPT;
  double2 X[K - 1][NS][RPW][PPT];  // X[k-1][m % 3]: level k of the plane computed at step m
  const int Rs = a - K >= 0 ? r0 + 2 : r0 + 1;
  const int Re = b + K;
  const int Ws = a + K, We = min(b + K, C + 1);
  const int ws = g.ws, sr0 = warp * RPW + 1;
  const int64_t pe = g.plane_elems, pitch = g.pitch;
  double *o = dst + (int64_t)(REV ? C + 1 - (Rs - K) : Rs - K) * pe;
  const int64_t ostep = REV ? -pe : pe;
  // exchange slots: [level k-1][parity][warp][0 = first row, 1 = last row][TX]
  auto xrow = [&](int k1, int par, int w, int side) { return xch + ((((k1 * 2 + par) * NCW + w) * 2 + side) * TX); };
  const int wu = warp > 0 ? warp - 1 : warp, wd = warp + 1 < NCW ? warp + 1 : warp;  // edge warps: any row
  RingPos pm = q, pc = Rs == r0 + 2 ? ring_add(q, 1u, R.S) : q, pn = pc;
  if (Rs <= r1) pn = ring_add(q, (uint32_t)(Rs - r0), R.S);
  R.wait_full(pm);
  R.wait_full(pc);
  auto publish = [&](int k1, int par, const double2 (*V)[PPT]) {
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      *reinterpret_cast<double2 *>(xrow(k1, par, warp, 0) + 2 * (lane * PPT + i)) = V[0][i];
      *reinterpret_cast<double2 *>(xrow(k1, par, warp, 1) + 2 * (lane * PPT + i)) = V[RPW - 1][i];
    }
  };
  // Steady state (TB3_PF): the warp's own level-0 rows of the three planes a step reads stay in
  // registers Z[m % 3] (newest plane of step m), so each step loads only its new plane's own rows
  // and the centre plane's two rows just outside the warp: RPW + 2 instead of 3 RPW + 2 row
  // loads (LDS.128) per step — the 3D march is bound by its shared-memory pipe.
  // (Loading the next step's plane right after level 1, as the 2D march does, needs more live
  // registers here and spills: measured slower.)
  constexpr bool PF = TB3_PF;
  double2 Z[PF ? 3 : 1][RPW][PPT];
  auto zload = [&](double2 (*z)[PPT], const RingPos &p) {
    const double *st = R.stage(p) + sr0 * ws + L.j0;
#pragma unroll
    for (int j = 0; j < RPW; ++j)
#pragma unroll
      for (int i = 0; i < PPT; ++i) z[j][i] = lds2(st + j * ws + 2 * i);
  };
  auto step = [&](auto u_ct, auto steady_ct, int Rr) {
    constexpr int U = decltype(u_ct)::value;
    constexpr bool ST = decltype(steady_ct)::value;
    constexpr int SN = U, SC = (U + NS - 1) % NS, SS = (U + NS - 2) % NS;
    const int par = Rr & 1, prv = par ^ 1;
    auto need = [&](int k, int r) { return r >= max(a - (K - k), 0) && r <= min(b + (K - k), C + 1); };
    if (ST && PF) {
      // level-0 planes Rr (newest, Z[U]), Rr-1 (centre, Z[U+2]), Rr-2 (Z[U+1])
      constexpr int ZN = PF ? U % 3 : 0, ZC = PF ? (U + 2) % 3 : 0, ZO = PF ? (U + 1) % 3 : 0;
      R.wait_full(pn);
      zload(Z[ZN], pn);
      bar_consumers<NCW>();  // the previous step's exchange rows are visible; its reads are done
      tb3k_level1_regs<PPT, RPW, FAST>(L, sr0, ws, R.stage(pc), Z[REV ? ZN : ZO], Z[ZC], Z[REV ? ZO : ZN], X[0][U]);
      publish(0, par, X[0][U]);
      R.release(pm, lane);  // plane Rr-2: its last reads were the register loads
    } else {
    if (ST || Rr <= r1) R.wait_full(pn);
    bar_consumers<NCW>();  // the previous step's exchange rows are visible; its reads are done
    if (ST || need(1, Rr - 1)) {
      tb3k_level1<PPT, RPW, FAST, ST>(L, sr0, ws, R.stage(REV ? pn : pm), R.stage(pc), R.stage(REV ? pm : pn),
                                      Rr - 1 >= 1 && Rr - 1 <= C,
                                      X[0][U]);
      publish(0, par, X[0][U]);
    }
    if (ST || (Rr - 2 >= r0 && Rr - 2 <= r1)) R.release(pm, lane);
    }
#pragma unroll
    for (int k = 2; k <= K; ++k) {
      const int r = Rr - k;
      if (!(ST || need(k, r))) continue;
      double2 yT[PPT], yB[PPT];
#pragma unroll
      for (int i = 0; i < PPT; ++i) {
        yT[i] = lds2(xrow(k - 2, prv, wu, 1) + 2 * (lane * PPT + i));
        yB[i] = lds2(xrow(k - 2, prv, wd, 0) + 2 * (lane * PPT + i));
      }
      if (k < K) {
        tb3k_levelk<PPT, RPW, FAST, ST, false>(L, X[k - 2][REV ? SN : SS], X[k - 2][SC], X[k - 2][REV ? SS : SN], yT, yB,
                                               r >= 1 && r <= C, lane, X[k - 1][U], nullptr, pitch);
        publish(k - 1, par, X[k - 1][U]);
      } else {
        tb3k_levelk<PPT, RPW, FAST, ST, true>(L, X[k - 2][REV ? SN : SS], X[k - 2][SC], X[k - 2][REV ? SS : SN], yT, yB,
                                              true, lane,
                                              nullptr, o, pitch);
      }
    }
    o += ostep;
    pm = pc;
    pc = pn;
    if ((ST && PF) || Rr + 1 <= r1) {  // (steady steps always have a next plane)
      const uint32_t sl = pn.slot + 1u;
      const bool wrap = sl == R.S;
      pn.slot = wrap ? 0u : sl;
      pn.phase ^= wrap ? 1u : 0u;
    }
  };
  using TT = std::integral_constant<bool, true>;
  using TF = std::integral_constant<bool, false>;
  auto group = [&](auto steady_ct, int Rr) {
    constexpr bool ST = decltype(steady_ct)::value;
    step(std::integral_constant<int, 0>{}, steady_ct, Rr);
    if (ST || Rr + 1 <= Re) step(std::integral_constant<int, 1>{}, steady_ct, Rr + 1);
    if (ST || Rr + 2 <= Re) step(std::integral_constant<int, 2>{}, steady_ct, Rr + 2);
  };
  int Rr = Rs;
  if (Ws <= We) {
    for (; Rr < Ws; Rr += NS) group(TF{}, Rr);
    // (the steady steps end at We - 1: every one has a next plane in the ring)
    const int Wend = PF ? We - 1 : We;
    if (Rr + NS - 1 <= Wend) {
      const int Rend = Rr + ((Wend - Rr + 1) / NS) * NS;
      if constexpr (PF) {  // the first steady step's older planes (Rr-1, Rr-2 -> Z[2], Z[1])
        R.wait_full(pn);
        zload(Z[PF ? 2 : 0], pc);
        zload(Z[PF ? 1 : 0], pm);
      }
      for (; Rr < Rend; Rr += NS) group(TT{}, Rr);
    }
  }
  for (; Rr <= Re; Rr += NS) group(TF{}, Rr);
  if (Re - 1 <= r1) R.release(pm, lane);
  if (Re <= r1) R.release(pc, lane);
}

template <int K, int PPT, int RPW, int NCW>
__device__ __forceinline__ void tb3k_item(const JbGeom &g, const Ring &R, RingPos &q, int unit, int64_t a, int64_t b,
                                          int64_t C, double *out, double *xch, int warp, int lane) {
  constexpr int TY = NCW * RPW;
  const int ux = unit % g.units_x, uy = unit / g.units_x;
  const int64_t x0 = 1 + (int64_t)ux * g.tx, y0 = 1 + (int64_t)uy * g.ty;
  const int64_t sx = x0 - (K - 1), sy = y0 - (K - 1);  // first computed column / row of the tile
  const int64_t r0 = max(a - K, (int64_t)0), r1 = min(b + K, C + 1);
  const RingPos q0 = q;
  q = ring_add(q, (uint32_t)(r1 - r0 + 1), R.S);
  Tb3kLane L;
  L.j0 = 2 + 2 * PPT * lane;
  L.ok = L.full = L.st = L.rok = L.rst = 0;
#pragma unroll
  for (int i = 0; i < PPT; ++i) {
    const int kk = PPT * lane + i;
    const int64_t c = sx + 2 * kk;
    const bool ok = c >= 1 && c <= g.nx - 2;
    L.ok |= (ok ? 1u : 0u) << i;
    L.full |= (ok && c + 1 <= g.nx - 2 ? 1u : 0u) << i;
    L.st |= (ok && kk >= (K - 1) / 2 && kk < 32 * PPT - (K - 1) / 2 ? 1u : 0u) << i;
  }
#pragma unroll
  for (int j = 0; j < RPW; ++j) {
    const int t = warp * RPW + j;  // tile row
    const int64_t y = sy + t;
    const bool rok = y >= 1 && y <= g.ny - 2;
    L.rok |= (rok ? 1u : 0u) << j;
    L.rst |= (rok && t >= K - 1 && t <= TY - K ? 1u : 0u) << j;
  }
  const bool fast = sx >= 1 && sx + 64 * PPT - 1 <= g.nx - 2 && sy >= 1 && sy + TY - 1 <= g.ny - 2;
  double *dst = out + (sy + (int64_t)warp * RPW) * g.pitch + 3 + sx + 2 * PPT * lane;
  const int ma = TB_REV ? (int)(C + 1 - b) : (int)a, mb = TB_REV ? (int)(C + 1 - a) : (int)b;
  const int m0 = TB_REV ? (int)(C + 1 - r1) : (int)r0, m1 = TB_REV ? (int)(C + 1 - r0) : (int)r1;
  if (fast)
    tb3k_march<K, PPT, RPW, NCW, true, TB_REV>(L, g, R, q0, ma, mb, (int)C, m0, m1, dst, xch, warp, lane);
  else
    tb3k_march<K, PPT, RPW, NCW, false, TB_REV>(L, g, R, q0, ma, mb, (int)C, m0, m1, dst, xch, warp, lane);
}

// Edge zone of a slab side with a neighbour (time block t -> t+K), computed by that side's
// boundary CTAs with the whole CTA, so the halo exchange stays per iteration.
// Phase m = 1..K: wait until the neighbour delivered its level m-1 plane (m = 1: the time-t halo
// in `cur`; m >= 2: our slot m-1 in the scratch), then compute level m (t+m) of the planes next to
// the halo — 2K-m of them for m < K over the strip window widened by K-m cells per side (the
// next phase reads one cell further), the K output planes (tile cells only) for m = K — and store
// the outermost plane also to the neighbour: its slot m (m < K) or its halo (m = K); signal t+m.
// The interior items then cover level-K planes K+1 .. C-K, which need no halo.
// Scratch E (per side, jb_edge_planes_k(K) planes; E_top after buf[0], E_bot after buf[1]):
//   [m-1], m = 1..K-1           the neighbour's level-m plane (written by the neighbour)
//   [lbase(m) + i], i < 2K-m    this side's level-m plane first(m) + i (top: 1 + i,
//                               bottom: C-2K+m+1 + i)
// Loads bypass L1 (ld.cg): these planes are rewritten by other CTAs / the neighbour GPU.
__device__ __forceinline__ double2 ldcg2(const double *p) { return __ldcg(reinterpret_cast<const double2 *>(p)); }

// One phase, vectorised: a thread owns one 16-byte cell pair (x odd, x+1; 3D: of one row y) of the
// window and marches it through the phase's NP planes, keeping the level-(m-1) pairs of the
// march's three consecutive planes in registers (loaded once each, every load issued up front),
// so a cell update costs 1.5 loads in 2D (pair + its two x neighbours per plane, the plane
// neighbours are the march's registers) and 2.5 in 3D, and every store is a 16-byte store into
// the local scratch / next buffer and, for the outermost plane, straight into the neighbour's
// slot or halo.  Same oracle order; cells outside the interior keep level m-1.
template <int DIM, int K, int M, int NT>
__device__ __forceinline__ void tb_edge_phase(const JbGeom &g, bool top, int64_t C, const double *cur, double *E,
                                              double *nxt, double *mid, double *remote, int ub, int ue) {
  constexpr int NP = M < K ? 2 * K - M : K;  // level-M planes of this side
  constexpr int NPV = 2 * K - (M - 1);       // level-(M-1) planes of this side (M >= 2)
  constexpr int MG = K - M;                  // window margin
  const int64_t pe = g.plane_elems, pitch = g.pitch;
  const int nx = (int)g.nx, ny = (int)g.ny;
  const int64_t pf = top ? 1 : C - NP + 1;  // first level-M plane
  const int64_t pfv = top ? 1 : C - NPV + 1;
  const int64_t halo = top ? 0 : C + 1;
  auto lbase = [](int m) { return (int64_t)(K - 1) + (int64_t)(m - 1) * 2 * K - (int64_t)(m - 1) * m / 2; };
  // level M-1 of plane p (element offset 3 of x = 0, row 0)
  auto src = [&](int64_t p) -> const double * {
    if (M == 1) return cur + p * pe + 3;
    if (p == halo) return E + (int64_t)(M - 2) * pe;
    return E + (lbase(M - 1) + (p - pfv)) * pe;
  };
  auto dst = [&](int k) -> double * { return M < K ? E + (lbase(M) + k) * pe : nxt + (pf + k) * pe + 3; };
  double *d2 = M < K ? mid + (int64_t)(M - 1) * pe : remote + 3;  // the neighbour's slot / halo
  const int kout = top ? 0 : NP - 1;                               // plane index of pout
  for (int u = ub; u < ue; ++u) {
    const int ux = u % g.units_x, uy = u / g.units_x;
    const int x0 = 1 + ux * g.tx;
    int xa, xb, ya = 0, yb = 0;
    if (M < K) {
      xa = max(x0 - MG, 0);
      xb = min(x0 + g.tx - 1 + MG, nx - 1);
    } else {
      xa = x0;
      xb = min(x0 + g.tx, nx - 1) - 1;
    }
    if (DIM == 3) {
      const int y0 = 1 + uy * g.ty;
      if (M < K) {
        ya = max(y0 - MG, 0);
        yb = min(y0 + g.ty - 1 + MG, ny - 1);
      } else {
        ya = y0;
        yb = min(y0 + g.ty, ny - 1) - 1;
      }
    }
    const int xp0 = (xa & 1) ? xa : xa - 1;  // first pair (x odd: 16-byte aligned)
    const int npx = (xb - xp0) / 2 + 1;
    const int items = npx * (yb - ya + 1);
    for (int c = threadIdx.x; c < items; c += NT) {
      const int ry = DIM == 3 ? c / npx : 0;
      const int x = xp0 + 2 * (c - ry * npx), y = ya + ry;
      const int64_t e = (DIM == 3 ? (int64_t)y * pitch : 0) + x;
      const bool yin = DIM == 2 || (y >= 1 && y <= ny - 2);
      const bool in0 = yin && x >= 1 && x <= nx - 2, in1 = yin && x + 1 >= 1 && x + 1 <= nx - 2;
      const bool st0 = x >= xa, st1 = x + 1 <= xb;
      // y neighbours of the Dirichlet rows are never used: keep their loads inside the plane
      const int64_t yn = (DIM == 3 && y < ny - 1) ? pitch : 0, ys = (DIM == 3 && y > 0) ? -pitch : 0;
      double2 Cp[NP + 2];  // level M-1 pairs of planes pf-1 .. pf+NP
#pragma unroll
      for (int i = 0; i < NP + 2; ++i) Cp[i] = ldcg2(src(pf - 1 + i) + e);
#pragma unroll
      for (int k = 0; k < NP; ++k) {
        const double *A = src(pf + k) + e;
        const double W = __ldcg(A - 1), Ee = __ldcg(A + 2);
        const double2 c0 = Cp[k + 1];
        double v0, v1;
        if (DIM == 2) {  // oracle order: x+1, x-1, y+1 (plane p+1), y-1 (plane p-1), then * 1/4
          v0 = 0.25 * (((c0.y + W) + Cp[k + 2].x) + Cp[k].x);
          v1 = 0.25 * (((Ee + c0.x) + Cp[k + 2].y) + Cp[k].y);
        } else {  // x+1, x-1, y+1, y-1, z+1 (plane p+1), z-1 (plane p-1), then * fl(1/6)
          const double2 N = ldcg2(A + yn), S = ldcg2(A + ys);
          v0 = kC6 * (((((c0.y + W) + N.x) + S.x) + Cp[k + 2].x) + Cp[k].x);
          v1 = kC6 * (((((Ee + c0.x) + N.y) + S.y) + Cp[k + 2].y) + Cp[k].y);
        }
        const double2 v = make_double2(in0 ? v0 : c0.x, in1 ? v1 : c0.y);
        auto put = [&](double *d) {
          if (st0 && st1) *reinterpret_cast<double2 *>(d) = v;
          else if (st0) d[0] = v.x;
          else if (st1) d[1] = v.y;
        };
        put(dst(k) + e);
        if (k == kout) put(d2 + e);
      }
    }
  }
}

// Not inlined: its fully unrolled phases would otherwise raise the register pressure of the
// interior march they share the kernel with (measured: spills in the hot loop).
// Run by the consumer warps (threads 0 .. NT-1) only, ordered among themselves by named barrier
// 2; the producer warp meanwhile already streams the block's interior rows.
template <int DIM, int K, int NT>
__device__ __noinline__ bool tb_edge(const JbGeom &g, const JbSlab &SL, const JbParams &P, int role, int ridx, int rcount,
                        const double *cur, double *nxt, double *remote, int64_t tg, int *s_flag) {
  const bool top = role == ROLE_TOP;
  const int64_t C = SL.chunk, pe = g.plane_elems;
  double *E = (top ? SL.buf[0] : SL.buf[1]) + (C + 2) * pe + 3;
  double *mid = (top ? SL.mid_top_out : SL.mid_bot_out) + 3;
  const unsigned long long *fin = top ? SL.flag_in_top : SL.flag_in_bot;
  const int kin = top ? SL.k_in_top : SL.k_in_bot;
  unsigned long long *fout = (top ? SL.flag_out_top : SL.flag_out_bot) + ridx;
  const int ub = (int)((int64_t)g.units * ridx / rcount), ue = (int)((int64_t)g.units * (ridx + 1) / rcount);
  const int tid = threadIdx.x;
  const bool drop = (P.flags & JACOBI_FLAG_DROP_SIGNAL) && SL.slab_id == 0;
  const int side = top ? 0 : 1;
  auto bar_edge = [] { asm volatile("barrier.sync 2, %0;" ::"n"(NT) : "memory"); };  // non-.aligned
  const bool mark = ridx == 0 && tid == 0;
  auto wait = [&](unsigned long long target) {
    if (tid < 32) {
      if (mark) halo_mark(SL, P, side, (int64_t)target - P.t0, 0);
      const bool ok = wait_slots(fin, kin, target, P, tid);
      if (tid == 0) *s_flag = ok ? 0 : 1;
      if (mark) halo_mark(SL, P, side, (int64_t)target - P.t0, 1);
    }
    bar_edge();
    return *s_flag == 0;
  };
#pragma unroll
  for (int m = 1; m <= K; ++m) {
    if (!wait((unsigned long long)(tg + m - 1))) return false;
    // level m (compile-time per phase: the march and its loads are fully unrolled)
    if (m == 1) tb_edge_phase<DIM, K, 1, NT>(g, top, C, cur, E, nxt, mid, remote, ub, ue);
    if constexpr (K >= 2) if (m == 2) tb_edge_phase<DIM, K, 2, NT>(g, top, C, cur, E, nxt, mid, remote, ub, ue);
    if constexpr (K >= 3) if (m == 3) tb_edge_phase<DIM, K, 3, NT>(g, top, C, cur, E, nxt, mid, remote, ub, ue);
    if constexpr (K >= 4) if (m == 4) tb_edge_phase<DIM, K, 4, NT>(g, top, C, cur, E, nxt, mid, remote, ub, ue);
    if constexpr (K >= 5) if (m == 5) tb_edge_phase<DIM, K, 5, NT>(g, top, C, cur, E, nxt, mid, remote, ub, ue);
    bar_edge();  // every thread's stores (local, neighbour's) precede the release below
    if (tid == 0 && !drop) st_release_flag(P, fout, (unsigned long long)(tg + m));
    if (mark) halo_mark(SL, P, side, tg + m - 1 - P.t0, 2);
  }
  return true;
}

// WS = 1: warp-specialised register split — 4 + NCW warps, the last warpgroup (warp NCW = the
// producer, three idle warps) gives registers back with setmaxnreg.dec and the NCW consumer
// warps (whole warpgroups) take them with setmaxnreg.inc: 12 compute warps at 160 registers
// where one producer warp per CTA would leave 11 at 168 (each SM sub-partition holds 16 K
// registers: 32 + 3 x 160 = 512 per lane slot).
template <int NCW, int DIM, int K, int TP, int LAG, int RPW, int WS = 0>
__device__ __forceinline__ void tb_body(const JbParams &P) {
  static_assert(!WS || NCW % 4 == 0, "warp specialisation needs whole consumer warpgroups");
  static_assert(K == 2 || (K & 1), "K = 2 or odd");
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int s_abort;
  __shared__ int s_edge;  // the edge zones' wait result (own variable: s_abort is read after the barrier)
  const JbGeom &g = P.g;
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
  Ring R;
  R.S = (uint32_t)g.stages;
  R.stage_doubles = g.stage_doubles;
  R.full = reinterpret_cast<uint64_t *>(smem);
  R.empty = R.full + R.S;
  uint64_t *qfull = R.empty + R.S;
  uint64_t *qempty = qfull + JB_RQ;
  TbDesc *desc = reinterpret_cast<TbDesc *>(qempty + JB_RQ);
  const uint32_t hdr = 2 * R.S * 8 + 2 * JB_RQ * 8 + JB_RQ * (uint32_t)sizeof(TbDesc);
  R.stages = reinterpret_cast<double *>(smem + ((hdr + 127) & ~127u));

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const bool producer = warp == NCW;
  const bool consumer = warp < NCW;  // (WS: warps NCW+1 .. NCW+3 are idle)
  if (threadIdx.x == 0) {
    for (uint32_t i = 0; i < R.S; ++i) {
      mbar_init(&R.full[i], 1);
      mbar_init(&R.empty[i], NCW * 32);  // one arrival per consumer thread (Ring::release)
    }
    for (int i = 0; i < JB_RQ; ++i) {
      mbar_init(&qfull[i], 1);
      mbar_init(&qempty[i], NCW);
    }
    fence_mbar_init();
    s_abort = 0;
  }
  __syncthreads();
  const int64_t C = SL.chunk;
  const int64_t nblocks = P.iters / K;
  RingPos q = {0u, 0u}, rq = {0u, 0u};
  // The time blocks.  RG = which warps run this copy of the loop: 0 every warp (WS = 0), 1 the
  // producer warpgroup, 2 the consumer warps (WS = 1: two separate loops, so the register limits
  // of setmaxnreg apply to whole code regions; both meet at the same grid-barrier bar.sync 0).
  auto blocks = [&](auto rg_ct) {
    constexpr int RG = decltype(rg_ct)::value;
    for (int64_t j = 0; j < nblocks; ++j) {
      const double *cur = SL.buf[(P.t0 + j) & 1];
      double *nxt = SL.buf[(P.t0 + j + 1) & 1];
      const int64_t tg = P.t0 + K * j;  // global iteration at the start of this time block
      if constexpr (RG != 1) {
        if (role != ROLE_INT && consumer) {  // edge zone with its per-iteration exchange, then help the interior
          double *remote = role == ROLE_TOP ? SL.peer_top[(P.t0 + j + 1) & 1] : SL.peer_bot[(P.t0 + j + 1) & 1];
          // (a watchdog timeout inside raises the abort flag: the consumers still drain this block's
          // interior items, so the producer never blocks, and the grid barrier below ends the run)
          tb_edge<DIM, K, NCW * 32>(g, SL, P, role, ridx, rcount, cur, nxt, remote, tg, &s_edge);
          fence_proxy_async_global();  // our generic-proxy stores before later bulk reads
        }
      }
      if constexpr (RG != 2) {
        if (producer) {
      fence_proxy_async_global();
      if (lane == 0 && c == 0) SL.work_ctr[(j + 1) & 1] = 0u;  // idle since block j-1
      // Guided self-scheduling over (plane block, strip) items, as jb_sweep.
      unsigned int *ctr = SL.work_ctr + (j & 1);
      int64_t item = (role == ROLE_INT && ridx < SL.dyn_first) ? ridx : -1;
      unsigned int claim = 0;
      if (item < 0) {
        if (lane == 0) claim = atomicAdd(ctr, 1u);
        item = SL.dyn_first + (int64_t)__shfl_sync(0xffffffffu, claim, 0);
      }
      while (item < SL.dyn_items) {
        const int64_t blk = item / g.units;
        const int32_t unit = (int32_t)(item - blk * g.units);
        const int64_t a = SL.tb_lo + SL.dyn_table[blk], b = SL.tb_lo + SL.dyn_table[blk + 1] - 1;
        const int64_t r0 = max(a - K, (int64_t)0), r1 = min(b + K, C + 1);
        const bool early = r1 - r0 + 1 <= (int64_t)R.S;
        if (early && lane == 0) claim = atomicAdd(ctr, 1u);
        if (lane == 0) {
          mbar_wait(&qempty[rq.slot], rq.phase ^ 1u);
          TbDesc d;
          d.kind = TB_WORK;
          d.unit = unit;
          d.a = a;
          d.b = b;
          d.pad = 0;
          desc[rq.slot] = d;
          mbar_arrive(&qfull[rq.slot]);
        }
        // level-0 rows r0..r1 of the tile: x window [x0-2, x0+tx+2) of rows y0-2 .. y0+TY+1
        // (3D; stage row i <-> y0-2+i, rows outside the grid are not loaded), one bulk copy
        // per row and lane; 2D with K odd: columns x0-K-1 .. x0+tx+K (stage index 0 <-> x0-K-1;
        // columns left of the row's padding are not loaded: they only feed Dirichlet cells)
        const int ux = unit % g.units_x, uy = unit / g.units_x;
        const int64_t xs_w = K > 2 ? 3 - K + (int64_t)ux * g.tx : 2 + (int64_t)ux * g.tx;
        const int64_t xs = max(xs_w, (int64_t)0);
        const int64_t xe = min(xs_w + (K > 2 ? g.tx + 2 * K + 2 : g.tx + 4), g.pitch);
        const uint32_t bytes = (uint32_t)((xe - xs) * 8);
        const int64_t dso = xs - xs_w;  // stage offset of the first loaded column
        // 3D: stage row i <-> y0-2+i (K = 2) or y0-K+i (odd K: the tile's rows y0-(K-1) ..
        // y0-(K-1)+TY-1 plus one on each side); lane i copies rows i, i+32, ...
        const int64_t ya = DIM == 3 ? (K > 2 ? (int64_t)uy * g.ty + 1 - K : (int64_t)uy * g.ty - 1) : 0;
        const int nrow = DIM == 3 ? g.rh : 1;
        const int64_t yl = max(ya, (int64_t)0), yh = DIM == 3 ? min(ya + nrow - 1, g.ny - 1) : 0;
        const uint32_t nvalid = (uint32_t)(yh - yl + 1);
        if (DIM == 3 && K > 2 && SL.tmap) {  // one TMA box per plane (zero fill outside the grid)
          const void *tm = static_cast<const char *>(SL.tmap) + 128 * ((P.t0 + j) & 1);
          const uint32_t box = (uint32_t)(nrow * g.ws * 8);
          for (int64_t p = r0; p <= r1; ++p) {
            if (lane == 0) {
              mbar_wait(&R.empty[q.slot], q.phase ^ 1u);
              mbar_expect_tx(&R.full[q.slot], box);
              tma_box3(R.stage(q), tm, (int)xs_w, (int)ya, (int)(TB_REV ? r0 + r1 - p : p), &R.full[q.slot]);
            }
            q.advance(R.S);
          }
          __syncwarp();
          rq.advance(JB_RQ);
          if (!early && lane == 0) claim = atomicAdd(ctr, 1u);
          item = SL.dyn_first + (int64_t)__shfl_sync(0xffffffffu, claim, 0);
          continue;
        }
        const bool down = K > 2 && TB_REV;  // the odd-K marches run towards row / plane 0
        for (int64_t i = r0; i <= r1; ++i) {
          const int64_t p = down ? r0 + r1 - i : i;
          if (lane == 0) {
            mbar_wait(&R.empty[q.slot], q.phase ^ 1u);
            mbar_expect_tx(&R.full[q.slot], bytes * nvalid);
          }
          __syncwarp();
          for (int rr = lane; rr < nrow; rr += 32) {
            const int64_t yrow = ya + rr;
            if (DIM == 2 || (yrow >= 0 && yrow <= g.ny - 1))
              bulk_g2s(R.stage(q) + (size_t)rr * g.ws + dso, cur + xs + (DIM == 3 ? yrow * g.pitch : 0) + p * g.plane_elems,
                       bytes, &R.full[q.slot]);
          }
          q.advance(R.S);
        }
        rq.advance(JB_RQ);
        if (!early && lane == 0) claim = atomicAdd(ctr, 1u);
        item = SL.dyn_first + (int64_t)__shfl_sync(0xffffffffu, claim, 0);
      }
      if (lane == 0) {
        mbar_wait(&qempty[rq.slot], rq.phase ^ 1u);
        desc[rq.slot].kind = TB_END;
        mbar_arrive(&qfull[rq.slot]);
      }
      rq.advance(JB_RQ);
        }
      }
      if constexpr (RG != 1) {
        if (consumer) {
      while (true) {
        mbar_wait(&qfull[rq.slot], rq.phase);
        const TbDesc d = desc[rq.slot];
        __syncwarp();
        if (lane == 0) mbar_arrive(&qempty[rq.slot]);
        rq.advance(JB_RQ);
        if (d.kind == TB_END) break;
        if constexpr (DIM == 3 && K > 2)
          tb3k_item<K, TP, RPW, NCW>(g, R, q, d.unit, d.a, d.b, C, nxt, R.stages + (size_t)R.S * R.stage_doubles, warp,
                                     lane);
        else if constexpr (DIM == 3) tb3_item<TP>(g, R, q, d.unit, d.a, d.b, C, nxt, warp, lane);
        else if constexpr (K == 2) tb2_item<TP>(g, R, q, d.unit, d.a, d.b, C, nxt, warp, lane);
        // (stage stride of the 2D odd-K strips: run_tblock sets ws = NCW (64 TP - 2(K-1)) + 2K + 2)
        else tbk_item<K, TP, LAG, NCW * (64 * TP - 2 * (K - 1)) + 2 * K + 2>(g, R, q, d.unit, d.a, d.b, C, nxt, warp,
                                                                              lane);
      }
      fence_proxy_async_global();  // generic-proxy stores before the next block's bulk reads
        }
      }
      // Device-side grid barrier between time blocks.  WS: the two warp-role loops reach
      // it at different instructions, so it is a named barrier over all 16 warps (bar.sync is
      // aligned per warp only; CUDA's __syncthreads would have to be one instruction).
      auto cta_sync = [] {
        // non-.aligned form: lanes of a warp may arrive unconverged after the march's branches
        if constexpr (WS) asm volatile("barrier.sync 3, %0;" ::"n"((NCW + 4) * 32) : "memory");
        else __syncthreads();
      };
      cta_sync();
      if (warp == 0) {
        const bool okb = slab_barrier(SL, P, c, (unsigned long long)(j + 1), (unsigned long long)(tg + K), lane);
        if (lane == 0) s_abort = okb ? 0 : 1;  // (slab_barrier also reports an abort flag)
      }
      cta_sync();
      if (s_abort) return;
    }
    // End of run: the neighbour's last halo has landed before the kernel completes (as jb_sweep).
    if constexpr (RG != 1) {
      if (role != ROLE_INT && warp == 0 && nblocks > 0) {
        if (role == ROLE_TOP) wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(P.t0 + P.iters), P, lane);
        else wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(P.t0 + P.iters), P, lane);
      }
    }
  };
  if constexpr (WS) {
    if (consumer) {
      // 32 (producer warpgroup) + NCW/4 consumer warpgroups x WSR <= 512 registers per lane slot
      // (8 consumer warps: 232, not 240 — measured: the .inc to 240 never completes)
      constexpr int WSR = NCW == 12 ? 160 : NCW == 8 ? 232 : 120;
      asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(WSR) : "memory");
      blocks(std::integral_constant<int, 2>{});
    } else {
      asm volatile("setmaxnreg.dec.sync.aligned.u32 32;" ::: "memory");
      blocks(std::integral_constant<int, 1>{});
    }
  } else {
    blocks(std::integral_constant<int, 0>{});
  }
}

// One CTA per SM (up to 224 registers per thread) or two (96: 2 x 9 warps fit the register file
// only at <= 96 registers, given the 4-warp allocation granularity).  K = iterations per time
// block; TP = pairs per thread along x (2D) or rows per tile (3D).
template <int DIM, int K, int TP, int NCW = JB_NCW, int LAG = 1, int RPW = 1>
__global__ void __launch_bounds__((NCW + 1) * 32, 1) jb_tblock(const __grid_constant__ JbParams P) {
  tb_body<NCW, DIM, K, TP, LAG, RPW>(P);
}
// warp-specialised register split (tb_body WS = 1): NCW consumer warps + one producer warpgroup
template <int DIM, int K, int TP, int NCW, int LAG = 1, int RPW = 1>
__global__ void __launch_bounds__(NCW * 32 + 128, 1) jb_tblock_ws(const __grid_constant__ JbParams P) {
  tb_body<NCW, DIM, K, TP, LAG, RPW, 1>(P);
}
template <int TP>
__global__ void __maxnreg__(96) jb_tblock2d_x2(const __grid_constant__ JbParams P) {
  tb_body<JB_NCW, 2, 2, TP, 1, 1>(P);
}

constexpr int TB_TY = 4;  // 3D tile rows (level-1 rows TY+2 carried per plane in registers)

// Kernel for (dim, K, pairs per thread, wavefront lag, CTAs per SM) and its consumer warp count;
// nullptr if not instantiated.  Odd K holds (LAG+2)(K-1) level rows per lane: beyond ~168
// registers, i.e. 7 consumer warps (256 threads: up to 255 registers).
#define JB_TB(...) reinterpret_cast<const void *>(&__VA_ARGS__)
const void *tblock_fn_plain(int dim, int k, int ppt, int lag, int per_sm, int ws, int *ncw) {
  *ncw = JB_NCW;
  if (ws) {  // warp-specialised register split, 12 consumer warps: 2D K = 5, one pair per lane;
             // 3D K = 3, one pair per lane, 2 rows per warp (tiles of 24 rows: 20 output rows)
    *ncw = 12;
    if (per_sm != 1) return nullptr;
    if (dim == 2 && k == 5 && ppt == 1 && lag == 1) return JB_TB(jb_tblock_ws<2, 5, 1, 12, 1>);
    if (dim == 3 && k == 3 && ppt == 1 && lag == 2) return JB_TB(jb_tblock_ws<3, 3, 1, 12, 1, 2>);
    return nullptr;
  }
#ifndef JB_TB_ONLY_WS  // (development builds: only the warp-specialised kernels)
  if (dim == 3) {
    if (k == 2) return JB_TB(jb_tblock<3, 2, TB_TY>);
    // odd K: (K, PPT, RPW = `lag`) -> NCW consumer warps x RPW rows per tile
    if (k != 3) return nullptr;
    *ncw = 11;
    if (ppt == 1 && lag == 2) return JB_TB(jb_tblock<3, 3, 1, 11, 1, 2>);
    *ncw = 7;
    if (ppt == 1 && lag == 3) return JB_TB(jb_tblock<3, 3, 1, 7, 1, 3>);
    if (ppt == 2 && lag == 2) return JB_TB(jb_tblock<3, 3, 2, 7, 1, 2>);
    return nullptr;
  }
  if (k == 2) {
    if (per_sm >= 2) return ppt >= 4 ? JB_TB(jb_tblock2d_x2<4>) : ppt == 2 ? JB_TB(jb_tblock2d_x2<2>) : JB_TB(jb_tblock2d_x2<1>);
    return ppt >= 4 ? JB_TB(jb_tblock<2, 2, 4>) : ppt == 2 ? JB_TB(jb_tblock<2, 2, 2>) : JB_TB(jb_tblock<2, 2, 1>);
  }
  if (per_sm >= 2) return nullptr;
  *ncw = 11;
  if (k == 5 && ppt == 1 && lag == 1) return JB_TB(jb_tblock<2, 5, 1, 11, 1>);
  *ncw = 7;
  if (lag == 2) {
    if (k == 3 && ppt == 2) return JB_TB(jb_tblock<2, 3, 2, 7, 2>);
    if (k == 5 && ppt == 1) return JB_TB(jb_tblock<2, 5, 1, 7, 2>);
    if (k == 5 && ppt == 2) return JB_TB(jb_tblock<2, 5, 2, 7, 2>);
    return nullptr;
  }
  if (k == 3 && ppt == 2) return JB_TB(jb_tblock<2, 3, 2, 7>);
  if (k == 3 && ppt == 4) return JB_TB(jb_tblock<2, 3, 4, 7>);
  if (k == 5 && ppt == 2) return JB_TB(jb_tblock<2, 5, 2, 7>);
#endif
  return nullptr;
}
#undef JB_TB
// ... and its block size: the consumer warps + one producer warp (WS: + a producer warpgroup).
const void *tblock_fn(int dim, int k, int ppt, int lag, int per_sm, int ws, int *ncw, int *threads) {
  const void *fn = tblock_fn_plain(dim, k, ppt, lag, per_sm, ws, ncw);
  *threads = (*ncw + (ws ? 4 : 1)) * 32;
  return fn;
}

}  // namespace

namespace jbk {

int tblock_ty() { return TB_TY; }
// consumer warps of the kernel for (dim, k, ppt) with one CTA per SM; 0 if not instantiated
int tblock_ncw(int dim, int k, int ppt, int lag, int per_sm, int ws) {
  int ncw = 0, threads = 0;
  return tblock_fn(dim, k, ppt, lag, per_sm, ws, &ncw, &threads) ? ncw : 0;
}

// Dynamic shared memory of the temporally blocked kernel: header + ring stages (+ the 3D
// odd-K row exchange).
size_t tblock_smem(const JbGeom &g) {
  const size_t hdr = (size_t)2 * g.stages * 8 + (size_t)2 * JB_RQ * 8 + (size_t)JB_RQ * sizeof(TbDesc);
  return (hdr + 127) / 128 * 128 + (size_t)g.stages * g.stage_doubles * 8 + (size_t)g.xch_doubles * 8;
}

cudaError_t prepare_tblock(const JbGeom &g, int k, int ppt, int lag, int per_sm, int ws, size_t smem,
                           int *blocks_per_sm) {
  int ncw = 0, threads = 0;
  const void *fn = tblock_fn(g.dim, k, ppt, lag, per_sm, ws, &ncw, &threads);
  if (!fn) return cudaErrorInvalidValue;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, fn, threads, smem);
}

cudaError_t launch_tblock(const JbParams &p, int k, int ppt, int lag, int per_sm, int ws, int grid, size_t smem,
                          cudaStream_t st) {
  void *args[] = {const_cast<JbParams *>(&p)};
  int ncw = 0, threads = 0;
  const void *fn = tblock_fn(p.g.dim, k, ppt, lag, per_sm, ws, &ncw, &threads);
  if (!fn) return cudaErrorInvalidValue;
  return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(threads), args, smem, st);
}

}  // namespace jbk
