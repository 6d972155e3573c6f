// tblock.cu — temporally blocked CPU-Free sweep: K = 2 Jacobi iterations per pass
// over HBM, for a slab without neighbours (P = 1, both outer halos are the Dirichlet planes).
//
// The method is unchanged — every cell is updated every iteration with the oracle's fp64 order
// (-fmad=false), each iteration reads only the previous time step, Dirichlet cells are
// never written — only the schedule of the updates differs: a work item (plane block
// [a, b] x x-strip) streams the time-t planes a-2 .. b+2 of its strip from HBM through the same
// TMA bulk-copy ring as jb_sweep, computes time t+1 for planes a-1 .. b+1 in registers (x
// neighbours by warp shuffles), and from those time t+2 for planes a .. b, columns
// x0 .. x0+tx-1, which it stores into the other buffer.  The intermediate time level never
// touches HBM, so the algorithmic traffic per cell-update is 16 B / K = 8 B instead of 16 B
// (overlapped tiling: the t+1 values of the 2 extra planes of each item and of one extra column
// at each end of each warp's segment are recomputed, < 2 % extra arithmetic at C2).
// The persistent structure of the paper is kept: one cooperative launch for the whole run, a
// device-side grid barrier between time blocks, no host involvement.
//
// Buffers: time block j of a launch reads buf[(t0 + j) & 1] and writes buf[(t0 + j + 1) & 1]
// (out of place — neighbouring strips still read the time-t columns of this strip); the host
// runs an even number of blocks, so the result lands in buf[(t0 + 2 nb) & 1] as in every other
// path (R10).
#include <type_traits>

#include "device_common.cuh"

namespace {

constexpr int TB_K = 2;  // iterations per time block

enum { TB_WORK = 0, TB_END = 1 };
struct TbDesc {
  int32_t kind;
  int32_t unit;
  int64_t a, b;  // output planes a..b of this item (time t+2)
  int64_t pad;
};

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

// Edge zone of a slab side with a neighbour (time block t -> t+2), computed by that side's
// boundary CTAs with the whole CTA, so the halo exchange stays per iteration:
//   A: wait for the neighbour's time-t halo plane; level 1 (t+1) of the three planes next to the
//      halo (top: 1..3, bottom: C-2..C) over the strip window [x0-1, x0+tx] into the slab's edge
//      scratch E, the outermost one also into the neighbour's intermediate slot; signal t+1.
//   B: wait for the neighbour's level-1 plane (our E slot); level 2 (t+2) of the two outermost
//      planes (top: 1, 2; bottom: C-1, C) into the next buffer, the outermost one also into the
//      neighbour's halo; signal t+2.
// E_top = buf[0] + (C+2) pe: [0] = neighbour's level-1 plane 0, [k] = level-1 plane k (k = 1..3);
// E_bot = buf[1] + (C+2) pe: [k] = level-1 plane C-2+k (k = 0..2), [3] = neighbour's plane C+1.
// Loads bypass L1 (ld.cg): these planes are rewritten by other CTAs / the neighbour GPU.
template <int DIM>
__device__ bool tb_edge(const JbGeom &g, const JbSlab &SL, const JbParams &P, int role, int ridx, int rcount,
                        const double *cur, double *nxt, double *remote, int64_t tg, int *s_flag) {
  const bool top = role == ROLE_TOP;
  const int64_t C = SL.chunk, pe = g.plane_elems, nx = g.nx, ny = g.ny, pitch = g.pitch;
  double *E = (top ? SL.buf[0] : SL.buf[1]) + (C + 2) * pe + 3;
  double *mid = (top ? SL.mid_top_out : SL.mid_bot_out) + 3;
  const unsigned long long *fin = top ? SL.flag_in_top : SL.flag_in_bot;
  const int kin = top ? SL.k_in_top : SL.k_in_bot;
  unsigned long long *fout = (top ? SL.flag_out_top : SL.flag_out_bot) + ridx;
  const int ub = (int)((int64_t)g.units * ridx / rcount), ue = (int)((int64_t)g.units * (ridx + 1) / rcount);
  const int tid = threadIdx.x, nt = blockDim.x;
  const bool drop = (P.flags & JACOBI_FLAG_DROP_SIGNAL) && SL.slab_id == 0;
  auto wait = [&](unsigned long long target) {
    if (tid < 32) {
      const bool ok = wait_slots(fin, kin, target, P, tid);
      if (tid == 0) *s_flag = ok ? 0 : 1;
    }
    __syncthreads();
    return *s_flag == 0;
  };
  // one stencil update of the field F (ld.cg) at element offset e = y*pitch + x of plane p
  auto upd = [&](const double *F, int64_t e) {
    const double *A = F + e;
    if (DIM == 2) return 0.25 * (((__ldcg(A + 1) + __ldcg(A - 1)) + __ldcg(A + pe)) + __ldcg(A - pe));
    return kC6 * (((((__ldcg(A + 1) + __ldcg(A - 1)) + __ldcg(A + pitch)) + __ldcg(A - pitch)) + __ldcg(A + pe)) +
                  __ldcg(A - pe));
  };
  // ---- A: level 1 of 3 planes over each tile window [y0-1, y0+ty] x [x0-1, x0+tx] (clamped)
  if (!wait((unsigned long long)tg)) return false;
  const int64_t pa = top ? 1 : C - 2;  // plane of E index e0
  const int e0 = top ? 1 : 0;
  const int64_t pout = top ? 1 : C;    // the plane the neighbour needs
  for (int u = ub; u < ue; ++u) {
    const int ux = u % g.units_x, uy = u / g.units_x;
    const int64_t x0 = 1 + (int64_t)ux * g.tx;
    const int64_t xa = max(x0 - 1, (int64_t)0), xb = min(x0 + g.tx, nx - 1), w = xb - xa + 1;
    int64_t ya = 0, h = 1;
    if (DIM == 3) {
      const int64_t y0 = 1 + (int64_t)uy * g.ty;
      ya = max(y0 - 1, (int64_t)0);
      h = min(y0 + g.ty, ny - 1) - ya + 1;
    }
    for (int64_t i = tid; i < 3 * h * w; i += nt) {
      const int64_t k = i / (h * w), r = i - k * h * w, yy = r / w;
      const int64_t x = xa + (r - yy * w), y = ya + yy, p = pa + k;
      const int64_t e = (DIM == 3 ? y * pitch : 0) + x;
      const bool in = x >= 1 && x <= nx - 2 && (DIM == 2 || (y >= 1 && y <= ny - 2));
      const double v = in ? upd(cur + p * pe + 3, e) : __ldcg(cur + p * pe + 3 + e);
      E[(e0 + k) * pe + e] = v;
      if (p == pout) mid[e] = v;
    }
  }
  __syncthreads();  // every thread's stores (local E, neighbour's slot) precede the release below
  if (tid == 0 && !drop) st_release_sys(fout, (unsigned long long)(tg + 1));
  // ---- B: level 2 of the 2 outermost planes over each tile's interior cells
  if (!wait((unsigned long long)(tg + 1))) return false;
  const int64_t pb = top ? 1 : C - 1;  // level-2 planes pb, pb+1 <-> E indices 1, 2
  for (int u = ub; u < ue; ++u) {
    const int ux = u % g.units_x, uy = u / g.units_x;
    const int64_t x0 = 1 + (int64_t)ux * g.tx;
    const int64_t w = min((int64_t)g.tx, nx - 1 - x0);
    int64_t y0 = 0, h = 1;
    if (DIM == 3) {
      y0 = 1 + (int64_t)uy * g.ty;
      h = min((int64_t)g.ty, ny - 1 - y0);
    }
    for (int64_t i = tid; i < 2 * h * w; i += nt) {
      const int64_t k = i / (h * w), r = i - k * h * w, yy = r / w;
      const int64_t x = x0 + (r - yy * w), p = pb + k;
      const int64_t e = (DIM == 3 ? (y0 + yy) * pitch : 0) + x;
      const double v = upd(E + (1 + k) * pe, e);
      nxt[p * pe + 3 + e] = v;
      if (p == pout) remote[3 + e] = v;
    }
  }
  __syncthreads();
  if (tid == 0 && !drop) st_release_sys(fout, (unsigned long long)(tg + 2));
  return true;
}

template <int NCW, int DIM, int TP>
__device__ __forceinline__ void tb_body(const JbParams &P) {
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
  if (threadIdx.x == 0) {
    for (uint32_t i = 0; i < R.S; ++i) {
      mbar_init(&R.full[i], 1);
      mbar_init(&R.empty[i], NCW);
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
  const int64_t nblocks = P.iters / TB_K;
  RingPos q = {0u, 0u}, rq = {0u, 0u};
  for (int64_t j = 0; j < nblocks; ++j) {
    const double *cur = SL.buf[(P.t0 + j) & 1];
    double *nxt = SL.buf[(P.t0 + j + 1) & 1];
    const int64_t tg = P.t0 + TB_K * j;  // global iteration at the start of this time block
    if (role != ROLE_INT) {  // edge zone with its per-iteration exchange, then help the interior
      double *remote = role == ROLE_TOP ? SL.peer_top[(P.t0 + j + 1) & 1] : SL.peer_bot[(P.t0 + j + 1) & 1];
      if (!tb_edge<DIM>(g, SL, P, role, ridx, rcount, cur, nxt, remote, tg, &s_edge)) return;
      fence_proxy_async_global();  // our generic-proxy stores before later bulk reads
    }
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
        const int64_t r0 = max(a - 2, (int64_t)0), r1 = min(b + 2, C + 1);
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
        // per row and lane
        const int ux = unit % g.units_x, uy = unit / g.units_x;
        const int64_t xs = 2 + (int64_t)ux * g.tx;
        const int64_t xe = min(xs + g.tx + 4, g.pitch);
        const uint32_t bytes = (uint32_t)((xe - xs) * 8);
        const int64_t ya = DIM == 3 ? (int64_t)uy * g.ty - 1 : 0;  // = y0 - 2
        const int nrow = DIM == 3 ? g.rh : 1;
        const int64_t yl = max(ya, (int64_t)0), yh = DIM == 3 ? min(ya + nrow - 1, g.ny - 1) : 0;
        const uint32_t nvalid = (uint32_t)(yh - yl + 1);
        const int64_t yrow = ya + lane;
        const bool mine = lane < nrow && (DIM == 2 || (yrow >= 0 && yrow <= g.ny - 1));
        const double *src = cur + xs + (DIM == 3 ? yrow * g.pitch : 0);
        for (int64_t p = r0; p <= r1; ++p) {
          if (lane == 0) {
            mbar_wait(&R.empty[q.slot], q.phase ^ 1u);
            mbar_expect_tx(&R.full[q.slot], bytes * nvalid);
          }
          __syncwarp();
          if (mine) bulk_g2s(R.stage(q) + (size_t)lane * g.ws, src + p * g.plane_elems, bytes, &R.full[q.slot]);
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
    } else {
      while (true) {
        mbar_wait(&qfull[rq.slot], rq.phase);
        const TbDesc d = desc[rq.slot];
        __syncwarp();
        if (lane == 0) mbar_arrive(&qempty[rq.slot]);
        rq.advance(JB_RQ);
        if (d.kind == TB_END) break;
        if (DIM == 2) tb2_item<TP>(g, R, q, d.unit, d.a, d.b, C, nxt, warp, lane);
        else tb3_item<TP>(g, R, q, d.unit, d.a, d.b, C, nxt, warp, lane);
      }
      fence_proxy_async_global();  // generic-proxy stores before the next block's bulk reads
    }
    // Device-side grid barrier between time blocks.
    __syncthreads();
    if (threadIdx.x == 0) {
      red_release_gpu_add(SL.barrier, 1ull);
      const bool okb = wait_geq<false>(SL.barrier, (unsigned long long)SL.cta_count * (j + 1), P);
      s_abort = (!okb || *(volatile int *)(P.status + 1)) ? 1 : 0;
    }
    __syncthreads();
    if (s_abort) return;
  }
  // End of run: the neighbour's last halo has landed before the kernel completes (as jb_sweep).
  if (role != ROLE_INT && warp == 0 && nblocks > 0) {
    if (role == ROLE_TOP) wait_slots(SL.flag_in_top, SL.k_in_top, (unsigned long long)(P.t0 + P.iters), P, lane);
    else wait_slots(SL.flag_in_bot, SL.k_in_bot, (unsigned long long)(P.t0 + P.iters), P, lane);
  }
}

// One CTA per SM (up to 224 registers per thread) or two (96: 2 x 9 warps fit the register file
// only at <= 96 registers, given the 4-warp allocation granularity).  TP = pairs per thread
// along x (2D) or rows per tile (3D).
template <int DIM, int TP>
__global__ void __launch_bounds__(JB_NC + 32, 1) jb_tblock(const __grid_constant__ JbParams P) {
  tb_body<JB_NCW, DIM, TP>(P);
}
template <int TP>
__global__ void __maxnreg__(96) jb_tblock2d_x2(const __grid_constant__ JbParams P) {
  tb_body<JB_NCW, 2, TP>(P);
}

constexpr int TB_TY = 4;  // 3D tile rows (level-1 rows TY+2 carried per plane in registers)

const void *tblock_fn(int dim, int ppt, int per_sm) {
#define JB_TB(K) reinterpret_cast<const void *>(&K)
  if (dim == 3) return JB_TB((jb_tblock<3, TB_TY>));
  if (per_sm >= 2) return ppt >= 4 ? JB_TB(jb_tblock2d_x2<4>) : ppt == 2 ? JB_TB(jb_tblock2d_x2<2>) : JB_TB(jb_tblock2d_x2<1>);
  return ppt >= 4 ? JB_TB((jb_tblock<2, 4>)) : ppt == 2 ? JB_TB((jb_tblock<2, 2>)) : JB_TB((jb_tblock<2, 1>));
#undef JB_TB
}

}  // namespace

namespace jbk {

int tblock_k() { return TB_K; }
int tblock_ty() { return TB_TY; }
int tblock_threads() { return JB_NC + 32; }

// Dynamic shared memory of the temporally blocked kernel: header + ring stages.
size_t tblock_smem(const JbGeom &g) {
  const size_t hdr = (size_t)2 * g.stages * 8 + (size_t)2 * JB_RQ * 8 + (size_t)JB_RQ * sizeof(TbDesc);
  return (hdr + 127) / 128 * 128 + (size_t)g.stages * g.stage_doubles * 8;
}

cudaError_t prepare_tblock(const JbGeom &g, int per_sm, size_t smem, int *blocks_per_sm) {
  const void *fn = tblock_fn(g.dim, g.tx / (2 * JB_NC), per_sm);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, fn, JB_NC + 32, smem);
}

cudaError_t launch_tblock(const JbParams &p, int per_sm, int grid, size_t smem, cudaStream_t st) {
  void *args[] = {const_cast<JbParams *>(&p)};
  return cudaLaunchCooperativeKernel(tblock_fn(p.g.dim, p.g.tx / (2 * JB_NC), per_sm), dim3(grid), dim3(JB_NC + 32), args, smem,
                                     st);
}

}  // namespace jbk
