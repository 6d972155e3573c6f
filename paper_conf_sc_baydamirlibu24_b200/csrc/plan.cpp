// plan.cpp — host-only planning logic of the CPU-Free Jacobi library: slab decomposition
// ("divided equally among GPUs"), the HBM layout and tile shape, and the thread-block
// split between boundary and interior blocks (§4.1.2).  No CUDA calls here, so the
// logic is testable on a CPU-only box through the C ABI (tests/test_host_logic.py).
#include <algorithm>
#include <cmath>
#include <cstring>

#include "jacobi_internal.h"
#include "../../include/jacobi.h"

namespace jbplan {

int64_t pow2ceil(int64_t v) {
  int64_t p = 1;
  while (p < v) p <<= 1;
  return p;
}

static int64_t round_up(int64_t v, int64_t m) { return (v + m - 1) / m * m; }

void decompose(int64_t n_out, int nslabs, int slab, int64_t *start, int64_t *chunk) {
  const int64_t inner = n_out - 2;
  const int64_t q = inner / nslabs, r = inner % nslabs;
  *chunk = q + (slab < r ? 1 : 0);
  *start = 1 + (int64_t)slab * q + std::min<int64_t>(slab, r);
}

size_t smem_bytes(const JbGeom &g) {
  size_t bar = (size_t)2 * g.stages * 8 + (size_t)2 * JB_RQ * 8 + (size_t)JB_RQ * 32;
  bar = (bar + 127) / 128 * 128;
  return bar + (size_t)g.stages * g.stage_doubles * 8;
}

int geometry(int64_t nx, int64_t ny, int64_t nz, int dim, int tile_x, int tile_y, int smem,
             int stages_req, JbGeom *g) {
  std::memset(g, 0, sizeof(*g));
  g->nx = nx; g->ny = ny; g->nz = nz; g->dim = dim;
  g->pitch = round_up(nx + 3, 4);
  g->plane_elems = dim == 2 ? g->pitch : ny * g->pitch;
  const int64_t ix = nx - 2;
  // 2D: up to 4 cell pairs per consumer thread (tx <= 8*JB_NC); 3D: one x pair per thread and
  // row group (tx <= 2*JB_NC).
  const int64_t tx_max = dim == 2 ? 8 * JB_NC : 2 * JB_NC;
  int64_t tx = tile_x > 0 ? pow2ceil(tile_x) : std::min<int64_t>(tx_max, pow2ceil(ix));
  tx = std::max<int64_t>(tx, 8);
  if (tx > tx_max) return -1;
  g->tx = (int)tx;
  int sh = 0;
  while ((int64_t(1) << sh) < tx / 2) ++sh;
  g->txp_shift = sh;
  g->ws = (int)tx + 4;
  g->units_x = (int)((ix + tx - 1) / tx);
  if (dim == 2) {
    g->ty = 1; g->rh = 1; g->units_y = 1;
  } else {
    int ty = tile_y > 0 ? tile_y : 8;
    ty = (int)std::min<int64_t>(ty, ny - 2);
    ty = std::max(ty, 1);
    if (ty + 2 > 32) return -1;  // producer warp issues one row per lane
    g->ty = ty; g->rh = ty + 2;
    g->units_y = (int)((ny - 2 + ty - 1) / ty);
  }
  g->units = g->units_x * g->units_y;
  g->stage_doubles = g->rh * g->ws;
  const size_t stage_b = (size_t)g->stage_doubles * 8;
  int s = (int)((smem - 512) / (stage_b + 16));
  s = std::min(s, JB_MAX_STAGES);
  if (stages_req > 0) s = std::min(s, stages_req);
  if (s < 4) return -1;  // need p-1, p, p+1 resident + one in flight
  g->stages = s;
  if (smem_bytes(*g) > (size_t)smem) return -1;
  return 0;
}

void tb_split(int ctas, int64_t inner, int has_top, int has_bot, int64_t units, int override_ps,
              int *n_top, int *n_bot, int *n_int) {
  const int sides = (has_top ? 1 : 0) + (has_bot ? 1 : 0);
  if (sides == 0) { *n_top = *n_bot = 0; *n_int = ctas; return; }
  // Reconstructed P:400: boundary_TB = TB_total * boundary_size / (inner_size + 2*boundary_size).
  // A boundary plane costs ~2.5 interior planes (it loads p-1, p, p+1 and stores twice).
  const double wb = 2.5;
  int ps;
  if (override_ps > 0) {
    ps = override_ps;
  } else {
    ps = (int)std::ceil((double)ctas * wb / ((double)std::max<int64_t>(inner, 0) + sides * wb));
  }
  ps = std::max(ps, 1);
  ps = (int)std::min<int64_t>(ps, units);
  if (inner > 0) ps = std::min(ps, std::max(1, (ctas - 1) / sides));
  else if (override_ps <= 0) ps = (int)std::min<int64_t>(std::max(1, ctas / sides), units);
  ps = std::min(ps, std::max(1, ctas / sides));
  *n_top = has_top ? ps : 0;
  *n_bot = has_bot ? ps : 0;
  *n_int = ctas - *n_top - *n_bot;
  if (inner <= 0) *n_int = std::max(*n_int, 0);
}

// Auto policies, functions of the global problem only, so that every rank /
// process takes the same decision: interior cells of the grid per CTA of the whole job.
int64_t cells_per_cta(int64_t nx, int64_t ny, int64_t nz, int dim, int64_t job_ctas) {
  const int64_t cells = (nx - 2) * (dim == 3 ? (ny - 2) * (nz - 2) : (ny - 2));
  return cells / std::max<int64_t>(1, job_ctas);
}
bool schedule_dynamic_auto(int64_t cpc) { return cpc >= JB_DYN_MIN_CELLS; }
bool tblock_neighbours_auto(int dim, int64_t cpc, int min_slab_ctas) {
  if (dim == 3) return cpc >= JB_TB3_NB_MIN_CELLS && min_slab_ctas >= 64;
  return cpc >= JB_TB2_NB_MIN_CELLS;
}

int lockstep_k(int units, int n_int, int64_t inner) {
  if (units <= 0 || n_int < units || inner <= 0) return 0;
  int64_t k = n_int / units;
  k = std::min<int64_t>(k, inner);
  return (int)std::max<int64_t>(k, 1);
}

int64_t dyn_blocks(int64_t npl, int units, int n, int min_blk, int32_t *table) {
  // Guided self-scheduling: each block hands every unit rem/(f*n) of the remaining work.  When a
  // CTA's share is small (< 4 minimum blocks) use f = 1 so the first round covers everything
  // (latency-bound grids); otherwise f = 2 (half the work in the first round, shrinking tail).
  const int64_t f = (npl * units < 4 * (int64_t)min_blk * n) ? 1 : 2;
  int64_t rem = npl, nb = 0;
  while (rem > 0) {
    if (table) table[nb] = (int32_t)(npl - rem);
    int64_t s = (rem * units + f * (int64_t)n - 1) / (f * (int64_t)n);
    s = std::max<int64_t>(s, min_blk);
    s = std::min(s, rem);
    rem -= s;
    ++nb;
  }
  if (table) table[nb] = (int32_t)npl;
  return nb;
}

void even_split(int64_t n, int k, int i, int64_t *start, int64_t *len) {
  const int64_t q = n / k, r = n % k;
  *len = q + (i < r ? 1 : 0);
  *start = (int64_t)i * q + std::min<int64_t>(i, r);
}

int resident_tiling(int64_t nx, int64_t ny, int dim, int64_t chunk, int count, int smem, int *nbz_out,
                    int *nby_out, int *cpp_out, size_t *smem_used) {
  const int64_t rs = round_up(nx + 1, 2);
  const int64_t ppr = (nx - 1) / 2;  // cell pairs per row covering x = 1 .. nx-2
  const int64_t rows_y = dim == 3 ? ny - 2 : 1;
  double best = -1;
  for (int nbz = 1; nbz <= std::min<int64_t>(chunk, count); ++nbz) {
    int nby = dim == 3 ? (int)std::min<int64_t>({(int64_t)(count / nbz), rows_y, (int64_t)JB_MAXK}) : 1;
    if (nby < 1) continue;
    const int64_t zb = (chunk + nbz - 1) / nbz, yb = (rows_y + nby - 1) / nby;
    const int64_t rows = (zb + 2) * (dim == 3 ? yb + 2 : 1);
    const size_t sm = (size_t)rows * rs * 8;
    if (sm > (size_t)smem) continue;
    const int64_t pairs = zb * yb * ppr;
    const int64_t cpp = (pairs + JB_RNT - 1) / JB_RNT;
    if (cpp > JB_RCPP_MAX) continue;
    // cost: cells per block (compute + write-back) plus its halo ring rows (L2 refresh)
    const double cost = (double)zb * yb * (nx - 2) + 2.0 * (zb + (dim == 3 ? yb : 0)) * nx;
    if (best < 0 || cost < best) {
      best = cost;
      *nbz_out = nbz;
      *nby_out = nby;
      int c = 1;
      while (c < cpp) c <<= 1;
      *cpp_out = c;
      *smem_used = sm;
    }
  }
  return best < 0 ? -1 : 0;
}

int tallest_ty(int64_t ny, int smem, int ws) {
  int best = 1;
  for (int ty = 1; ty <= 12; ++ty) {
    if (ty > std::max<int64_t>(ny - 2, 1)) break;
    const size_t stage_b = (size_t)(ty + 2) * ws * 8;
    if ((size_t)(smem - 512) / (stage_b + 16) < 5) break;
    best = ty;
  }
  return best;
}

int choose_ty(int64_t ny, int units_x, int n_int, int smem, int ws) {
  // Largest-utilisation ty in [4, 12] whose stage still leaves a >= 5-deep ring.
  int best = 8;
  double best_score = -1;
  for (int ty = 4; ty <= 12; ++ty) {
    if (ty > ny - 2) break;
    const size_t stage_b = (size_t)(ty + 2) * ws * 8;
    if ((size_t)(smem - 256) / (stage_b + 16) < 5) break;
    const int64_t uy = (ny - 2 + ty - 1) / ty;
    const int64_t u = uy * units_x;
    double util;
    if (u > n_int) {
      util = 0.5;  // not lockstep-able; linear fallback
    } else {
      const int64_t k = n_int / u;
      util = (double)(u * k) / n_int;
    }
    // Prefer fewer halo rows when utilisation ties (reads (ty+2)/ty rows per row from L2).
    const double score = util - 0.02 * (2.0 / ty);
    if (score > best_score + 1e-9) { best_score = score; best = ty; }
  }
  return best;
}

}  // namespace jbplan

extern "C" {

int jacobi_decompose(int64_t n_out, int nslabs, int slab, int64_t *start, int64_t *chunk) {
  if (n_out < 3 || nslabs < 1 || slab < 0 || slab >= nslabs || !start || !chunk) return JACOBI_EINVAL;
  jbplan::decompose(n_out, nslabs, slab, start, chunk);
  return JACOBI_OK;
}

int jacobi_tb_split(int ctas, int64_t chunk, int has_top, int has_bottom, int64_t units,
                    int override_per_side, int *out3) {
  if (!out3 || ctas < 1 || chunk < 1 || units < 1) return JACOBI_EINVAL;
  const int64_t lo = has_top ? 2 : 1, hi = has_bottom ? chunk - 1 : chunk;
  const int64_t inner = hi - lo + 1;
  const int sides = (has_top ? 1 : 0) + (has_bottom ? 1 : 0);
  if (ctas < sides + (inner > 0 ? 1 : 0)) return JACOBI_EINVAL;
  jbplan::tb_split(ctas, inner, has_top, has_bottom, units, override_per_side, &out3[0], &out3[1], &out3[2]);
  return JACOBI_OK;
}

int jacobi_geometry(int64_t nx, int64_t ny, int64_t nz, int stencil, int tile_x, int tile_y,
                    int64_t *out8) {
  if (!out8 || nx < 3 || ny < 3) return JACOBI_EINVAL;
  if (!((stencil == 5 && nz == 1) || (stencil == 7 && nz >= 3))) return JACOBI_EINVAL;
  JbGeom g;
  if (jbplan::geometry(nx, ny, nz, stencil == 5 ? 2 : 3, tile_x, tile_y, JB_SMEM_DEFAULT, 0, &g))
    return JACOBI_EINVAL;
  out8[0] = g.pitch; out8[1] = g.plane_elems; out8[2] = g.tx; out8[3] = g.ty;
  out8[4] = g.units_x; out8[5] = g.units_y; out8[6] = g.rh; out8[7] = g.ws;
  return JACOBI_OK;
}

int jacobi_auto_policy(int64_t nx, int64_t ny, int64_t nz, int stencil, int nslabs, int virtual_slabs, int sms,
                       int64_t *out4) {
  if (!out4 || nx < 3 || ny < 3 || nslabs < 1 || sms < 1) return JACOBI_EINVAL;
  if (!((stencil == 5 && nz == 1) || (stencil == 7 && nz >= 3))) return JACOBI_EINVAL;
  const int dim = stencil == 5 ? 2 : 3;
  const int64_t job_ctas = virtual_slabs ? sms : (int64_t)sms * nslabs;
  const int min_slab_ctas = virtual_slabs ? sms / nslabs : sms;
  const int64_t cpc = jbplan::cells_per_cta(nx, ny, nz, dim, job_ctas);
  out4[0] = cpc;
  out4[1] = jbplan::schedule_dynamic_auto(cpc) ? 1 : 0;
  out4[2] = nslabs == 1 ? 1 : (jbplan::tblock_neighbours_auto(dim, cpc, min_slab_ctas) ? 1 : 0);
  out4[3] = min_slab_ctas;
  return JACOBI_OK;
}

const char *jacobi_strerror(int code) {
  switch (code) {
    case JACOBI_OK: return "ok";
    case JACOBI_EINVAL: return "invalid argument";
    case JACOBI_ENODEV: return "not enough CUDA devices";
    case JACOBI_ENOPEER: return "peer access between neighbouring GPUs unavailable";
    case JACOBI_ENOCOOP: return "cooperative launch unavailable or grid not co-resident";
    case JACOBI_ENOMEM: return "out of memory";
    case JACOBI_ECUDA: return "CUDA runtime error";
    case JACOBI_ETIMEOUT: return "device watchdog timeout: a neighbour never signalled";
    case JACOBI_ENCCL: return "NCCL unavailable or failed";
    case JACOBI_ESTATE: return "invalid state for this call";
    default: return "unknown error";
  }
}

int jacobi_version(void) { return 100; }

}  // extern "C"
