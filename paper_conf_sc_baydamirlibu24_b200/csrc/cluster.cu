// cluster.cu — the CPU-Free kernel for 2D grids that fit in the shared memory of ONE thread-block
// cluster: the latency-bound small configurations (C1, 256^2).
//
// The paper's persistent kernel ends every iteration with a device-wide grid barrier (P:372,
// Listing 4.1); for a grid of 65 K cells that barrier (~1.7 us over 148 CTAs) costs
// more than the sweep.  On sm_100a up to 16 CTAs of a cluster are co-scheduled on one GPC and can
// read each other's shared memory (DSMEM), and the cluster barrier is a hardware barrier.  So the
// whole grid lives on chip for the run: CTA c of an NC-CTA cluster keeps its band of rows (both
// time levels) in its shared memory; per iteration it sweeps its rows from one level into the
// other (oracle order, no FMA contraction: bit-identical to the other kernels), reading the rows
// just outside its band straight from the neighbour CTAs' shared memory (ld.shared::cluster), and
// joins the cluster barrier (barrier.cluster.arrive.release / wait.acquire) — the device-side
// iteration barrier of P:372 at cluster scope.  The final level is written back to the global
// buffer buf[(t0 + iters) & 1] at the end, so runs of every kernel mix.  One slab (P = 1) only.
#include "device_common.cuh"

namespace {

#ifndef JB_CNT_
#define JB_CNT_ 512
#endif
constexpr int JB_CNT = JB_CNT_;  // threads per CTA

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// 32-bit shared::cluster address of the same shared-memory location in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t map_rank(const void *p, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(sptr(p)), "r"(rank));
  return r;
}
__device__ __forceinline__ double2 ld_dsmem2(uint32_t a) {
  double2 v;
  asm volatile("ld.shared::cluster.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void cluster_barrier() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Shared memory of CTA c: two buffers of (n_max + 2) rows x pitch doubles (the global row layout:
// cell x at column x + 3, so cell pairs (x, x+1), x odd, are 16-byte aligned); local row r <->
// slab plane a - 1 + r, rows 0 and n + 1 the halo rows.
__global__ void __launch_bounds__(JB_CNT, 1) jb_cluster2d(const __grid_constant__ JbParams P) {
  extern __shared__ __align__(16) double sm[];
  const JbGeom &g = P.g;
  const JbSlab &SL = P.s[0];
  const int NC = (int)gridDim.x;  // the grid is one cluster
  const int c = (int)cluster_rank();
  const int tid = threadIdx.x;
  int64_t a64, n64;
  jbplan_even_split(SL.chunk, NC, c, &a64, &n64);
  const int a = (int)a64 + 1, n = (int)n64;  // owned planes a .. a + n - 1
  const int nmax = (int)((SL.chunk + NC - 1) / NC);
  const int rs = (int)g.pitch;
  double *buf[2] = {sm, sm + (size_t)(nmax + 2) * rs};
  // the neighbours' edge rows: the last owned row of CTA c-1, the first of CTA c+1
  int64_t au, nu;
  jbplan_even_split(SL.chunk, NC, c > 0 ? c - 1 : 0, &au, &nu);
  const bool up = c > 0, dn = c < NC - 1;

  // rows a-1 .. a+n of the current global level into both buffers (boundary cells included)
  {
    const double *src = SL.buf[P.t0 & 1] + (int64_t)(a - 1) * g.plane_elems;
    const int nd = (n + 2) * rs / 2;
    for (int k = tid; k < nd; k += JB_CNT) {
      const double2 v = __ldcg(reinterpret_cast<const double2 *>(src) + k);
      reinterpret_cast<double2 *>(buf[0])[k] = v;
      reinterpret_cast<double2 *>(buf[1])[k] = v;
    }
  }
  cluster_barrier();

  // work of this thread: cell pair j (x = 1 + 2j) over a band of its CTA's rows
  const int nx = (int)g.nx;
  const int ppr = (nx - 1) / 2;
  const int G = ppr <= JB_CNT ? JB_CNT / ppr : 1;  // row groups
  const int gi = ppr <= JB_CNT ? tid / ppr : 0;
  int r0 = 1, r1 = 0;
  if (gi < G) {
    int64_t s, l;
    jbplan_even_split(n, G, gi, &s, &l);
    r0 = 1 + (int)s;
    r1 = r0 + (int)l - 1;
  }
  const int jfirst = ppr <= JB_CNT ? tid - gi * ppr : tid;
  const int jstep = ppr <= JB_CNT ? ppr : JB_CNT;

  for (int64_t t = 0; t < P.iters; ++t) {
    const double *src = buf[t & 1];
    double *dst = buf[(t + 1) & 1];
    // the sweep: march this thread's pair down its rows, y-1 / y rows in registers; the rows
    // just above / below the CTA's band are the neighbour CTAs' edge rows of this level, read
    // straight from their shared memory (same layout: mapa of our own address; the upper
    // neighbour's last row is its local row nu)
    if (r0 <= r1)
      for (int j = jfirst; j < ppr; j += jstep) {
        const int x = 1 + 2 * j;
        const bool full = x + 1 <= nx - 2;
        const double *col = src + x + 3;
        double2 S = up && r0 == 1 ? ld_dsmem2(map_rank(col + (size_t)nu * rs, c - 1)) : lds2(col + (size_t)(r0 - 1) * rs);
        double2 C = lds2(col + (size_t)r0 * rs);
        double *o = dst + x + 3 + (size_t)r0 * rs;
        for (int r = r0; r <= r1; ++r, o += rs) {
          const double *cc = col + (size_t)r * rs;
          const double2 N = dn && r == n ? ld_dsmem2(map_rank(col + rs, c + 1)) : lds2(cc + rs);
          const double w = cc[-1], e = cc[2];
          // oracle order: ((x+1) + (x-1)) + (y+1) + (y-1), then * 0.25
          const double o0 = 0.25 * (((C.y + w) + N.x) + S.x);
          const double o1 = 0.25 * (((e + C.x) + N.y) + S.y);
          if (full) *reinterpret_cast<double2 *>(o) = make_double2(o0, o1);
          else o[0] = o0;
          S = C;
          C = N;
        }
      }
    // (a split-phase variant — inner rows swept before waiting, only the edge rows after — measured
    // slower: 1.32 vs 1.29 us/iteration for C1)
    cluster_barrier();  // this level is complete everywhere; nobody reads the older one any more
  }
  // the final level's owned rows back to the global buffer of the result
  {
    const double *res = buf[P.iters & 1] + rs;
    double *out = SL.buf[(P.t0 + P.iters) & 1] + (int64_t)a * g.plane_elems;
    const int nd = n * rs / 2;
    for (int k = tid; k < nd; k += JB_CNT)
      __stcg(reinterpret_cast<double2 *>(out) + k, reinterpret_cast<const double2 *>(res)[k]);
  }
}

}  // namespace

namespace jbk {

// Cluster size (16, else the largest power of two <= the rows that fits) and shared memory for a 2D slab of `chunk` rows, or 0 if it does not
// fit in one cluster.
int cluster_choice(const JbGeom &g, int64_t chunk, int smem_optin, size_t *smem_out) {
  const void *fn = reinterpret_cast<const void *>(&jb_cluster2d);
  for (int nc : {16, 8, 4, 2, 1}) {
    if (nc > chunk) continue;  // every CTA owns at least one row
    const int64_t nmax = (chunk + nc - 1) / nc;
    const size_t smem = (size_t)2 * (nmax + 2) * g.pitch * sizeof(double);
    if (nmax < 1 || smem > (size_t)smem_optin) continue;
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) continue;
    if (nc > 8 && cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess) continue;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(nc);
    cfg.blockDim = dim3(JB_CNT);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = nc;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int clusters = 0;
    if (cudaOccupancyMaxActiveClusters(&clusters, fn, &cfg) != cudaSuccess || clusters < 1) {
      cudaGetLastError();
      continue;
    }
    *smem_out = smem;
    return nc;
  }
  cudaGetLastError();
  return 0;
}

cudaError_t launch_cluster(const JbParams &p, int nc, size_t smem, cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(nc);
  cfg.blockDim = dim3(JB_CNT);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = nc;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, jb_cluster2d, p);
}

}  // namespace jbk
