// Microbenchmark: device-wide barrier variants (the CPU-Free kernels' per-iteration grid
// barrier), G CTAs x 288 threads (one per SM), ns per barrier via %globaltimer.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubb scripts/ubench_barrier.cu && /tmp/ubb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long *p) {
  unsigned long long v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ unsigned long long ld_rlx(const unsigned long long *p) {
  unsigned long long v; asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ unsigned long long ld_vol(const unsigned long long *p) {
  unsigned long long v; asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void red_rel(unsigned long long *p, unsigned long long v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_rlx(unsigned long long *p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long atom_acqrel(unsigned long long *p, unsigned long long v) {
  unsigned long long o; asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;" : "=l"(o) : "l"(p), "l"(v) : "memory"); return o;
}
__device__ __forceinline__ void st_rel(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ void cl_arrive() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void cl_wait() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ unsigned cl_rank() { unsigned r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned cl_n() { unsigned r; asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r)); return r; }

// MODE 0: counter (production form): lane 0 red.release + ld.acquire spin
// MODE 1: counter, relaxed spin + one fence after
// MODE 2: atom.acq_rel arrive; last arriver st.release on a separate flag line; others spin on it
// MODE 3: counter without the release (INCORRECT, measures the release's cost)
// MODE 4: MODE 0 + fence.proxy.async by every thread (as the streaming kernel does)
// MODE 5: cluster-hierarchical: cluster barrier, rank 0 counter (clusters arrive), cluster barrier
// MODE 6: counter, volatile spin + fence after
// MODE 7: production arrival, lane 0 of NPW warps polls (naturally staggered), the first to see
//         the count raises a shared-memory flag the others also watch
// bounded spin: a barrier that never completes (CTAs not co-resident) gives up after 0.5 s
#define SPIN(cond) { const uint64_t ts_ = gt(); while (cond) { if (*(volatile unsigned long long *)(out + 148)) break; if (gt() - ts_ > 500000000ull) { out[148] = 1; break; } } }
template <int MODE>
__global__ void k(unsigned long long *ctr, unsigned long long *flag, int n, unsigned long long *out, int nunits) {
  const int tid = threadIdx.x;
  __shared__ volatile int s_done[2];
  if (tid == 0) s_done[0] = s_done[1] = 0;
  __syncthreads();
  uint64_t t0 = gt();
  for (int i = 0; i < n; ++i) {
    const unsigned long long target = (unsigned long long)nunits * (i + 1);
    if (MODE == 4) fence_proxy();
    if (MODE == 5) {
      cl_arrive(); cl_wait();
      if (cl_rank() == 0 && tid == 0) {
        red_rel(ctr, 1ull);
        SPIN(ld_acq(ctr) < target)
      }
      cl_arrive(); cl_wait();
      continue;
    }
    if (MODE >= 7) {
      const int NPW = MODE - 5;  // 7: 2 warps, 8: 3, 9: 4
      __syncthreads();
      const int par = i & 1;
      if (tid == 0) { s_done[par ^ 1] = 0; red_rel(ctr, 1ull); }
      if ((tid & 31) == 0 && (tid >> 5) < NPW) {
        const uint64_t ts_ = gt();
        while (!s_done[par]) {
          if (ld_acq(ctr) >= target) { s_done[par] = 1; break; }
          if (*(volatile unsigned long long *)(out + 148)) break;
          if (gt() - ts_ > 500000000ull) { out[148] = 1; break; }
        }
      }
      __syncthreads();
      continue;
    }
    __syncthreads();
    if (tid == 0) {
      if (MODE == 0 || MODE == 4) { red_rel(ctr, 1ull); SPIN(ld_acq(ctr) < target) }
      else if (MODE == 1) { red_rel(ctr, 1ull); SPIN(ld_rlx(ctr) < target) fence_gpu(); }
      else if (MODE == 6) { red_rel(ctr, 1ull); SPIN(ld_vol(ctr) < target) fence_gpu(); }
      else if (MODE == 3) { red_rlx(ctr, 1ull); SPIN(ld_rlx(ctr) < target) }
      else if (MODE == 2) {
        const unsigned long long o = atom_acqrel(ctr, 1ull);
        if (o + 1 == target) st_rel(flag, (unsigned long long)(i + 1));
        else SPIN(ld_acq(flag) < (unsigned long long)(i + 1))
      }
    }
    __syncthreads();
  }
  uint64_t t1 = gt();
  if (tid == 0) out[blockIdx.x] = t1 - t0;
}

template <int MODE>
float run(int grid, int cluster, unsigned long long *ctr, unsigned long long *flag, unsigned long long *out) {
  const int n = 4000;
  cudaMemset(ctr, 0, 8); cudaMemset(flag, 0, 8);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid); cfg.blockDim = dim3(288); cfg.dynamicSmemBytes = 0; cfg.stream = 0;
  cudaLaunchAttribute at[1];
  int na = 0;
  if (cluster > 1) {
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cluster; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    na = 1;
  }
  cfg.attrs = at; cfg.numAttrs = na;
  const int nunits = MODE == 5 ? grid / cluster : grid;
  cudaError_t e = cudaLaunchKernelEx(&cfg, k<MODE>, ctr, flag, n, out, nunits);
  if (e != cudaSuccess) { printf("launch error %s\n", cudaGetErrorString(e)); cudaGetLastError(); return -1; }
  e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return -1; }
  unsigned long long h, bad;
  cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(&bad, out + 148, 8, cudaMemcpyDeviceToHost);
  if (bad) { printf("(timed out: not co-resident)\n"); cudaMemset(out + 148, 0, 8); return -1; }
  return (float)h / n;
}

int main() {
  unsigned long long *ctr, *flag, *out;
  cudaMalloc(&ctr, 256); cudaMalloc(&flag, 256); cudaMalloc(&out, 149 * 8); cudaMemset(out, 0, 149 * 8);
  const char *names[] = {"counter red.release + ld.acquire spin (production)", "counter, relaxed spin + fence",
                         "atom.acq_rel + last-arriver release flag", "counter without release (incorrect)",
                         "production + fence.proxy.async", "cluster-hierarchical", "counter, volatile spin + fence",
                         "production arrival, 2 polling warps", "production arrival, 3 polling warps",
                         "production arrival, 4 polling warps"};
  for (int grid : {1, 8, 32, 74, 148}) {
    for (int m = 0; m < 10; ++m) {
      if (m == 5 || m == 1 || m == 2 || m == 3 || m == 4 || m == 6) continue;
      float v = 0;
      for (int rep = 0; rep < 2; ++rep) {
        if (m == 0) v = run<0>(grid, 1, ctr, flag, out);
        if (m == 1) v = run<1>(grid, 1, ctr, flag, out);
        if (m == 2) v = run<2>(grid, 1, ctr, flag, out);
        if (m == 3) v = run<3>(grid, 1, ctr, flag, out);
        if (m == 4) v = run<4>(grid, 1, ctr, flag, out);
        if (m == 6) v = run<6>(grid, 1, ctr, flag, out);
        if (m == 7) v = run<7>(grid, 1, ctr, flag, out);
        if (m == 8) v = run<8>(grid, 1, ctr, flag, out);
        if (m == 9) v = run<9>(grid, 1, ctr, flag, out);
      }
      printf("ctas %3d  %-52s %8.1f ns/barrier\n", grid, names[m], v);
    }
  }
  for (int cl : {0}) {  // (cluster-hierarchical: profiles/r02_ubench_barrier.txt)
    if (!cl) continue;
    for (int grid : {cl * 8, 144}) {
      if (cl == 16) {
        cudaFuncSetAttribute(k<5>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      }
      float v = 0;
      for (int rep = 0; rep < 2; ++rep) v = run<5>(grid / cl * cl, cl, ctr, flag, out);
      printf("ctas %3d  %-44s cl=%2d %8.1f ns/barrier\n", grid / cl * cl, names[5], cl, v);
    }
  }
  return 0;
}
