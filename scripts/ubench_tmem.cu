// Microbenchmark: Tensor Memory (TMEM) as register spill space for a stencil march — dependent
// round trip tcgen05.st (32x32b.x4: one double2 per lane) + wait::st + tcgen05.ld + wait::ld, in
// SM cycles, vs an LDS.128 / STS.128 round trip.  One CTA of 4 warps (one TMEM lane quarter each).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubt scripts/ubench_tmem.cu && /tmp/ubt
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k(unsigned long long *out, int n, double seed) {
  __shared__ uint32_t tmem_base;
  __shared__ __align__(16) double sm[128 * 2];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(&tmem_base)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t taddr = tmem_base + ((uint32_t)(warp * 32) << 16);  // lane quarter of this warp
  double a = seed + lane, b = seed * 2 + lane;
  // TMEM round trip
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) {
    uint32_t r0 = __double2loint(a), r1 = __double2hiint(a), r2 = __double2loint(b), r3 = __double2hiint(b);
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};" ::"r"(taddr), "r"(r0), "r"(r1),
                 "r"(r2), "r"(r3) : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(taddr) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    a = __hiloint2double(r1, r0) + 1.0;
    b = __hiloint2double(r3, r2) + 1.0;
  }
  long long t1 = clock64();
  // TMEM load only (independent of the previous iteration's load: pipelined issue + one wait)
  long long t2 = clock64();
  for (int i = 0; i < n; ++i) {
    uint32_t r0, r1, r2, r3;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(taddr) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    a += __hiloint2double(r1, r0);
    b += __hiloint2double(r3, r2);
  }
  long long t3 = clock64();
  // shared-memory round trip
  long long t4 = clock64();
  for (int i = 0; i < n; ++i) {
    double2 *p = reinterpret_cast<double2 *>(sm) + (threadIdx.x & 127);
    *p = make_double2(a, b);
    __syncwarp();
    double vx, vy;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(vx), "=d"(vy) : "r"((uint32_t)__cvta_generic_to_shared(p)) : "memory");
    a = vx + 1.0;
    b = vy + 1.0;
  }
  long long t5 = clock64();
  if (threadIdx.x == 0) {
    out[0] = t1 - t0;
    out[1] = t3 - t2;
    out[2] = t5 - t4;
    out[3] = (unsigned long long)(a + b);
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tmem_base) : "memory");
}

int main() {
  unsigned long long *d, h[4];
  cudaMalloc(&d, 64);
  const int n = 10000;
  for (int rep = 0; rep < 2; ++rep) {
    k<<<1, 128>>>(d, n, 0.5);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    cudaMemcpy(h, d, 32, cudaMemcpyDeviceToHost);
    if (rep == 1)
      printf("cycles per iteration: TMEM st+wait+ld+wait round trip %.1f, TMEM ld+wait %.1f, STS.128+LDS.128 %.1f\n",
             (double)h[0] / n, (double)h[1] / n, (double)h[2] / n);
  }
  return 0;
}
