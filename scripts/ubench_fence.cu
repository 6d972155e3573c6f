// Microbenchmark: cost of (stores by 256 threads; bar.sync; thread 0 st.release.{sys,gpu} flag),
// per iteration, one CTA (and 148 CTAs), in ns via %globaltimer.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
template <int MODE>
__global__ void k(double *buf, unsigned long long *flag, int n, int bytes_per_thread, unsigned long long *out) {
  const int tid = threadIdx.x;
  double *b = buf + (size_t)blockIdx.x * 4096;
  __syncthreads();
  uint64_t t0 = gt();
  for (int i = 0; i < n; ++i) {
    for (int j = tid; j < bytes_per_thread * blockDim.x / 8; j += blockDim.x) b[j] = (double)i;
    __syncthreads();
    if (tid == 0) {
      if (MODE == 0) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(flag + blockIdx.x * 16), "l"((unsigned long long)i) : "memory");
      else if (MODE == 1) asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(flag + blockIdx.x * 16), "l"((unsigned long long)i) : "memory");
      else if (MODE == 2) asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(flag + blockIdx.x * 16), "l"((unsigned long long)i) : "memory");
      else if (MODE == 3) { asm volatile("fence.acq_rel.sys;" ::: "memory"); asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(flag + blockIdx.x * 16), "l"((unsigned long long)i) : "memory"); }
    }
    __syncthreads();
  }
  uint64_t t1 = gt();
  if (tid == 0) out[blockIdx.x] = t1 - t0;
}
int main() {
  double *buf; unsigned long long *flag, *out;
  cudaMalloc(&buf, 148 * 4096 * 8); cudaMalloc(&flag, 148 * 16 * 8); cudaMalloc(&out, 148 * 8);
  unsigned long long h[148];
  const char *names[] = {"st.release.sys", "st.release.gpu", "st.relaxed.gpu (no fence)", "fence.acq_rel.sys+st.relaxed.sys"};
  for (int grid : {1, 148})
  for (int bpt : {0, 32, 128}) {
    for (int m = 0; m < 4; ++m) {
      for (int rep = 0; rep < 2; ++rep) {
        const int n = 2000;
        if (m == 0) k<0><<<grid, 256>>>(buf, flag, n, bpt, out);
        if (m == 1) k<1><<<grid, 256>>>(buf, flag, n, bpt, out);
        if (m == 2) k<2><<<grid, 256>>>(buf, flag, n, bpt, out);
        if (m == 3) k<3><<<grid, 256>>>(buf, flag, n, bpt, out);
        cudaDeviceSynchronize();
        cudaMemcpy(h, out, grid * 8, cudaMemcpyDeviceToHost);
        if (rep == 1) printf("grid %3d bytes/thread %3d %-36s %8.1f ns/iter\n", grid, bpt, names[m], (double)h[0] / n);
      }
    }
  }
  return 0;
}
