// util.cu — initialisation and flag utility kernels of libjacobi_b200.
#include "device_common.cuh"

namespace {

// ---------------------------------------------------------------- init / utility kernels
__device__ __forceinline__ double u12_value(unsigned long long idx, unsigned long long seed) {
  unsigned long long z = seed + (idx + 1ull) * kGolden;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z = z ^ (z >> 31);
  return __longlong_as_double((long long)(0x3FF0000000000000ull | (z >> 12)));
}

// Fill planes 0..nplanes-1 of a slab whose plane 0 is global outer index z_first with U12.
__global__ void jb_init_u12(double *b0, double *b1, int64_t nplanes, JbGeom g, int64_t z_first,
                            unsigned long long seed) {
  const int64_t n = nplanes * g.plane_elems;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = i / g.plane_elems, rem = i - p * g.plane_elems;
    int64_t y, pos, idx = -1;
    if (g.dim == 2) {
      y = z_first + p;
      pos = rem;
      const int64_t x = pos - 3;
      if (x >= 0 && x < g.nx) idx = y * g.nx + x;
    } else {
      y = rem / g.pitch;
      pos = rem - y * g.pitch;
      const int64_t x = pos - 3;
      if (x >= 0 && x < g.nx) idx = ((z_first + p) * g.ny + y) * g.nx + x;
    }
    const double v = idx >= 0 ? u12_value((unsigned long long)idx, seed) : 0.0;
    b0[i] = v;
    if (b1) b1[i] = v;
  }
}

__global__ void jb_flag_max(unsigned long long *flags, int n, unsigned long long v) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) atomicMax(flags + i, v);
}

}  // namespace

namespace jbk {

cudaError_t launch_init(double *b0, double *b1, int64_t nplanes, const JbGeom &g, int64_t z_first,
                        unsigned long long seed, cudaStream_t st) {
  jb_init_u12<<<1184, 256, 0, st>>>(b0, b1, nplanes, g, z_first, seed);
  return cudaGetLastError();
}

cudaError_t launch_flag_max(unsigned long long *flags, int n, unsigned long long v, cudaStream_t st) {
  jb_flag_max<<<1, 64, 0, st>>>(flags, n, v);
  return cudaGetLastError();
}

}  // namespace jbk
