// device_common.cuh — PTX helpers, waits, ring positions and small device utilities shared by
// the kernels of libjacobi_b200 (sweep.cu, resident.cu, util.cu).  Internal linkage per TU.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/jacobi.h"
#include "jacobi_internal.h"
#ifdef JB_NVSHMEM
#include <nvshmem.h>
#include <nvshmemx.h>
#endif

namespace {

constexpr double kC6 = 0x1.5555555555555p-3;  // fl(1/6), reading R3
constexpr unsigned long long kGolden = 0x9E3779B97F4A7C15ull;

enum Role { ROLE_INT = 0, ROLE_TOP = 1, ROLE_BOT = 2 };

// Same even split as jbplan::even_split (host): part i of n items over k parts.
__device__ __forceinline__ void jbplan_even_split(int64_t n, int k, int i, int64_t *start, int64_t *len) {
  const int64_t q = n / k, r = n % k;
  *len = q + (i < r ? 1 : 0);
  *start = (int64_t)i * q + min((int64_t)i, r);
}

// ---------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t sptr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sptr(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sptr(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sptr(b)) : "memory");
}
// 32-bit shared-window address forms (the address computed once by the caller)
__device__ __forceinline__ void mbar_arrive_s(uint32_t a) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ void mbar_wait_s(uint32_t a, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(a), "r"(parity)
      : "memory");
}
// A value the compiler must keep (it cannot re-derive it from special registers inside a loop).
__device__ __forceinline__ uint32_t opaque_u32(uint32_t v) {
  asm volatile("mov.b32 %0, %0;" : "+r"(v));
  return v;
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      " selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(sptr(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  while (!mbar_try_wait(b, parity)) {
  }
}
// 1D bulk copy global -> shared (TMA engine), completion counted in bytes on an mbarrier.
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          sptr(dst)),
      "l"(src), "r"(bytes), "r"(sptr(bar))
      : "memory");
}
// Same bulk copy with an L2 cache-eviction policy (createpolicy).
__device__ __forceinline__ void bulk_g2s_hint(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                              uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          sptr(dst)),
      "l"(src), "r"(bytes), "r"(sptr(bar)), "l"(policy)
      : "memory");
}
__device__ __forceinline__ uint64_t l2_policy(bool evict_last) {
  uint64_t p;
  if (evict_last) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  else asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_gpu(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// Halo flags: .sys scope when a neighbour may sit on another GPU or in another
// process; .gpu when the host marked the launch as one device (virtual slabs, JB_PFLAG_GPU_SCOPE):
// the release then skips the system-wide MEMBAR (1.5-3.9 us measured, profiles/r02_ubench_fence.txt).
__device__ __forceinline__ bool flag_gpu_scope(const JbParams &P) { return (P.flags & JB_PFLAG_GPU_SCOPE) != 0; }
__device__ __forceinline__ void st_release_flag(const JbParams &P, unsigned long long *p, unsigned long long v) {
  if (flag_gpu_scope(P)) st_release_gpu(p, v);
  else st_release_sys(p, v);
}
__device__ __forceinline__ unsigned long long ld_acquire_flag(const JbParams &P, const unsigned long long *p) {
  return flag_gpu_scope(P) ? ld_acquire_gpu(p) : ld_acquire_sys(p);
}
__device__ __forceinline__ void red_release_gpu_add(unsigned long long *p, unsigned long long v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void named_bar_consumers() {
  asm volatile("bar.sync 1, %0;" ::"r"(JB_NC) : "memory");
}

// Spin until *p >= target (acquire at sys or gpu scope).  Watchdog: after timeout_ns set
// status = ETIMEOUT and the abort flag; also gives up once another CTA raised abort.
template <bool SYS>
__device__ bool wait_geq(const unsigned long long *p, unsigned long long target, const JbParams &P) {
  auto ld = [&]() { return SYS ? ld_acquire_sys(p) : ld_acquire_gpu(p); };
  if (ld() >= target) return true;
  const unsigned long long t_start = globaltimer();
  uint32_t n = 0;
  volatile int *abort_flag = P.status + 1;
  while (true) {
    if (ld() >= target) return true;
    if ((++n & 127u) == 0) {
      if (*abort_flag) return false;
      if (globaltimer() - t_start > P.timeout_ns) {
        atomicCAS(P.status, 0, JACOBI_ETIMEOUT);
        atomicExch(P.status + 1, 1);
        return false;
      }
    }
  }
}

// Warp-cooperative wait until flag slots 0..k-1 all reach `target` (lane i polls slot i).
__device__ bool wait_slots(const unsigned long long *slots, int k, unsigned long long target, const JbParams &P,
                           int lane) {
  const unsigned long long t_start = globaltimer();
  uint32_t n = 0;
  volatile int *abort_flag = P.status + 1;
  while (true) {
    const bool ok = lane >= k || ld_acquire_flag(P, slots + lane) >= target;
    if (__all_sync(0xffffffffu, ok)) return true;
    if ((++n & 127u) == 0) {
      int stop = 0;
      if (lane == 0) {
        if (*abort_flag) {
          stop = 1;
        } else if (globaltimer() - t_start > P.timeout_ns) {
          atomicCAS(P.status, 0, JACOBI_ETIMEOUT);
          atomicExch(P.status + 1, 1);
          stop = 1;
        }
      }
      if (__shfl_sync(0xffffffffu, stop, 0)) return false;
    }
  }
}

// Wait until flags[idx[i]] >= target for i < n (n <= 32; lane i polls entry i), gpu scope.
__device__ bool wait_slots_idx(const unsigned long long *flags, const int *idx, int n, unsigned long long target,
                               const JbParams &P, int lane) {
  const unsigned long long *mine = nullptr;
#pragma unroll
  for (int i = 0; i < 4; ++i)
    if (i == lane && i < n) mine = flags + idx[i];
  const unsigned long long t_start = globaltimer();
  uint32_t cnt = 0;
  volatile int *abort_flag = P.status + 1;
  while (true) {
    const bool ok = mine == nullptr || ld_acquire_gpu(mine) >= target;
    if (__all_sync(0xffffffffu, ok)) return true;
    if ((++cnt & 127u) == 0) {
      int stop = 0;
      if (lane == 0) {
        if (*abort_flag) {
          stop = 1;
        } else if (globaltimer() - t_start > P.timeout_ns) {
          atomicCAS(P.status, 0, JACOBI_ETIMEOUT);
          atomicExch(P.status + 1, 1);
          stop = 1;
        }
      }
      if (__shfl_sync(0xffffffffu, stop, 0)) return false;
    }
  }
}

// Halo-exchange trace (measurement only, JbSlab::halo_trace): exchange e of side `side` (0 top,
// 1 bottom), event `which` (0 wait begins, 1 neighbour's flag acquired, 2 own signal released).
__device__ __forceinline__ void halo_mark(const JbSlab &SL, const JbParams &P, int side, int64_t e, int which) {
  if (SL.halo_trace && e >= 0 && e < P.halo_trace_n)
    SL.halo_trace[((int64_t)side * P.halo_trace_n + e) * 3 + which] = globaltimer();
}

__device__ __forceinline__ unsigned long long ld_relaxed_gpu(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

// Device-side grid barrier of a slab's CTAs (P:372 grid.sync()), called by warp 0 of every CTA
// after a CTA barrier (whose cumulativity puts the whole CTA's writes before the arrival), followed
// by a CTA barrier.  epoch = the global iteration count after this barrier (unique and increasing
// across runs); k = the barrier's 1-based index in this launch (counter form).  Two forms:
//  * counter (default): lane 0 red.release.gpu.add 1 on the slab counter, spins until it reaches
//    cta_count * k (acquire);
//  * flags (SL.bar_flags): lane 0 st.release.gpu of the epoch into this CTA's own slot; the warp
//    polls all cta_count slots with relaxed loads issued in parallel (lane i: slots i, i+32, ..),
//    then one fence.acq_rel.gpu (the acquire pattern) — no atomic serialised on one L2 address.
// Returns false on abort / watchdog timeout (as wait_slots).
// sig (lane 0, optional): a halo flag (P:394's signal) to raise with value sigv as part of the
// arrival — one release fence (at the flag's scope) then relaxed stores of the flag and the
// arrival, instead of the flag's own release store followed by the arrival's release.
__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ void st_relaxed_sys(unsigned long long *p, unsigned long long v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed_gpu_add(unsigned long long *p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu(unsigned long long *p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ bool slab_barrier(const JbSlab &SL, const JbParams &P, int c, unsigned long long k,
                             unsigned long long epoch, int lane, unsigned long long *sig = nullptr,
                             unsigned long long sigv = 0, unsigned long long *sig2 = nullptr) {
  // release pattern: fence, then relaxed stores of the flag(s) and the arrival (sig2: a second
  // flag with the same value — a block that borders both neighbours)
  auto fence_and_signal = [&]() {
    if (flag_gpu_scope(P)) {
      fence_acq_rel_gpu();
      st_relaxed_gpu(sig, sigv);
      if (sig2) st_relaxed_gpu(sig2, sigv);
    } else {
      fence_acq_rel_sys();
      st_relaxed_sys(sig, sigv);
      if (sig2) st_relaxed_sys(sig2, sigv);
    }
  };
  // The abort flag (another CTA's watchdog / error) is read right AFTER the arrival (not before:
  // the arrival's release fence would wait for the load), so its L2 round trip overlaps the spin
  // instead of following the barrier on every iteration's critical path; an abort raised later
  // is seen by the spins (every 128 polls) or at the next barrier.
  int aborted = 0;
  if (!SL.bar_flags) {
    bool ok = true;
    if (lane == 0) {
      if (sig) {
        fence_and_signal();
        red_relaxed_gpu_add(SL.barrier, 1ull);
      } else {
        red_release_gpu_add(SL.barrier, 1ull);
      }
      aborted = *(volatile int *)(P.status + 1);
      ok = wait_geq<false>(SL.barrier, (unsigned long long)SL.cta_count * k, P) && !aborted;
    }
    return __shfl_sync(0xffffffffu, ok ? 1 : 0, 0) != 0;
  }
  if (lane == 0) {
    if (sig) {
      fence_and_signal();
      st_relaxed_gpu(SL.bar_flags + c, epoch);
    } else {
      st_release_gpu(SL.bar_flags + c, epoch);
    }
    aborted = *(volatile int *)(P.status + 1);
  }
  aborted = __shfl_sync(0xffffffffu, aborted, 0);
  const int n = SL.cta_count;
  const unsigned long long t_start = globaltimer();
  uint32_t cnt = 0;
  volatile int *abort_flag = P.status + 1;
  while (true) {
    bool mine = true;
#pragma unroll 4
    for (int s = lane; s < n; s += 32) mine &= ld_relaxed_gpu(SL.bar_flags + s) >= epoch;
    if (__all_sync(0xffffffffu, mine)) break;
    if ((++cnt & 127u) == 0) {
      int stop = 0;
      if (lane == 0) {
        if (*abort_flag) {
          stop = 1;
        } else if (globaltimer() - t_start > P.timeout_ns) {
          atomicCAS(P.status, 0, JACOBI_ETIMEOUT);
          atomicExch(P.status + 1, 1);
          stop = 1;
        }
      }
      if (__shfl_sync(0xffffffffu, stop, 0)) return false;
    }
  }
  fence_acq_rel_gpu();
  return !aborted;
}

// Position in the shared-memory ring: slot and the parity of the current use of that slot.
struct RingPos {
  uint32_t slot, phase;
  __device__ __forceinline__ void advance(uint32_t S) {
    if (++slot == S) {
      slot = 0;
      phase ^= 1u;
    }
  }
};

struct Ring {
  uint64_t *full, *empty;
  double *stages;
  uint32_t S;
  int stage_doubles;
  __device__ __forceinline__ double *stage(const RingPos &p) const {
    return stages + (size_t)p.slot * stage_doubles;
  }
  __device__ __forceinline__ void wait_full(const RingPos &p) const { mbar_wait(&full[p.slot], p.phase); }
  // A consumer warp releases a stage: every lane arrives after its own last read (the empty
  // barrier counts consumer THREADS), so each reading thread orders its reads before the
  // producer's next bulk copy into the slot itself (mbarrier release/acquire) — the canonical
  // TMA-pipeline form, which compute-sanitizer's racecheck can follow (a __syncwarp + one
  // lane's arrive is ordered by the PTX model too, but racecheck flags it once the ring wraps).
  __device__ __forceinline__ void release(const RingPos &p, int /*lane*/) const { mbar_arrive(&empty[p.slot]); }
};

// ---------------------------------------------------------------- small load/store helpers
__device__ __forceinline__ double2 lds2(const double *p) { return *reinterpret_cast<const double2 *>(p); }
// 32-bit shared-window addresses (sptr): one register per address, no generic-to-shared conversion
__device__ __forceinline__ double2 lds2_s(uint32_t a) {
  double2 v;
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ double lds_s(uint32_t a) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ void store_pair(double *p, double o0, double o1, bool pair) {
  if (pair) *reinterpret_cast<double2 *>(p) = make_double2(o0, o1);
  else *p = o0;
}

}  // namespace
