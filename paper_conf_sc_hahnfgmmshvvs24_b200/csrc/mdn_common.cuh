// mdn_common.cuh -- helpers shared by the MDNorm (mdn_kernels.cu) and BinMD (mdn_binmd.cu)
// translation units: matrix staging (M0 / B0), histogram accumulation (M7 / B3), work counters and
// launch-size arithmetic.  Internal; not part of the ABI.
#pragma once
#include <algorithm>
#include <cstdint>
#include <type_traits>

#include "mdn_kernels.cuh"

namespace mdn {
namespace common {

constexpr int kThreads = 256;
constexpr unsigned kFull = 0xffffffffu;

// M0: M_{r,s} (run-major m = r * nops + s) and the per-matrix charge into shared memory; a
// singular composition stages NaNs (the cull drops non-finite directions, as the oracle does).
__device__ __forceinline__ void stage_mdnorm_mats(const MatBlock& mb, double* sM, double* sC) {
  for (int m = threadIdx.x; m < mb.nmat; m += blockDim.x) {
    if (mb.compose) {
      const int r = m / mb.nops, s = m - r * mb.nops;
      if (!compose_mdnorm(mb.u.c.R + 9 * r, mb.UB, mb.u.c.ops + 9 * s, mb.W, sM + 9 * m))
        for (int i = 0; i < 9; ++i) sM[9 * m + i] = CUDART_NAN;
      sC[m] = mb.charge[r];
    } else {
      for (int i = 0; i < 9; ++i) sM[9 * m + i] = mb.u.M[9 * m + i];
      sC[m] = mb.charge[m];
    }
  }
}

// B0: N_s into shared memory.
__device__ __forceinline__ void stage_binmd_mats(const MatBlock& mb, double* sN) {
  for (int m = threadIdx.x; m < mb.nmat; m += blockDim.x) {
    if (mb.compose) {
      if (!compose_binmd(mb.UB, mb.u.c.ops + 9 * m, mb.W, sN + 9 * m))
        for (int i = 0; i < 9; ++i) sN[9 * m + i] = CUDART_NAN;
    } else {
      for (int i = 0; i < 9; ++i) sN[9 * m + i] = mb.u.M[9 * m + i];
    }
  }
}

// One warp-aggregated atomic per counter per warp (tracing only; compiled out when kStats off).
__device__ __forceinline__ void flush_counter(unsigned long long* dst, unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(kFull, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}

// h[b] += v (and h2[b] += v2 when two).  Warp-aggregated reductions (__match_any_sync on the bin,
// shuffle sums, one reduction per distinct bin; north_star "warp-aggregated atomics") were
// measured slower on this B200 -- BinMD 2x on the Morton-ordered CORELLI events, 1.8x on TOPAZ
// 48 ops, 1.6x into a private shared-memory grid; the walk 1.4-1.75x -- so every
// contribution is its own reduction.
// The global fp64 form is an explicit fire-and-forget reduction (red.global.add.f64): the
// compiler otherwise emits an atomic with a (discarded) return in code that also holds
// acquire/release operations, which waits for the L2 round trip.
__device__ __forceinline__ void red_add(double* p, double v) {
  asm volatile("red.relaxed.gpu.global.add.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
template <typename T>
__device__ __forceinline__ void hist_add(T* h, T* h2, int b, T v, T v2, bool two) {
  atomicAdd(h + b, v);
  if (two) atomicAdd(h2 + b, v2);
}
__device__ __forceinline__ void hist_add(double* h, double* h2, int b, double v, double v2, bool two) {
  red_add(h + b, v);
  if (two) red_add(h2 + b, v2);
}

// Zero the CTA's private histogram (before the kernel's first __syncthreads).
template <typename T>
__device__ __forceinline__ void priv_zero(T* h, int64_t n) {
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) h[i] = T(0);
}

// Fold the CTA's private histogram into the global fp64 one: one red.add per touched bin
// (every contribution is >= 0 for MDNorm; a BinMD bin whose weights cancel to 0 is skipped,
// which leaves the same sum).  Call after a __syncthreads.
template <typename T>
__device__ __forceinline__ void priv_flush(const T* h, double* dst, int64_t n) {
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const T v = h[i];
    if (v != T(0)) red_add(dst + i, (double)v);
  }
}

// kPriv: 0 = global fp64 red.add, 1 = fp64 shared-memory partials, 2 = fp32 shared-memory partials
template <int kPriv>
using priv_t = typename std::conditional<kPriv == 2, float, double>::type;

// bytes of a private histogram of n bins, rounded up to 16
__host__ __device__ constexpr size_t priv_bytes(int kind, int64_t n) {
  return kind == 0 ? 0 : (((size_t)n * (kind == 2 ? 4 : 8) + 15) & ~(size_t)15);
}

inline int grid_for(int64_t work, int num_sms, int per_sm, int threads = kThreads) {
  int64_t blocks = (work + threads - 1) / threads;
  blocks = std::min<int64_t>(blocks, (int64_t)num_sms * per_sm);
  return (int)std::max<int64_t>(blocks, 1);
}

inline int smem_optin(cudaError_t* err) {
  int dev = 0, smem_max = 0;
  if ((*err = cudaGetDevice(&dev)) != cudaSuccess) return 0;
  *err = cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return smem_max;
}

}  // namespace common
}  // namespace mdn
