// mdn_kernels.cu -- sm_100a kernels of the MDNorm / BinMD cross-section hot path.
//
// Rows of SURVEY.md §8(a):  M0 compose (prologue of mdnorm_kernel), M1-M7 mdnorm_kernel,
// B0 compose (prologue of binmd_kernel), B1-B3 binmd_kernel, X2 xs_kernel.  The parity entry
// points (debug_*) run the very same device functions (mdn_device.cuh).
#include <algorithm>

#include "mdn_kernels.cuh"

namespace mdn {

namespace {

constexpr int kThreads = 256;

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
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}

struct AtomicEmit {
  double* h;
  __device__ __forceinline__ void operator()(int64_t b, double val) const { atomicAdd(h + b, val); }
};

// ---------------------------------------------------------------- M1-M7: one thread per pixel,
// looping over every (run, op) matrix of the launch (pixel read once, P:102 collapse(2) space).
template <bool kSmemFlux, bool kStats>
__global__ void __launch_bounds__(kThreads)
mdnorm_kernel(const __grid_constant__ MdnParams p, const __grid_constant__ MatBlock mb) {
  extern __shared__ double smem[];
  double* sM = smem;
  double* sC = sM + 9 * mb.nmat;
  double* sK = sC + mb.nmat;
  double* sF = sK + (kSmemFlux ? p.nflux : 0);
  stage_mdnorm_mats(mb, sM, sC);
  if (kSmemFlux)
    for (int i = threadIdx.x; i < p.nflux; i += blockDim.x) {
      sK[i] = p.flux_k[i];
      sF[i] = p.flux_F[i];
    }
  __syncthreads();
  const FluxView fx{kSmemFlux ? sK : p.flux_k, kSmemFlux ? sF : p.flux_F, p.nflux};
  AtomicEmit emit{p.norm};
  unsigned long long c_traj = 0, c_hit = 0, c_cross = 0, c_seg = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < p.nshard; i += stride) {
    const double4 px = p.pix[p.pix_begin + i * p.pix_stride];
    if (kStats) c_traj += mb.nmat;
    if (px.w == 0.0) continue;  // masked pixel contributes 0 (reading #16)
    for (int m = 0; m < mb.nmat; ++m) {
      const double* M = sM + 9 * m;
      double v[3] = {row_dot(M, px.x, px.y, px.z), row_dot(M + 3, px.x, px.y, px.z),
                     row_dot(M + 6, px.x, px.y, px.z)};
      double kin, kout;
      if (!traj_clip(p.g, v, p.kmin, p.kmax, kin, kout)) continue;
      int nc;
      const int ns = traj_walk(p.g, fx, v, kin, kout, dmul(px.w, sC[m]), emit, &nc);
      if (kStats) {
        c_hit += 1;
        c_cross += nc - 2;
        c_seg += ns;
      }
    }
  }
  if (kStats) {
    flush_counter(p.stats + 0, c_traj);
    flush_counter(p.stats + 1, c_hit);
    flush_counter(p.stats + 2, c_cross);
    flush_counter(p.stats + 3, c_seg);
  }
}

// ---------------------------------------------------------------- B1-B3: one thread per event
template <bool kPacked, bool kStats>
__global__ void __launch_bounds__(kThreads)
binmd_kernel(const __grid_constant__ BinParams p, const __grid_constant__ MatBlock mb) {
  __shared__ double sN[kMaxMats * 9];
  stage_binmd_mats(mb, sN);
  __syncthreads();
  unsigned long long c_pairs = 0, c_in = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < p.nevents; e += stride) {
    float w, q0, q1, q2;
    if (kPacked) {
      const float4 ev = __ldcs(reinterpret_cast<const float4*>(p.events) + e);
      w = ev.x; q0 = ev.y; q1 = ev.z; q2 = ev.w;
    } else {
      const float* ev = p.events + e * p.stride;
      w = __ldcs(ev + p.col_w);
      q0 = __ldcs(ev + p.col_q);
      q1 = __ldcs(ev + p.col_q + 1);
      q2 = __ldcs(ev + p.col_q + 2);
    }
    const double wd = (double)w, d0 = (double)q0, d1 = (double)q1, d2 = (double)q2;
    if (kStats) c_pairs += mb.nmat;
    for (int m = 0; m < mb.nmat; ++m) {
      const int64_t b = event_bin(p.g, sN + 9 * m, d0, d1, d2);
      if (b >= 0) {
        atomicAdd(p.binmd + b, wd);
        if (kStats) c_in += 1;
      }
    }
  }
  if (kStats) {
    flush_counter(p.stats + 4, c_pairs);
    flush_counter(p.stats + 5, c_in);
  }
}

// ---------------------------------------------------------------- X2
__global__ void __launch_bounds__(kThreads)
xs_kernel(const double* __restrict__ norm, const double* __restrict__ binmd, double* __restrict__ xs,
          int64_t n) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const double d = norm[i];
    xs[i] = d > 0.0 ? ddiv(binmd[i], d) : CUDART_NAN;
  }
}

// ---------------------------------------------------------------- instrument table (M1 q_p)
__global__ void pixels_prepare_kernel(const double* __restrict__ dir, const double* __restrict__ solid,
                                      double4* __restrict__ pix, int64_t npix) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < npix; i += stride) {
    // q_p = z - d_p (reading #1): (-d_x, -d_y, 1 - d_z)
    pix[i] = make_double4(-dir[3 * i], -dir[3 * i + 1], dsub(1.0, dir[3 * i + 2]), solid[i]);
  }
}

// ---------------------------------------------------------------- parity entry points
struct RecordEmit {
  int64_t* bins;
  double* vals;
  int64_t max;
  int64_t n;
  __device__ __forceinline__ void operator()(int64_t b, double val) {
    if (n < max) {
      bins[n] = b;
      vals[n] = val;
    }
    ++n;
  }
};

__global__ void __launch_bounds__(kThreads)
debug_traj_kernel(const __grid_constant__ MdnParams p, const __grid_constant__ MatBlock mb,
                  int64_t ntraj, const int64_t* ids, int64_t npix, int32_t* n_cross, int32_t* n_seg,
                  int64_t* seg_bins, double* seg_vals, int64_t max_segs) {
  __shared__ double sM[kMaxMats * 9];
  __shared__ double sC[kMaxMats];
  stage_mdnorm_mats(mb, sM, sC);
  __syncthreads();
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= ntraj) return;
  const int64_t id = ids[t];
  const int m = (int)(id / npix);
  const int64_t pi = id - (int64_t)m * npix;
  const double4 px = p.pix[pi];
  const double* M = sM + 9 * m;
  double v[3] = {row_dot(M, px.x, px.y, px.z), row_dot(M + 3, px.x, px.y, px.z),
                 row_dot(M + 6, px.x, px.y, px.z)};
  double kin, kout;
  if (!traj_clip(p.g, v, p.kmin, p.kmax, kin, kout)) {
    n_cross[t] = 0;
    n_seg[t] = 0;
    return;
  }
  const FluxView fx{p.flux_k, p.flux_F, p.nflux};
  RecordEmit rec{seg_bins + t * max_segs, seg_vals + t * max_segs, max_segs, 0};
  int nc;
  n_seg[t] = traj_walk(p.g, fx, v, kin, kout, dmul(px.w, sC[m]), rec, &nc);
  n_cross[t] = nc;
}

__global__ void __launch_bounds__(kThreads)
debug_bins_kernel(const __grid_constant__ BinParams p, const __grid_constant__ MatBlock mb,
                  int64_t* bins) {
  __shared__ double sN[kMaxMats * 9];
  stage_binmd_mats(mb, sN);
  __syncthreads();
  const int64_t total = p.nevents * mb.nmat;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const int m = (int)(t / p.nevents);
    const int64_t e = t - (int64_t)m * p.nevents;
    const float* ev = p.events + e * p.stride;
    bins[t] = event_bin(p.g, sN + 9 * m, (double)ev[p.col_q], (double)ev[p.col_q + 1],
                        (double)ev[p.col_q + 2]);
  }
}

__global__ void debug_compose_kernel(const __grid_constant__ MatBlock mdn,
                                     const __grid_constant__ MatBlock bin, double* M, double* N,
                                     int32_t* ok) {
  for (int m = threadIdx.x; m < mdn.nmat; m += blockDim.x) {
    const int r = m / mdn.nops, s = m - r * mdn.nops;
    if (!compose_mdnorm(mdn.u.c.R + 9 * r, mdn.UB, mdn.u.c.ops + 9 * s, mdn.W, M + 9 * m)) ok[0] = 0;
  }
  for (int m = threadIdx.x; m < bin.nmat; m += blockDim.x)
    if (!compose_binmd(bin.UB, bin.u.c.ops + 9 * m, bin.W, N + 9 * m)) ok[0] = 0;
}

int grid_for(int64_t work, int num_sms, int per_sm) {
  int64_t blocks = (work + kThreads - 1) / kThreads;
  blocks = std::min<int64_t>(blocks, (int64_t)num_sms * per_sm);
  return (int)std::max<int64_t>(blocks, 1);
}

}  // namespace

cudaError_t launch_pixels_prepare(const double* dir, const double* solid, double4* pix, int64_t npix,
                                  cudaStream_t s) {
  pixels_prepare_kernel<<<grid_for(npix, 148, 8), kThreads, 0, s>>>(dir, solid, pix, npix);
  return cudaGetLastError();
}

template <bool kSmemFlux, bool kStats>
cudaError_t launch_mdnorm_t(const MdnParams& p, const MatBlock& mb, int num_sms, size_t smem, cudaStream_t s) {
  cudaError_t err = cudaFuncSetAttribute(mdnorm_kernel<kSmemFlux, kStats>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  mdnorm_kernel<kSmemFlux, kStats><<<grid_for(p.nshard, num_sms, 8), kThreads, smem, s>>>(p, mb);
  return cudaGetLastError();
}

cudaError_t launch_mdnorm(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.nshard <= 0 || mb.nmat <= 0) return cudaSuccess;
  const bool smem_flux = p.nflux <= kFluxSmemMax;
  const size_t smem = sizeof(double) * (10 * (size_t)mb.nmat + (smem_flux ? 2 * (size_t)p.nflux : 0));
  if (smem_flux)
    return p.stats ? launch_mdnorm_t<true, true>(p, mb, num_sms, smem, s)
                   : launch_mdnorm_t<true, false>(p, mb, num_sms, smem, s);
  return p.stats ? launch_mdnorm_t<false, true>(p, mb, num_sms, smem, s)
                 : launch_mdnorm_t<false, false>(p, mb, num_sms, smem, s);
}

cudaError_t launch_binmd(const BinParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.nevents <= 0 || mb.nmat <= 0) return cudaSuccess;
  const bool packed = p.stride == 4 && p.col_w == 0 && p.col_q == 1 &&
                      (reinterpret_cast<uintptr_t>(p.events) & 15) == 0;
  const int blocks = grid_for(p.nevents, num_sms, 8);
  if (packed) {
    if (p.stats) binmd_kernel<true, true><<<blocks, kThreads, 0, s>>>(p, mb);
    else binmd_kernel<true, false><<<blocks, kThreads, 0, s>>>(p, mb);
  } else {
    if (p.stats) binmd_kernel<false, true><<<blocks, kThreads, 0, s>>>(p, mb);
    else binmd_kernel<false, false><<<blocks, kThreads, 0, s>>>(p, mb);
  }
  return cudaGetLastError();
}

cudaError_t launch_cross_section(const double* norm, const double* binmd, double* xs, int64_t nbins,
                                 int num_sms, cudaStream_t s) {
  xs_kernel<<<grid_for(nbins, num_sms, 8), kThreads, 0, s>>>(norm, binmd, xs, nbins);
  return cudaGetLastError();
}

cudaError_t launch_debug_traj(const MdnParams& p, const MatBlock& mb, int64_t ntraj,
                              const int64_t* ids, int64_t npix, int32_t* n_cross, int32_t* n_seg,
                              int64_t* seg_bins, double* seg_vals, int64_t max_segs, cudaStream_t s) {
  if (ntraj <= 0) return cudaSuccess;
  const int blocks = (int)((ntraj + kThreads - 1) / kThreads);
  debug_traj_kernel<<<blocks, kThreads, 0, s>>>(p, mb, ntraj, ids, npix, n_cross, n_seg, seg_bins,
                                                seg_vals, max_segs);
  return cudaGetLastError();
}

cudaError_t launch_debug_bins(const BinParams& p, const MatBlock& mb, int64_t* bins, cudaStream_t s) {
  if (p.nevents <= 0) return cudaSuccess;
  debug_bins_kernel<<<grid_for(p.nevents * mb.nmat, 148, 8), kThreads, 0, s>>>(p, mb, bins);
  return cudaGetLastError();
}

cudaError_t launch_debug_compose(const MatBlock& mdn, const MatBlock& bin, double* M, double* N,
                                 int32_t* ok, cudaStream_t s) {
  debug_compose_kernel<<<1, kThreads, 0, s>>>(mdn, bin, M, N, ok);
  return cudaGetLastError();
}

}  // namespace mdn
