// mdn_kernels.cu -- sm_100a kernels of the MDNorm / BinMD cross-section hot path.
//
// Rows of SURVEY.md §8(a):
//   M0 compose        prologue of mdnorm_cull_kernel / debug kernels (matrices in smem)
//   M1-M3 (cull)      mdnorm_cull_kernel: one thread per trajectory (pixel x op x run): v, clip,
//                     per-axis crossing ranges; hitters are compacted (warp ballot + one atomic
//                     per warp) into a hitter list with their piece plan
//   M3-M7 (walk)      mdnorm_walk_kernel: persistent warps claim batches of 32 hitters, cut them
//                     into pieces of ~kPieceSegs segments at crossings of the busiest axis, and
//                     every lane walks one piece (streaming 3-way merge, flux from smem, midpoint
//                     bin, fp64 red.add into the L2-resident histogram)
//   B0-B3             binmd_kernel (compose prologue, streaming event loads, ops in smem)
//   X2                xs_kernel
// The parity entry points (debug_*) run the very same device functions (mdn_device.cuh).
#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "mdn_kernels.cuh"
#include "mdn_walk.cuh"

namespace mdn {

#if MDN_WALK_TRACE
__device__ unsigned long long g_walk_trace[4 * 148 * 32];  // timing experiment (per walk warp)
#endif

namespace {

// One persistent walk CTA per SM (the shared-memory flux table takes up to 196 KB): 1024
// threads for 2-D slices (64 registers: measured 1024 > 896 > 768 on the CORELLI slab), 768 for
// 3-D grids (the unrolled walk needs more registers).
#ifndef MDN_WALK_THREADS
#define MDN_WALK_THREADS 1024
#endif
#ifndef MDN_WALK_THREADS_3D
#define MDN_WALK_THREADS_3D 768
#endif
#ifndef MDN_WALK_MINB
#define MDN_WALK_MINB 1
#endif
// walk warps claim hitters kWalkChunk at a time into a per-warp ring of kWalkRing entries
#ifndef MDN_WALK_CHUNK
#define MDN_WALK_CHUNK 8
#endif
constexpr int kWalkChunk = MDN_WALK_CHUNK;
// the last MDN_WALK_SPLIT_TAIL hitters per warp are cut into MDN_WALK_SPLIT x more pieces
#ifndef MDN_WALK_SPLIT
#define MDN_WALK_SPLIT 2
#endif
#ifndef MDN_WALK_SPLIT_TAIL
#define MDN_WALK_SPLIT_TAIL 4  // measured: 4 > 8 > 16 > 32 (-1% CORELLI walk at 4), split 4 slower
#endif
#ifndef MDN_WALK_TRACE
#define MDN_WALK_TRACE 0  // timing experiment: per-warp start / first round / end timestamps
#endif
#ifndef MDN_WALK_STATIC_PCT
#define MDN_WALK_STATIC_PCT 60  // % of a launch's hitters in static per-CTA blocks
#endif
#ifndef MDN_WALK_STATIC_CHUNK
#define MDN_WALK_STATIC_CHUNK 32  // hitters per claim from the CTA's block
#endif
// claims shrink to kWalkChunk hitters once fewer than MDN_WALK_TAIL x 32 hitters per warp remain
#ifndef MDN_WALK_TAIL
#define MDN_WALK_TAIL 4
#endif
// claimed hitters sorted by piece length before they enter the warp's queue
#ifndef MDN_WALK_SORT
#define MDN_WALK_SORT 1
#endif
#ifndef MDN_BINMD_WAGG
#define MDN_BINMD_WAGG 0  // warp-aggregated BinMD reductions (measured 1.3-1.9x slower: off)
#endif
#ifndef MDN_WALK_WAGG
#define MDN_WALK_WAGG 0  // warp-aggregated walk reductions (measured 1.4-1.75x slower: off)
#endif
#ifndef MDN_BINMD_CT
#define MDN_BINMD_CT 1  // class test rows gathered per class (BinMD -3%)
#endif
#ifndef MDN_BINMD_MINB
#define MDN_BINMD_MINB 4  // resident 256-thread CTAs per SM (caps registers at 64)
#endif
// auto privatisation of the walk: trajectories per (bin x CTA) of the flush (3-D grids; x16 for 2-D)
#ifndef MDN_PRIV_TRAJ_PER_BIN
#define MDN_PRIV_TRAJ_PER_BIN 1
#endif
constexpr int kWalkRing = 64;  // >= 31 + the largest claim (32), a power of two
static_assert(kWalkChunk >= 1 && kWalkChunk <= 32, "walk claim size");
constexpr int kThreads = 256;
constexpr int walk_threads(bool k3D) { return k3D ? MDN_WALK_THREADS_3D : MDN_WALK_THREADS; }
constexpr unsigned kFull = 0xffffffffu;

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

#ifdef MDN_BINMD_BOX
// Warp min / max of a float with one REDUX each: IEEE floats compare like the signed integers
// i ^ ((i >> 31) & 0x7fffffff) (an involution), and __reduce_{min,max}_sync reduce ints.
__device__ __forceinline__ int float_key(float f) {
  const int i = __float_as_int(f);
  return i ^ ((i >> 31) & 0x7fffffff);
}
__device__ __forceinline__ float warp_min(float f) {
  return __int_as_float(float_key(__int_as_float(__reduce_min_sync(0xffffffffu, float_key(f)))));
}
__device__ __forceinline__ float warp_max(float f) {
  return __int_as_float(float_key(__int_as_float(__reduce_max_sync(0xffffffffu, float_key(f)))));
}
#endif

// One warp-aggregated atomic per counter per warp (tracing only; compiled out when kStats off).
__device__ __forceinline__ void flush_counter(unsigned long long* dst, unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(kFull, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}

// h[b] += v (and h2[b] += v2 when two); with kAgg warp-aggregated: the converged lanes that add
// to the same bin (events of one Bragg peak arrive together in the MDBox/Morton order) are
// summed with shuffles and their lowest lane makes the single reduction (S§2.8 G3; north_star
// "warp-aggregated atomics").  Only the order of the additions changes.  Measured on this B200
// (DESIGN.md §9): __match_any_sync + the shuffles cost more than the same-address reductions
// they save -- BinMD 2x slower on the Morton-ordered CORELLI events, 1.8x on TOPAZ 48 ops, 1.6x
// into a private shared-memory grid; the walk 1.4-1.75x -- so both switches are off.
template <bool kAgg, typename T>
__device__ __forceinline__ void agg_add(T* h, T* h2, int b, T v, T v2, bool two) {
  if constexpr (kAgg) {
    const unsigned act = __activemask();
    const unsigned peers = __match_any_sync(act, b);
    const int lane = threadIdx.x & 31;
    const int most = (int)__reduce_max_sync(act, (unsigned)__popc(peers));
    if (most > 1) {
      unsigned rest = peers & ~(1u << lane);  // the other lanes of this lane's bin
      for (int r = 1; r < most; ++r) {
        const int src = rest ? __ffs(rest) - 1 : lane;
        const T o = __shfl_sync(act, v, src);
        const T o2 = two ? __shfl_sync(act, v2, src) : T(0);
        if (rest) {
          v += o;
          v2 += o2;
          rest &= rest - 1u;
        }
      }
    }
    if (lane != __ffs(peers) - 1) return;
  }
  atomicAdd(h + b, v);
  if (two) atomicAdd(h2 + b, v2);
}

// Shared-memory privatised histogram (S§2.8 G2/G3): T = double (MDN_ACC_F64) or float
// (MDN_ACC_F32 partials); flushed into the fp64 global histogram at the end of the kernel.
template <typename T>
struct SmemEmit {
  T* h;
  __device__ __forceinline__ void operator()(int b, double val) const {
    agg_add<MDN_WALK_WAGG != 0, T>(h, nullptr, b, (T)val, T(0), false);
  }
};

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
    if (v != T(0)) atomicAdd(dst + i, (double)v);
  }
}

// kPriv: 0 = global fp64 red.add, 1 = fp64 shared-memory partials, 2 = fp32 shared-memory partials
template <int kPriv>
using priv_t = typename std::conditional<kPriv == 2, float, double>::type;

// bytes of a private histogram of n bins, rounded up to 16
__host__ __device__ constexpr size_t priv_bytes(int kind, int64_t n) {
  return kind == 0 ? 0 : (((size_t)n * (kind == 2 ? 4 : 8) + 15) & ~(size_t)15);
}

struct AtomicEmit {
  double* h;
#ifdef MDN_EXP_NOATOMIC  // timing experiment only: keeps the value alive without the reduction
  __device__ __forceinline__ void operator()(int b, double val) const {
    if (val == -1.2345e300) h[b] = val;
  }
#else
  __device__ __forceinline__ void operator()(int b, double val) const {
    agg_add<MDN_WALK_WAGG != 0, double>(h, nullptr, b, val, 0.0, false);
  }
#endif
};

// Momentum range of a pixel's trajectories: the call's [k_min, k_max], intersected with the
// pixel's own limits when set (Mantid MDNorm_low/high; oracle orc_mdnorm_krange).
__device__ __forceinline__ void pixel_krange(const MdnParams& p, int64_t pixel, double& lo, double& hi) {
  lo = p.kmin;
  hi = p.kmax;
  if (p.pkr) {
    const double2 r = p.pkr[pixel];
    if (r.x > lo) lo = r.x;
    if (r.y < hi) hi = r.y;
  }
}

// ---------------------------------------------------------------- M1-M3: cull + compaction
// One thread per pixel of the slab, looping over every (run, op) matrix of the launch (pixel
// read once; matrices are warp-uniform smem broadcasts).  A conservative fp32 slab test with a
// proven error margin rejects most misses without any fp64 division; every
// survivor gets the exact fp64 v and clip, so the hit decision is the definition's.
// Rows are stored in test order (fewest bins first: the thin axis of a 2-D slice rejects almost
// every trajectory after one row product, so the other two rows are only read when a lane of the
// warp survives it).
struct alignas(16) CullMat {
  float4 a[3];  // test-order axis k: (row of fp32(M), acceptance window low lo - delta)
  float4 hi;    // acceptance window high hi + delta per test-order axis (w unused)
};

template <bool kStats>
__global__ void __launch_bounds__(kThreads, 4)  // 64 registers: four resident CTAs per SM
mdnorm_cull_kernel(const __grid_constant__ MdnParams p, const __grid_constant__ MatBlock mb) {
  extern __shared__ double smem[];
  double* sM = smem;
  double* sC = sM + 9 * mb.nmat;
  CullMat* sF = reinterpret_cast<CullMat*>(sC + mb.nmat);
  // the walk (launched with programmatic stream serialisation, MDN_PDL_WALK) may start its
  // prologue on SMs this one-wave grid leaves; it waits for this grid before reading hitters
  asm volatile("griddepcontrol.launch_dependents;");
  stage_mdnorm_mats(mb, sM, sC);
  __syncthreads();
  // test order: fewest bins first (stable)
  int ord[3] = {0, 1, 2};
  if (p.g.n[ord[1]] < p.g.n[ord[0]]) { const int t = ord[0]; ord[0] = ord[1]; ord[1] = t; }
  if (p.g.n[ord[2]] < p.g.n[ord[1]]) { const int t = ord[1]; ord[1] = ord[2]; ord[2] = t; }
  if (p.g.n[ord[1]] < p.g.n[ord[0]]) { const int t = ord[0]; ord[0] = ord[1]; ord[1] = t; }
  for (int m = threadIdx.x; m < mb.nmat; m += blockDim.x) {
    float hi[3];
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      const int a = ord[k];
      const double* row = sM + 9 * m + 3 * a;
      const double sum = fabs(row[0]) + fabs(row[1]) + fabs(row[2]);
      // |q_i| <= 2; fp32 v and x = k v are within 1e-6 kmax sum|M_a| of the exact values
      const double delta = 4e-6 * p.kmax * sum + 1e-6 * (fabs(p.g.lo[a]) + fabs(p.g.hi[a])) + 1e-30;
      sF[m].a[k] = make_float4((float)row[0], (float)row[1], (float)row[2], (float)p.g.lo[a] - (float)delta);
      hi[k] = (float)p.g.hi[a] + (float)delta;
    }
    sF[m].hi = make_float4(hi[0], hi[1], hi[2], 0.f);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  // per-warp ring of fp32 survivors (pixel offset, matrix); the exact fp64 path runs only when
  // 32 of them are queued, so it executes with the whole warp converged
  uint32_t* qoff = reinterpret_cast<uint32_t*>(sF + mb.nmat) + (threadIdx.x >> 5) * 128;
  uint32_t* qmat = qoff + 64;
  int qhead = 0, qcnt = 0;
  unsigned long long c_traj = 0, c_hit = 0, c_cross = 0;

  // exact M1-M3 for queued candidates [qhead, qhead + n) (n <= 32), hitters appended
  auto drain = [&](int n) {
    __syncwarp();
    bool hit = false;
    Hitter h;
    if (lane < n) {
      const int slot = (qhead + lane) & 63;
      const uint32_t off = qoff[slot], m = qmat[slot];
      const int64_t pixel = p.pix_begin + (int64_t)(p.p0 + off) * p.pix_stride;
      const double4 px = p.pix[pixel];
      double klo, khi;
      pixel_krange(p, pixel, klo, khi);
      {
        const double* M = sM + 9 * m;
        const double v0 = row_dot(M, px.x, px.y, px.z);
        const double v1 = row_dot(M + 3, px.x, px.y, px.z);
        const double v2 = row_dot(M + 6, px.x, px.y, px.z);
        const double vv[3] = {v0, v1, v2};
        double kin, kout;
        // one reciprocal per axis serves the clip and the crossing ranges (the same RN(1/v))
        const double rr[3] = {v0 != 0.0 ? ddiv(1.0, v0) : 0.0, v1 != 0.0 ? ddiv(1.0, v1) : 0.0,
                              v2 != 0.0 ? ddiv(1.0, v2) : 0.0};
        // a non-finite v (only from a singular composition) contributes nothing in the oracle
        if (isfinite(v0) && isfinite(v1) && isfinite(v2) && traj_clip_r(p.g, vv, rr, klo, khi, kin, kout)) {
          hit = true;
          const AxisStream s0 = axis_stream(p.g, 0, v0, rr[0], kin, kout);
          const AxisStream s1 = axis_stream(p.g, 1, v1, rr[1], kin, kout);
          const AxisStream s2 = axis_stream(p.g, 2, v2, rr[2], kin, kout);
          const int total = s0.cnt + s1.cnt + s2.cnt;
          // piece plan: cut at crossings of the busiest axis A, ~kPieceSegs segments per piece
          const bool a1 = s1.cnt > s0.cnt;
          const AxisStream s01 = a1 ? s1 : s0;
          const bool a2 = s2.cnt > s01.cnt;
          const AxisStream sa = a2 ? s2 : s01;
          const int A = a2 ? 2 : (a1 ? 1 : 0);
          int P = 1, G = 1;
          const int S = p.g.n[2] > 1 ? kPieceSegs3D : kPieceSegs;
          if (total + 1 > S && sa.cnt > 1) {
            // G crossings of A per piece bring ~G (total + 1) / cA segments: aim at S
            G = max(1, (S * sa.cnt + (total + 1) / 2) / (total + 1));
            P = (sa.cnt + G - 1) / G;
          }
          h.v0 = v0; h.v1 = v1; h.v2 = v2; h.kin = kin; h.kout = kout;
          h.oc = dmul(px.w, sC[m]);
          // busiest axis | flux table << 2 | min(segments per piece, 1023) << 22 (walk sort key)
          const int plen = min((total + P) / P, 1023);
          h.A = A | ((p.ptab ? p.ptab[pixel] : 0) << 2) | (plen << 22);
#if MDN_PIECE_BALANCED
          // cuts at crossings floor(p cA / P) of axis A (p = 1 .. P-1): the crossings of every axis
          // are equally spaced in k, so the P pieces get equal segment counts (no short remainder)
          h.jA = sa.j; h.stepG = sa.step * sa.cnt; h.P = P;
#else
          h.jA = sa.j; h.stepG = sa.step * G; h.P = P;
#endif
          if (kStats) {
            c_hit += 1;
            c_cross += total;
          }
        }
      }
    }
    const unsigned ballot = __ballot_sync(kFull, hit);
    if (ballot) {
      unsigned idx = 0;
      if (lane == 0) idx = atomicAdd(&p.ctr->nhit, (unsigned)__popc(ballot));
      idx = __shfl_sync(kFull, idx, 0);
      if (hit) p.hit[idx + __popc(ballot & ((1u << lane) - 1u))] = h;
    }
    qhead = (qhead + n) & 63;
    qcnt -= n;
    __syncwarp();
  };

  // warps claim 32 pixels at a time from a global cursor (the hit fraction varies strongly over
  // the detector, so a static split leaves a tail of busy warps); loops are warp-uniform so the
  // ballots below always have the full warp
  for (;;) {
    uint32_t base = 0;
    if (lane == 0) base = atomicAdd(&p.ctr->pclaim, 32u);
    base = __shfl_sync(kFull, base, 0);
    if (base >= p.plen) break;
    const uint32_t off = base + lane;
    const bool valid = off < p.plen;
    double4 px = make_double4(0.0, 0.0, 0.0, 0.0);
    double klo = p.kmin, khi = p.kmax;
    if (valid) {
      const int64_t pixel = p.pix_begin + (int64_t)(p.p0 + off) * p.pix_stride;
      px = p.pix[pixel];
      pixel_krange(p, pixel, klo, khi);
    }
    if (kStats && valid) c_traj += mb.nmat;
    // masked pixels contribute 0 (reading #16); an empty per-pixel k range contributes 0
    const bool live = valid && px.w != 0.0 && klo < khi;
    const float q0 = (float)px.x, q1 = (float)px.y, q2 = (float)px.z;
    const float kmin32 = (float)klo, kmax32 = (float)khi;
    if (!__any_sync(kFull, live)) continue;
    for (int m = 0; m < mb.nmat; ++m) {
      const CullMat* cm = sF + m;
      const float4 hw = cm->hi;
      bool maybe = live;
      {  // the most selective axis first
        const float4 r = cm->a[0];
        const float v = fmaf(r.z, q2, fmaf(r.y, q1, r.x * q0));
        const float xa = kmin32 * v, xb = kmax32 * v;
        maybe &= (fmaxf(xa, xb) >= r.w) & (fminf(xa, xb) < hw.x);
      }
      if (__any_sync(kFull, maybe)) {
#pragma unroll
        for (int k = 1; k < 3; ++k) {
          const float4 r = cm->a[k];
          const float v = fmaf(r.z, q2, fmaf(r.y, q1, r.x * q0));
          const float xa = kmin32 * v, xb = kmax32 * v;
          maybe &= (fmaxf(xa, xb) >= r.w) & (fminf(xa, xb) < (k == 1 ? hw.y : hw.z));
        }
        const unsigned mask = __ballot_sync(kFull, maybe);
        if (maybe) {
          const int slot = (qhead + qcnt + __popc(mask & ((1u << lane) - 1u))) & 63;
          qoff[slot] = off;
          qmat[slot] = (uint32_t)m;
        }
        qcnt += __popc(mask);
        if (qcnt >= 32) drain(32);
      }
    }
  }
  if (qcnt > 0) drain(qcnt);
  if (kStats) {
    flush_counter(p.stats + 0, c_traj);
    flush_counter(p.stats + 1, c_hit);
    flush_counter(p.stats + 2, c_cross);
  }
}

// ---------------------------------------------------------------- M3-M7: balanced piece walk
// kFlux: 0 = one flux table read from global memory, 1 = one table staged in shared memory,
// 2 = per-bank tables (pixel -> table map, NEXT #1) read from global memory
template <int kFlux, bool kStats, bool k3D, int kPriv>
__global__ void __launch_bounds__(walk_threads(k3D), MDN_WALK_MINB)
mdnorm_walk_kernel(const __grid_constant__ MdnParams p) {
  constexpr bool kSmemFlux = kFlux == 1;
  using PT = priv_t<kPriv>;
  extern __shared__ double4 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  // shared layout: private histogram (kPriv, 16-byte rounded) | interval records ka, kb (n
  // double2 each) | knots (n + 2, even) | cell table (uint16, even) | per-warp prefix sums (32
  // int) | per-warp hitter rings (kWalkRing unsigned)
  PT* sHist = reinterpret_cast<PT*>(wsm);
  if (kPriv) priv_zero(sHist, p.g.nbins);
  const int n_rec = kSmemFlux ? p.flux.n : 0;
  const int n_kn = kSmemFlux && !MDN_FLUX_NOKN ? (p.flux.n + 3) & ~1 : 0;
  double2* sKa = reinterpret_cast<double2*>(reinterpret_cast<char*>(wsm) + priv_bytes(kPriv, p.g.nbins));
  double2* sKb = sKa + n_rec;
  double* sKn = reinterpret_cast<double*>(sKb + n_rec);
  uint16_t* sTab = reinterpret_cast<uint16_t*>(sKn + n_kn);
  int* sPre = reinterpret_cast<int*>(sTab + (kSmemFlux ? (p.flux.ntab + 1) & ~1 : 0));
  unsigned* sRing = reinterpret_cast<unsigned*>(sPre + 32 * nwarps);
  if (kSmemFlux) {
    for (int i = threadIdx.x; i < p.flux.n; i += blockDim.x) {
      sKa[i] = p.flux.ka[i];
      sKb[i] = p.flux.kb[i];
    }
    if (!MDN_FLUX_NOKN)
      for (int i = threadIdx.x; i < p.flux.n + 2; i += blockDim.x) sKn[i] = p.flux.kn[i];
    const int* gtab = static_cast<const int*>(p.flux.tab);
    for (int i = threadIdx.x; i < p.flux.ntab; i += blockDim.x) {
      const unsigned e = (unsigned)gtab[i];
      sTab[i] = (uint16_t)((e & (kFluxDense32 - 1)) | ((e & kFluxDense32) ? kFluxDense16 : 0u));
    }
  }
  __shared__ unsigned sCur;  // claims taken from this CTA's static block of hitters
  if (threadIdx.x == 0) sCur = 0;
  __syncthreads();
#if MDN_WALK_TRACE
  unsigned long long tr_t0 = 0, tr_first = 0, tr_rounds = 0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr_t0));
#endif
  FluxView fx = p.flux;
  if (kSmemFlux) {
    if (!MDN_FLUX_NOKN) fx.kn = sKn;  // else the rare general path bisects the global knots
    fx.ka = sKa;
    fx.kb = sKb;
    fx.tab = sTab;
  }
  int* pre = sPre + 32 * warp;
  typename std::conditional<kPriv != 0, SmemEmit<PT>, AtomicEmit>::type emit;
  if constexpr (kPriv != 0) emit.h = sHist;
  else emit.h = p.norm;
  // everything above (flux staging, private histogram zeroing) overlaps the cull's tail under
  // programmatic dependent launch; the hitter list and count are read only after the cull
  // grid has completed.  No-op without the attribute.
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const unsigned nhit = *(volatile unsigned*)&p.ctr->nhit;
  unsigned long long c_seg = 0;
  // Per-warp queue of hitters (ring of kWalkRing indices; the head hitter may be partly
  // consumed: `skip` of its pieces are done) holding `qpieces` pieces.  Each round hands the next
  // 32 pieces of the queue to the 32 lanes, which walk them to completion together (so the piece
  // set-up -- divisions, per-axis ranges, first flux look-up -- runs converged).  The queue is
  // topped up by claiming kWalkChunk hitters at a time from the global cursor, so rounds are full
  // across hitter boundaries and the end-of-kernel imbalance is one small chunk.
  unsigned* ring = sRing + 2 * kWalkRing * warp;  // hitter indices
  int* ringP = reinterpret_cast<int*>(ring + kWalkRing);  // their piece counts
  unsigned head = 0, nq = 0;
  int skip = 0, qpieces = 0;
  bool more = true;
  const unsigned tail = (unsigned)MDN_WALK_TAIL * 32u * gridDim.x * (unsigned)nwarps;
  unsigned chunk = nhit > tail ? 32u : (unsigned)kWalkChunk;
  // static per-CTA blocks of hitters cover MDN_WALK_STATIC_PCT % of them; [rest, nhit) is dynamic
  // (only for launches small enough to claim in small chunks from the start: with 32-hitter
  // claims the global counter is not contended, and static blocks unbalance 3-D walks)
  const unsigned blk_n =
      nhit > tail ? 0u : (unsigned)(((unsigned long long)nhit * MDN_WALK_STATIC_PCT / 100) / gridDim.x);
  const unsigned blk = blockIdx.x * blk_n, rest = blk_n * gridDim.x;
  constexpr int kStaticChunk = MDN_WALK_STATIC_CHUNK;
  bool sdone = false;  // lane 0: this CTA's block is used up
  const unsigned split_tail = (unsigned)MDN_WALK_SPLIT_TAIL * gridDim.x * (unsigned)nwarps;
  (void)split_tail;
  for (;;) {
    while (qpieces < 32 && more) {
      // Claims come first from this CTA's static block of hitters (a shared-memory atomic), then
      // from the launch's remaining hitters (one global atomic): the block keeps the 4736 warps
      // from queueing on one global counter (at the start every warp claims at once, measured
      // 10 us before the last warp's first round), the global remainder balances the CTAs.
      unsigned b = 0, n = 0;
      if (lane == 0) {
        const unsigned o = sdone ? blk_n : atomicAdd(&sCur, (unsigned)kStaticChunk);
        if (o < blk_n) {
          b = blk + o;
          n = min((unsigned)kStaticChunk, blk_n - o);
        } else {
          sdone = true;
          b = rest + atomicAdd(&p.ctr->claimed, chunk);
          n = chunk;
        }
      }
      b = __shfl_sync(kFull, b, 0);
      n = __shfl_sync(kFull, n, 0);
      if (b >= nhit) {
        more = false;
        // this warp claims nothing more: once every warp of every CTA is here (the start of the
        // end spread) a BinMD launched with programmatic stream serialisation may take the SMs
        // that walk CTAs leave
        asm volatile("griddepcontrol.launch_dependents;");
        break;
      }
      const unsigned nnew = min(n, nhit - b);
      // large claims (hitter locality, fewer atomics) until the last few claims per warp, then
      // small ones so that the warps finish together
      if (b >= rest) chunk = nhit - b > tail ? 32u : (unsigned)kWalkChunk;
      int P = 0;
#if MDN_WALK_SORT
      // Claimed hitters enter the queue longest pieces first (warp bitonic sort on the piece
      // length the cull stored), so that a round's 32 pieces have similar lengths and its lanes
      // finish together.  Key = length << 5 | lane: unique, invalid lanes (0) last.
      int A = 0;
      if ((unsigned)lane < nnew) {
        const int4 t = *reinterpret_cast<const int4*>(&p.hit[b + lane].A);  // (A, jA, stepG, P)
        A = t.x;
        P = t.w;
#if MDN_PIECE_BALANCED && MDN_WALK_SPLIT > 1
        // the last hitters of the launch are cut into MDN_WALK_SPLIT times more (shorter) pieces
        // at crossings of the same axis, so that the final rounds -- and the kernel -- end sooner
        if (nhit - b <= split_tail) P = max(P, min(abs(t.z), P * MDN_WALK_SPLIT));
#endif
      }
      unsigned key = (unsigned)lane < nnew ? ((((unsigned)A >> 22) + 1u) << 5) | (unsigned)lane : 0u;
#pragma unroll
      for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
          const unsigned o = __shfl_xor_sync(kFull, key, j);
          const bool desc = (lane & k) == 0 || k == 32;  // final merge: descending
          const bool low = (lane & j) == 0;
          key = (low == desc) ? max(key, o) : min(key, o);
        }
      }
      const int src = key & 31;
      P = __shfl_sync(kFull, P, src);
      if ((unsigned)lane >= nnew) P = 0;
      if ((unsigned)lane < nnew) {
        ring[(head + nq + lane) & (kWalkRing - 1)] = b + src;
        ringP[(head + nq + lane) & (kWalkRing - 1)] = P;
      }
#else
      if ((unsigned)lane < nnew) {
        P = p.hit[b + lane].P;
        ring[(head + nq + lane) & (kWalkRing - 1)] = b + lane;
        ringP[(head + nq + lane) & (kWalkRing - 1)] = P;
      }
#endif
      nq += nnew;
      qpieces += __reduce_add_sync(kFull, P);
      __syncwarp();
    }
    if (qpieces == 0) break;
#if MDN_WALK_TRACE
    if (tr_rounds++ == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr_first));
#endif
    // pieces of the first (up to) 32 queued hitters: inclusive scan of their remaining counts
    const bool inq = (unsigned)lane < nq;
    int incl = inq ? ringP[(head + lane) & (kWalkRing - 1)] - (lane == 0 ? skip : 0) : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    pre[lane] = incl;
    __syncwarp();
    const int nr = min(qpieces, 32);
    unsigned myh = 0;
    int mypi = 0, myP = 1;
    if (lane < nr) {
      int l = 0;  // owner: first queued hitter l with pre[l] > lane
#pragma unroll
      for (int s = 16; s > 0; s >>= 1)
        if (pre[l + s - 1] <= lane) l += s;
      myh = ring[(head + l) & (kWalkRing - 1)];
      myP = ringP[(head + l) & (kWalkRing - 1)];  // the piece count this hitter was queued with
      mypi = lane - (l ? pre[l - 1] : 0) + (l == 0 ? skip : 0);
    }
    // advance the queue past the nr pieces handed out
    const int k = __popc(__ballot_sync(kFull, inq && incl <= nr));  // hitters fully consumed
    const int kpre = k ? __shfl_sync(kFull, incl, (k - 1) & 31) : 0;
    skip = k ? nr - kpre : skip + nr;
    head += k;
    nq -= k;
    qpieces -= nr;
    __syncwarp();
    if (lane < nr) {
      const Hitter& h = p.hit[myh];
      const double v0 = h.v0, v1 = h.v1, v2 = h.v2;
      const int A = h.A & 3;
      double lo_k = h.kin, hi_k = h.kout;
      if (myP > 1) {
        const double vA = A == 0 ? v0 : (A == 1 ? v1 : v2);
        const double rA = ddiv(1.0, vA);
#if MDN_PIECE_BALANCED
        const int cA = abs(h.stepG), st = h.stepG < 0 ? -1 : 1;
        if (mypi > 0) lo_k = plane_k(p.g, A, h.jA + st * ((mypi * cA) / myP), rA);
        if (mypi < myP - 1) hi_k = plane_k(p.g, A, h.jA + st * (((mypi + 1) * cA) / myP), rA);
#else
        if (mypi > 0) lo_k = plane_k(p.g, A, h.jA + mypi * h.stepG, rA);
        if (mypi < myP - 1) hi_k = plane_k(p.g, A, h.jA + (mypi + 1) * h.stepG, rA);
#endif
      }
      int nc;
      int ns;
      if (kFlux == 1) {
        ns = traj_walk<k3D, uint16_t>(p.g, fx, v0, v1, v2, lo_k, hi_k, h.oc, emit, &nc);
      } else if (kFlux == 2) {
        const FluxView fv = p.fviews[(h.A >> 2) & 0xFFFFF];
        ns = traj_walk<k3D, int>(p.g, fv, v0, v1, v2, lo_k, hi_k, h.oc, emit, &nc);
      } else {
        ns = traj_walk<k3D, int>(p.g, fx, v0, v1, v2, lo_k, hi_k, h.oc, emit, &nc);
      }
      if (kStats) c_seg += ns;
    }
    __syncwarp();
  }
  if (kPriv) {
    __syncthreads();
    priv_flush(sHist, p.norm, p.g.nbins);
  }
#if MDN_WALK_TRACE
  if (lane == 0) {
    unsigned long long t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    unsigned long long* o = g_walk_trace + 4 * ((size_t)blockIdx.x * nwarps + warp);
    o[0] = tr_t0;
    o[1] = tr_first;
    o[2] = t1;
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    o[3] = tr_rounds | ((unsigned long long)smid << 32);
  }
#endif
  if (kStats) flush_counter(p.stats + 3, c_seg);
}

// ---------------------------------------------------------------- B1-B3: one thread per event
// fp32 fast path with a proven error bound: per (op, axis) the grid coordinate
// t = x s - lo s is evaluated in fp32; |t32 - t64| < delta = c |q|max + d.  A pair whose t32 is
// further than delta from every decision point (0, n and the integer bin edges) has exactly
// the bin the fp64 definition gives; the rest (a ~1e-4 fraction) take the exact fp64 path.
// Axes are tested in the order p.ord (fewest bins first: the thin L axis of a 2-D slice rejects
// almost every pair after one row product).
struct BinAxis32 {
  float r0, r1, r2, s, los, c, d, n;
};

// Member loop of one queued (event, class) pair: the remaining two axes of every op of the
// class, bin and fp64 red.add.  Out of line so that its constants are not hoisted into the
// class-test loop.  Returns the number of (event, op) pairs that landed inside the grid.
template <int kPriv>
__device__ __noinline__ unsigned binmd_members(const BinParams& p, const double* sN, const BinAxis32* sA,
                                               const int* sCls, const int* sMem, float4 ev, float e2, int c,
                                               int a0, int a1, priv_t<kPriv>* hb, priv_t<kPriv>* he) {
  const float w = ev.x, q0 = ev.y, q1 = ev.z, q2 = ev.w;
  const float qm = fmaxf(fabsf(q0), fmaxf(fabsf(q1), fabsf(q2)));
  const int j0 = sCls[c], j1 = sCls[c + 1];
  const BinAxis32 ax = sA[3 * sMem[j0]];
  const float x = fmaf(ax.r2, q2, fmaf(ax.r1, q1, ax.r0 * q0));
  const float t = fmaf(x, ax.s, -ax.los);
  const float dl = fmaf(ax.c, qm, ax.d);
  const float fl = floorf(t);
  const float fr = t - fl;
  const bool near0 = t < dl || t > ax.n - dl || fr < dl || fr > 1.0f - dl;
  const int ifirst = (int)fl;
  unsigned inside = 0;
  for (int j = j0; j < j1; ++j) {
    const int m = sMem[j];
    bool out = false, near = near0;
    int ik[3] = {ifirst, 0, 0};
#pragma unroll
    for (int k = 1; k < 3; ++k) {
      const BinAxis32 bx = sA[3 * m + k];
      const float xk = fmaf(bx.r2, q2, fmaf(bx.r1, q1, bx.r0 * q0));
      const float tk = fmaf(xk, bx.s, -bx.los);
      const float dk = fmaf(bx.c, qm, bx.d);
      out = out || tk < -dk || tk >= bx.n + dk;
      const float fk = floorf(tk);
      const float rk = tk - fk;
      near = near || tk < dk || tk > bx.n - dk || rk < dk || rk > 1.0f - dk;
      ik[k] = (int)fk;
    }
    if (out) continue;
    // bin indices back in axis order (ord is a permutation of 0, 1, 2)
    const int i0 = a0 == 0 ? ik[0] : (a1 == 0 ? ik[1] : ik[2]);
    const int i1 = a0 == 1 ? ik[0] : (a1 == 1 ? ik[1] : ik[2]);
    const int i2 = a0 == 2 ? ik[0] : (a1 == 2 ? ik[1] : ik[2]);
    int b;
    if (!near) {
      b = i0 + p.g.n[0] * (i1 + p.g.n[1] * i2);
    } else {  // within the error bound of a decision point: the fp64 definition decides
      const int64_t be = event_bin(p.g, sN + 9 * m, (double)q0, (double)q1, (double)q2);
      if (be < 0) continue;
      b = (int)be;
    }
    if constexpr (kPriv != 0) {
      agg_add<MDN_BINMD_WAGG != 0>(hb, he, b, (priv_t<kPriv>)w, (priv_t<kPriv>)e2, p.col_e >= 0);
    } else {
      agg_add<MDN_BINMD_WAGG != 0>(p.binmd, p.err2, b, (double)w, (double)e2, p.col_e >= 0);
    }
    ++inside;
  }
  return inside;
}

// Block size: 256 threads with global reductions (several CTAs per SM); 512 with a private
// shared-memory histogram (fewer, larger CTAs: the histogram is zeroed and flushed per CTA).
__host__ __device__ constexpr int bin_threads(int kPriv) { return kPriv ? 512 : kThreads; }

template <bool kPacked, bool kStats, int kPriv>
__global__ void __launch_bounds__(bin_threads(kPriv), kPriv ? 2 : MDN_BINMD_MINB)
binmd_kernel(const __grid_constant__ BinParams p, const __grid_constant__ MatBlock mb) {
  constexpr int kBT = bin_threads(kPriv);
  using PT = priv_t<kPriv>;
  __shared__ double sN[kMaxMats * 9];
  __shared__ BinAxis32 sA[kMaxMats * 3];
  // private histograms (kPriv): binmd, then err2 when the error column is read
  extern __shared__ double4 bsm[];
  PT* hb = reinterpret_cast<PT*>(bsm);
  PT* he = reinterpret_cast<PT*>(reinterpret_cast<char*>(bsm) + priv_bytes(kPriv, p.g.nbins));
  if (kPriv) {
    priv_zero(hb, p.g.nbins);
    if (p.col_e >= 0) priv_zero(he, p.g.nbins);
  }
  // the divide after BinMD (launch_cross_section, programmatic dependent launch) may launch now;
  // it waits for this grid to complete before reading either histogram
  asm volatile("griddepcontrol.launch_dependents;");
  stage_binmd_mats(mb, sN);
  __syncthreads();
  for (int i = threadIdx.x; i < 3 * mb.nmat; i += blockDim.x) {
    const int m = i / 3, a = p.ord[i - 3 * m];
    const double* row = sN + 9 * m + 3 * a;
    const double s = p.g.s[a], lo = p.g.lo[a];
    const double sum = fabs(row[0]) + fabs(row[1]) + fabs(row[2]);
    BinAxis32 ax;
    ax.r0 = (float)row[0];
    ax.r1 = (float)row[1];
    ax.r2 = (float)row[2];
    ax.s = (float)s;
    ax.los = (float)(lo * s);
    ax.c = (float)(1e-6 * s * sum);
    ax.d = (float)(1e-6 * s * fabs(lo) + 1e-6 * (p.g.n[a] + 1.0));
    ax.n = (float)p.g.n[a];
    sA[i] = ax;
  }
  __syncthreads();
  // Ops whose first-tested row is the same fp32 vector give the same t on that axis, so the
  // test is done once per class (symmetry ops map L -> +-L: 2 classes for 6/mmm on a slice).
  __shared__ int sRep[kMaxMats], sCid[kMaxMats], sCls[kMaxMats + 1], sMem[kMaxMats];
  __shared__ int sNcls;
  for (int m = threadIdx.x; m < mb.nmat; m += blockDim.x) {
    const BinAxis32 am = sA[3 * m];
    int rep = m;
    for (int r = 0; r < m; ++r) {
      const BinAxis32 ar = sA[3 * r];
      if (ar.r0 == am.r0 && ar.r1 == am.r1 && ar.r2 == am.r2 &&
          __float_as_uint(ar.r0) == __float_as_uint(am.r0) && __float_as_uint(ar.r1) == __float_as_uint(am.r1) &&
          __float_as_uint(ar.r2) == __float_as_uint(am.r2)) {
        rep = r;
        break;
      }
    }
    sRep[m] = rep;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int ncls = 0;
    for (int m = 0; m < mb.nmat; ++m) {
      sCid[m] = sRep[m] == m ? ncls++ : sCid[sRep[m]];
    }
    for (int c = 0; c <= ncls; ++c) sCls[c] = 0;
    for (int m = 0; m < mb.nmat; ++m) sCls[sCid[m] + 1] += 1;
    for (int c = 0; c < ncls; ++c) sCls[c + 1] += sCls[c];
    int fill[kMaxMats];
    for (int c = 0; c < ncls; ++c) fill[c] = sCls[c];
    for (int m = 0; m < mb.nmat; ++m) sMem[fill[sCid[m]]++] = m;
    sNcls = ncls;
  }
  __syncthreads();
  const int ncls = sNcls;
#if MDN_BINMD_CT
  // class test rows gathered by class index (one level of shared-memory indirection less in the
  // per-event class loop)
  __shared__ BinAxis32 sCT[kMaxMats];
  for (int c = threadIdx.x; c < ncls; c += blockDim.x) sCT[c] = sA[3 * sMem[sCls[c]]];
  __syncthreads();
#endif
  const int a0 = p.ord[0], a1 = p.ord[1], a2 = p.ord[2];
  const int lane = threadIdx.x & 31;
  // per-warp queue of (event, class) pairs that pass the class test: their member loop runs
  // only when 32 are queued, with the warp converged
  __shared__ float4 sQv[(kBT / 32) * 64];
  __shared__ int sQc[(kBT / 32) * 64];
  __shared__ float sQe[(kBT / 32) * 64];  // error-squared column (col_e >= 0 only)
  float4* qv = sQv + (threadIdx.x >> 5) * 64;
  int* qc = sQc + (threadIdx.x >> 5) * 64;
  float* qe = sQe + (threadIdx.x >> 5) * 64;
  const bool has_err = !kPacked && p.col_e >= 0;
  int qhead = 0, qcnt = 0;
  unsigned long long c_pairs = 0, c_in = 0;

  (void)a2;
  auto drain = [&](int n) {
    __syncwarp();
    if (lane < n) {
      const int slot = (qhead + lane) & 63;
      c_in += binmd_members<kPriv>(p, sN, sA, sCls, sMem, qv[slot], has_err ? qe[slot] : 0.0f, qc[slot], a0,
                                   a1, hb, he);
    }
    qhead = (qhead + n) & 63;
    qcnt -= n;
    __syncwarp();
  };

  auto load = [&](int64_t e) {
    if (kPacked) return __ldcs(reinterpret_cast<const float4*>(p.events) + e);
    const float* ev = p.events + e * p.stride;
    return make_float4(__ldcs(ev + p.col_w), __ldcs(ev + p.col_q), __ldcs(ev + p.col_q + 1),
                       __ldcs(ev + p.col_q + 2));
  };

  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31);  // warp-uniform
  auto load_e = [&](int64_t e) { return has_err ? __ldcs(p.events + e * p.stride + p.col_e) : 0.0f; };
  float4 cur = make_float4(0.f, 0.f, 0.f, 0.f);
  float cur_e = 0.f;
  if (base + lane < p.nevents) {
    cur = load(base + lane);
    cur_e = load_e(base + lane);
  }
  // the class tests of one event (per-warp queue of passing (event, class) pairs)
  auto test_event = [&](const float4 ev, const float ev_e, const bool valid) {
    const float q0 = ev.y, q1 = ev.z, q2 = ev.w;
    const float qm = fmaxf(fabsf(q0), fmaxf(fabsf(q1), fabsf(q2)));
    if (kStats && valid) c_pairs += mb.nmat;
#ifdef MDN_BINMD_BOX
    // Warp box (S§8(f) NEXT #4, Mantid's MDBox idea on the Morton-ordered stream): the 32
    // events' Q bounding box, transformed by interval arithmetic, rejects a whole class at once
    // when it misses [0, n) on the class axis by more than the fp32 error bound.  Measured
    // slower than the per-event test on the CORELLI slab, so it is off.
    const float b0l = warp_min(valid ? q0 : CUDART_INF_F), b0h = warp_max(valid ? q0 : -CUDART_INF_F);
    const float b1l = warp_min(valid ? q1 : CUDART_INF_F), b1h = warp_max(valid ? q1 : -CUDART_INF_F);
    const float b2l = warp_min(valid ? q2 : CUDART_INF_F), b2h = warp_max(valid ? q2 : -CUDART_INF_F);
    const float bqm = fmaxf(fmaxf(fmaxf(fabsf(b0l), fabsf(b0h)), fmaxf(fabsf(b1l), fabsf(b1h))),
                            fmaxf(fabsf(b2l), fabsf(b2h)));
#endif
    for (int c = 0; c < ncls; ++c) {
      // first-tested axis, once for the whole class
#if MDN_BINMD_CT
      const BinAxis32 ax = sCT[c];
#else
      const BinAxis32 ax = sA[3 * sMem[sCls[c]]];
#endif
#ifdef MDN_BINMD_BOX
      {  // warp-uniform box test
        const float p0a = ax.r0 * b0l, p0b = ax.r0 * b0h, p1a = ax.r1 * b1l, p1b = ax.r1 * b1h;
        const float p2a = ax.r2 * b2l, p2b = ax.r2 * b2h;
        const float xl = fminf(p0a, p0b) + fminf(p1a, p1b) + fminf(p2a, p2b);
        const float xh = fmaxf(p0a, p0b) + fmaxf(p1a, p1b) + fmaxf(p2a, p2b);
        const float tl = fmaf(xl, ax.s, -ax.los), th = fmaf(xh, ax.s, -ax.los);
        const float bdl = 2.0f * fmaf(ax.c, bqm, ax.d);
        if (th < -bdl || tl >= ax.n + bdl) continue;  // no event of this warp can land: skip
      }
#endif
      const float x = fmaf(ax.r2, q2, fmaf(ax.r1, q1, ax.r0 * q0));
      const float t = fmaf(x, ax.s, -ax.los);
      const float dl = fmaf(ax.c, qm, ax.d);
      const bool pass = valid && t >= -dl && t < ax.n + dl;
      const unsigned mask = __ballot_sync(kFull, pass);
      if (pass) {
        const int slot = (qhead + qcnt + __popc(mask & ((1u << lane) - 1u))) & 63;
        qv[slot] = ev;
        qc[slot] = c;
        if (has_err) qe[slot] = ev_e;
      }
      qcnt += __popc(mask);
      if (qcnt >= 32) drain(32);
    }
  };
  for (; base < p.nevents; base += stride) {
    float4 nxt = make_float4(0.f, 0.f, 0.f, 0.f);  // software prefetch of the next event
    float nxt_e = 0.f;
    if (base + stride + lane < p.nevents) {
      nxt = load(base + stride + lane);
      nxt_e = load_e(base + stride + lane);
    }
    test_event(cur, cur_e, base + lane < p.nevents);
    cur = nxt;
    cur_e = nxt_e;
  }
  if (qcnt > 0) drain(qcnt);
  if (kPriv) {
    __syncthreads();
    priv_flush(hb, p.binmd, p.g.nbins);
    if (p.col_e >= 0) priv_flush(he, p.err2, p.g.nbins);
  }
  if (kStats) {
    flush_counter(p.stats + 4, c_pairs);
    flush_counter(p.stats + 5, c_in);
  }
  // Programmatic dependent launch (launch_binmd_t): this grid may start while the walk before it
  // is still running (BinMD reads nothing the walk writes), but it does not complete before the
  // walk has, so a kernel after BinMD still sees the norm histogram.  No-op without the attribute.
  if (threadIdx.x == 0) asm volatile("griddepcontrol.wait;" ::: "memory");
}

// ---------------------------------------------------------------- X2
__global__ void __launch_bounds__(kThreads)
xs_kernel(const double* __restrict__ norm, const double* __restrict__ binmd, double* __restrict__ xs,
          int64_t n) {
  // launched with programmatic stream serialisation: the histograms are read only after the
  // preceding grid has completed (no-op without the attribute)
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const double d = norm[i];
    xs[i] = d > 0.0 ? ddiv(binmd[i], d) : CUDART_NAN;
  }
}

__global__ void __launch_bounds__(kThreads)
xs_err_kernel(const double* __restrict__ norm, const double* __restrict__ binmd, const double* __restrict__ err2,
              double* __restrict__ xs, double* __restrict__ xs_err, int64_t n) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const double d = norm[i];
    xs[i] = d > 0.0 ? ddiv(binmd[i], d) : CUDART_NAN;
    xs_err[i] = d > 0.0 ? ddiv(__dsqrt_rn(err2[i]), d) : CUDART_NAN;  // IEEE sqrt, as the oracle
  }
}

// ---------------------------------------------------------------- setup kernels
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
  __device__ __forceinline__ void operator()(int b, double val) {
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
  const double v[3] = {row_dot(M, px.x, px.y, px.z), row_dot(M + 3, px.x, px.y, px.z),
                       row_dot(M + 6, px.x, px.y, px.z)};
  double kin, kout, klo, khi;
  pixel_krange(p, pi, klo, khi);
  if (!traj_clip(p.g, v, klo, khi, kin, kout)) {
    n_cross[t] = 0;
    n_seg[t] = 0;
    return;
  }
  RecordEmit rec{seg_bins + t * max_segs, seg_vals + t * max_segs, max_segs, 0};
  int nc;
  const FluxView fv = p.fviews ? p.fviews[p.ptab[pi]] : p.flux;
  n_seg[t] = traj_walk<true>(p.g, fv, v[0], v[1], v[2], kin, kout, dmul(px.w, sC[m]), rec, &nc);
  n_cross[t] = nc + 2;  // |L| = clip endpoints + crossings
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

int grid_for(int64_t work, int num_sms, int per_sm, int threads = kThreads) {
  int64_t blocks = (work + threads - 1) / threads;
  blocks = std::min<int64_t>(blocks, (int64_t)num_sms * per_sm);
  return (int)std::max<int64_t>(blocks, 1);
}

// dynamic shared memory of the walk kernel (layout in mdnorm_walk_kernel)
size_t walk_smem(const MdnParams& p, bool smem_flux, int threads) {
  return (smem_flux ? 2 * sizeof(double2) * p.flux.n + (MDN_FLUX_NOKN ? 0 : sizeof(double) * ((p.flux.n + 3) & ~1)) +
                          sizeof(uint16_t) * ((p.flux.ntab + 1) & ~1)
                    : 0) +
         (sizeof(int) * 32 + 2 * sizeof(unsigned) * kWalkRing) * (threads / 32);
}

template <int kFlux, bool kStats, bool k3D, int kPriv>
cudaError_t launch_walk(const MdnParams& p, int num_sms, cudaStream_t s) {
  constexpr int threads = walk_threads(k3D);
  const size_t smem = walk_smem(p, kFlux == 1, threads) + priv_bytes(kPriv, p.g.nbins);
  auto k = mdnorm_walk_kernel<kFlux, kStats, k3D, kPriv>;
  cudaError_t err = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, threads, smem);
  if (err != cudaSuccess) return err;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(num_sms * std::max(per_sm, 1)));
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  // programmatic dependent launch after the cull (see griddepcontrol.wait in mdnorm_walk_kernel):
  // the walk's prologue and launch overlap the cull's tail.  Measured on CORELLI: MDNorm 0.362 ms
  // vs 0.372, step 0.481 vs 0.490.  MDN_PDL_WALK=0 turns it off.
  static const bool pdl = [] { const char* e = std::getenv("MDN_PDL_WALK"); return !e || std::atoi(e) != 0; }();
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, p);
}

template <int kFlux, int kPriv>
cudaError_t launch_walk_d(const MdnParams& p, bool d3, int num_sms, cudaStream_t s) {
  if (d3) return p.stats ? launch_walk<kFlux, true, true, kPriv>(p, num_sms, s)
                         : launch_walk<kFlux, false, true, kPriv>(p, num_sms, s);
  return p.stats ? launch_walk<kFlux, true, false, kPriv>(p, num_sms, s)
                 : launch_walk<kFlux, false, false, kPriv>(p, num_sms, s);
}

thread_local int g_last_mdnorm_path = 0;
thread_local int g_last_binmd_path = 0;

int smem_optin(cudaError_t* err) {
  int dev = 0, smem_max = 0;
  if ((*err = cudaGetDevice(&dev)) != cudaSuccess) return 0;
  *err = cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return smem_max;
}

template <bool kStats>
cudaError_t launch_cull(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  const size_t smem = (sizeof(double) * 10 + sizeof(CullMat)) * (size_t)mb.nmat +
                      sizeof(uint32_t) * 128 * (kThreads / 32);
  auto k = mdnorm_cull_kernel<kStats>;
  cudaError_t err = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  // one wave of resident CTAs (grid-stride): no tail wave of unevenly loaded blocks
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kThreads, smem);
  if (err != cudaSuccess) return err;
  k<<<grid_for(p.plen, num_sms, std::max(per_sm, 1)), kThreads, smem, s>>>(p, mb);
  return cudaGetLastError();
}

template <bool kPacked, bool kStats, int kPriv>
cudaError_t launch_binmd_t(const BinParams& p, const MatBlock& mb, int num_sms, size_t smem, cudaStream_t s) {
  constexpr int threads = bin_threads(kPriv);
  auto k = binmd_kernel<kPacked, kStats, kPriv>;
  cudaError_t err = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, threads, smem);
  if (err != cudaSuccess) return err;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid_for(p.nevents, num_sms, std::max(per_sm, 1), threads));
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  // MDN_PDL=1 lets BinMD start during the preceding walk's end spread (programmatic dependent
  // launch; see the end of binmd_kernel).  Off by default: measured on CORELLI 0.536 ms/step
  // against 0.492 without -- BinMD's grid-stride CTAs get equal shares but start staggered over
  // the walk's tail, so BinMD ends later than it gains.
  static const bool pdl = [] { const char* e = std::getenv("MDN_PDL"); return e && std::atoi(e) != 0; }();
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, p, mb);
}

template <int kPriv>
cudaError_t launch_binmd_p(const BinParams& p, const MatBlock& mb, bool packed, int num_sms, size_t smem,
                           cudaStream_t s) {
  if (packed) return p.stats ? launch_binmd_t<true, true, kPriv>(p, mb, num_sms, smem, s)
                             : launch_binmd_t<true, false, kPriv>(p, mb, num_sms, smem, s);
  return p.stats ? launch_binmd_t<false, true, kPriv>(p, mb, num_sms, smem, s)
                 : launch_binmd_t<false, false, kPriv>(p, mb, num_sms, smem, s);
}

}  // namespace

cudaError_t launch_pixels_prepare(const double* dir, const double* solid, double4* pix, int64_t npix,
                                  cudaStream_t s) {
  pixels_prepare_kernel<<<grid_for(npix, 148, 8), kThreads, 0, s>>>(dir, solid, pix, npix);
  return cudaGetLastError();
}

cudaError_t launch_mdnorm(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.plen == 0 || mb.nmat <= 0) return cudaSuccess;
  cudaError_t err = cudaMemsetAsync(p.ctr, 0, sizeof(DevCounters), s);
  if (err != cudaSuccess) return err;
  err = p.stats ? launch_cull<true>(p, mb, num_sms, s) : launch_cull<false>(p, mb, num_sms, s);
  if (err != cudaSuccess) return err;
  // 2-D slices (a single bin on the last axis, "lBins=1") merge two crossing streams
  const bool d3 = p.g.n[2] > 1;
  const int smem_max = smem_optin(&err);
  if (err != cudaSuccess) return err;
  const int threads = walk_threads(d3);
  // the flux table goes to shared memory when it fits one CTA (uint16 cell entries)
  const bool flux_fits = p.flux.n <= kFluxSmemMax && walk_smem(p, true, threads) <= (size_t)smem_max;
  // Private shared-memory histogram (S§2.8 G2) when the grid fits next to the walk's other shared
  // data: with the flux table in shared memory if both fit, else with the flux read through L1.
  // priv = 1 takes it whenever it fits; auto (-1) when the launch's trajectories outnumber the
  // bins the flush touches (one CTA per SM flushes every bin) by MDN_PRIV_TRAJ_PER_BIN (3-D
  // grids: every trajectory crosses the box) or 16x that (2-D slices: a few % hit the slab).
  // Measured (tools/priv_sweep.sh): TOPAZ 8 ops on 16^3 - 25^3 grids 2.1-3.2x faster; CORELLI
  // 24 ops on 16^2 / 60^2 slabs 2.7x / 1.2x faster, on 100^2 equal, on 150^2 1.35x slower.
  const int kind = p.acc_f32 ? 2 : 1;
  const size_t hb = priv_bytes(kind, p.g.nbins);
  const bool priv_ok = p.priv != 0 && !p.fviews;
  const uint64_t per_bin = (uint64_t)MDN_PRIV_TRAJ_PER_BIN * (d3 ? 1u : 16u);
  const bool worth = p.priv == 1 ||
                     (uint64_t)p.plen * (uint64_t)mb.nmat >= (uint64_t)p.g.nbins * (uint64_t)num_sms * per_bin;
  const bool with_sflux = priv_ok && worth && flux_fits && walk_smem(p, true, threads) + hb <= (size_t)smem_max;
  const bool with_gflux = priv_ok && worth && !with_sflux && walk_smem(p, false, threads) + hb <= (size_t)smem_max;
  if (with_sflux || with_gflux) {
    g_last_mdnorm_path = kind;
    if (with_sflux) return kind == 2 ? launch_walk_d<1, 2>(p, d3, num_sms, s) : launch_walk_d<1, 1>(p, d3, num_sms, s);
    return kind == 2 ? launch_walk_d<0, 2>(p, d3, num_sms, s) : launch_walk_d<0, 1>(p, d3, num_sms, s);
  }
  g_last_mdnorm_path = 0;
  if (p.fviews) return launch_walk_d<2, 0>(p, d3, num_sms, s);
  if (flux_fits) return launch_walk_d<1, 0>(p, d3, num_sms, s);
  return launch_walk_d<0, 0>(p, d3, num_sms, s);
}

cudaError_t launch_binmd(const BinParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.nevents <= 0 || mb.nmat <= 0) return cudaSuccess;
  const bool packed = p.stride == 4 && p.col_w == 0 && p.col_q == 1 &&
                      (reinterpret_cast<uintptr_t>(p.events) & 15) == 0;
  // Private shared-memory histogram(s) (S§2.8 G3) when binmd (+ err2) fit one 512-thread CTA
  // next to its static shared data.  priv = 1 takes it whenever it fits; auto (-1) only when two
  // CTAs fit per SM (with one, 16 warps per SM cannot keep the event stream going) and the
  // (event, op) pairs outnumber the flushed bins by 64 (measured, tools/priv_sweep.sh: TOPAZ
  // 8 ops on 16^3 / 20^3 2.5x faster, CORELLI 24 ops on 16^2 2.6x and 60^2 1.1x faster; a
  // 100^2 slab, one CTA per SM, 1.5x slower).
  cudaError_t err = cudaSuccess;
  const int smem_max = smem_optin(&err);
  if (err != cudaSuccess) return err;
  const int kind = p.acc_f32 ? 2 : 1;
  const size_t hb = priv_bytes(kind, p.g.nbins) * (p.col_e >= 0 ? 2 : 1);
  if (p.priv != 0) {
    cudaFuncAttributes fa{};
    err = packed ? cudaFuncGetAttributes(&fa, binmd_kernel<true, false, 1>)
                 : cudaFuncGetAttributes(&fa, binmd_kernel<false, false, 1>);
    if (err != cudaSuccess) return err;
    int dev = 0, sm_smem = 0;
    if ((err = cudaGetDevice(&dev)) != cudaSuccess) return err;
    if ((err = cudaDeviceGetAttribute(&sm_smem, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev)) != cudaSuccess)
      return err;
    const size_t per_cta = fa.sharedSizeBytes + hb + 1024;  // + the per-CTA reservation
    const bool fits = per_cta <= (size_t)smem_max;
    const uint64_t ctas = (uint64_t)num_sms * 2;
    const bool worth = p.priv == 1 || (2 * per_cta <= (size_t)sm_smem &&
                                       (uint64_t)p.nevents * (uint64_t)mb.nmat >= (uint64_t)p.g.nbins * ctas * 64);
    if (fits && worth) {
      g_last_binmd_path = kind;
      return kind == 2 ? launch_binmd_p<2>(p, mb, packed, num_sms, hb, s) : launch_binmd_p<1>(p, mb, packed, num_sms, hb, s);
    }
  }
  g_last_binmd_path = 0;
  return launch_binmd_p<0>(p, mb, packed, num_sms, 0, s);
}

int last_mdnorm_path() { return g_last_mdnorm_path; }
int last_binmd_path() { return g_last_binmd_path; }

cudaError_t launch_cross_section(const double* norm, const double* binmd, double* xs, int64_t nbins,
                                 int num_sms, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid_for(nbins, num_sms, 8));
  cfg.blockDim = dim3(kThreads);
  cfg.stream = s;
  // programmatic dependent launch after BinMD (MDN_PDL_XS=0 turns it off)
  static const bool pdl = [] { const char* e = std::getenv("MDN_PDL_XS"); return !e || std::atoi(e) != 0; }();
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, xs_kernel, norm, binmd, xs, nbins);
}

cudaError_t launch_cross_section_err(const double* norm, const double* binmd, const double* err2, double* xs,
                                     double* xs_err, int64_t nbins, int num_sms, cudaStream_t s) {
  xs_err_kernel<<<grid_for(nbins, num_sms, 8), kThreads, 0, s>>>(norm, binmd, err2, xs, xs_err, nbins);
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

#if MDN_WALK_TRACE
}  // namespace mdn
extern "C" int mdn_debug_walk_trace(unsigned long long* out, int n) {
  return (int)cudaMemcpyFromSymbol(out, mdn::g_walk_trace, sizeof(unsigned long long) * (size_t)n);
}
namespace mdn {
#endif
}  // namespace mdn
