// mdn_binmd.cu -- B0-B3 of SURVEY.md §8(a): BinMD (Listings 2-3) on sm_100a.
//
// binmd[b] += w_e * 1[N_s Q_e in b] for every (event e, symmetry op s).  The definition (oracle
// step 9) decides each (event, op) pair in fp64: x_a = ((N_a0 q0 + N_a1 q1) +
// N_a2 q2), t_a = (x_a - lo_a) s_a, inside iff 0 <= t_a < n_a, bin i_a = floor(t_a).  The kernel
// decides almost every pair in fp32 inside a proven error band and hands the rest (a t within the
// band of a decision point) to that exact fp64 formula, so every bin index is the definition's.
//
// fp32 fast path ("binmd_kernel").  Per (matrix m, axis a) the folded constants
//   a_i = RN32(N_ai s_a), b = RN32(lo_a s_a),  t32 = fma(a2, q2, fma(a1, q1, fma(a0, q0, -b)))
// satisfy |t32 - t64| <= 2^-24 * 4.1 * (s_a sum_i |N_ai| |q|max + |lo_a s_a| + n_a) + fp64 terms,
// and the band used is dl = c |q|max + d with c = 1e-6 s_a sum|N_ai|, d = 1e-6 (|lo_a s_a| + n_a
// + 1): at least 4x that bound.  A pair is decided in fp32 only when t32 lies further than dl from
// 0, n_a and every integer on every axis.
//
// Op classes.  Axes are tested in the order ord (fewest bins first: the thin L axis of a 2-D
// slice).  Ops whose fp32 first-axis constants are identical form a class and share one test
// (symmetry ops map L -> +-L: 2 classes for 6/mmm on an HK0 slice).  The class test is folded
// around the slab centre, u = t32 - n/2, and passes iff |u| < n/2 + dl -- a superset of the pairs
// the definition keeps on that axis.  Classes are tested per event with their constants in
// registers (1 or 2 classes; more classes read them from shared memory as broadcasts); an
// event that passes some class is queued with its class mask in a per-warp shared-memory ring,
// and the members of its classes are decided when 32 entries are queued (the warp converged).
#include <cstdint>

#include "mdn_common.cuh"

namespace mdn {

#ifdef MDN_EXP_CLOCK
__device__ long long g_bin_clock[1024 * 8];
#define BIN_CLK(i) do { if ((threadIdx.x & 31) == 0 && blockIdx.x < 1024 && (threadIdx.x >> 5) == 0) { long long t_; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_)); g_bin_clock[blockIdx.x * 8 + (i)] = t_; } } while (0)
#else
#define BIN_CLK(i) do {} while (0)
#endif

namespace {

using namespace common;

#ifndef MDN_BIN_MINB
#define MDN_BIN_MINB 4
#endif
#ifndef MDN_BIN_DEPTH
#define MDN_BIN_DEPTH 3
#endif
constexpr int kBinMinBlocks = MDN_BIN_MINB;  // resident 256-thread CTAs per SM (global path)
constexpr int kDepth = MDN_BIN_DEPTH;        // 32-event blocks in flight per warp
// per-warp ring of (event, class mask) entries: >= kDepth x 32 + 31, a power of two
constexpr int kBinQueue = kDepth * 32 + 31 < 128 ? 128 : (kDepth * 32 + 31 < 256 ? 256 : 512);

// fp32 test constants of one axis: t32 = fma(a2, q2, fma(a1, q1, fma(a0, q0, -b))) and the band
// dl = fma(c, |q|max, d); for the class test b includes n/2 and d includes n/2 (hw = n/2 + dl).
struct alignas(16) AxisF {
  float a0, a1, a2, b;
  float c, d, n, pad;
};

__device__ __forceinline__ float axis_t(const AxisF& x, float q0, float q1, float q2) {
  return fmaf(x.a2, q2, fmaf(x.a1, q1, fmaf(x.a0, q0, -x.b)));
}

__host__ __device__ constexpr int bin_threads(int kPriv) { return kPriv ? 512 : kThreads; }

// dynamic shared memory of the per-warp queues (events, class masks, error-squared column)
constexpr size_t queue_bytes(int threads) {
  return (size_t)(threads / 32) * kBinQueue * (sizeof(float4) + sizeof(unsigned) + sizeof(float));
}

// Shared tables of one launch (built by every CTA's prologue from the composed N_s).
struct BinTables {
  double sN[kMaxMats * 9];   // N_s (fp64, the exact fallback)
  AxisF sMA[kMaxMats * 2];   // member constants, test-order axes 1 and 2 (by matrix)
  AxisF mC0[kMaxMats];       // test-order axis 0 constants (by matrix)
  AxisF mCT[kMaxMats];       // class test constants, folded around n/2 (by matrix)
  AxisF sC0[kMaxMats];       // the same by class
  AxisF sCT[kMaxMats];
  int sCid[kMaxMats];        // class of matrix m
  int sCls[kMaxMats + 1];    // members of class c: sMem[sCls[c] .. sCls[c+1])
  int sMem[kMaxMats];
  int sCnt[2][kMaxMats];     // grouping scratch: class sizes in each half of the matrices
  int ncls;
};

__device__ __forceinline__ AxisF make_axis(const BinParams& p, const double* N, int k, bool fold) {
  const int a = p.ord[k];
  const double* row = N + 3 * a;
  const double s = p.g.s[a], lo = p.g.lo[a], n = (double)p.g.n[a];
  const double sum = fabs(row[0]) + fabs(row[1]) + fabs(row[2]);
  AxisF x;
  x.a0 = (float)(row[0] * s);
  x.a1 = (float)(row[1] * s);
  x.a2 = (float)(row[2] * s);
  x.b = (float)(fold ? lo * s + 0.5 * n : lo * s);
  x.c = (float)(1e-6 * s * sum);
  x.d = (float)(1e-6 * (fabs(lo * s) + n + 1.0) + (fold ? 0.5 * n : 0.0));
  x.n = (float)n;
  x.pad = 0.f;
  return x;
}

// Lanes (of the calling lanes `act`) whose six test floats equal this lane's: one match per float.
__device__ __forceinline__ unsigned match_axis(unsigned act, const AxisF& x) {
  return __match_any_sync(act, __float_as_uint(x.a0)) & __match_any_sync(act, __float_as_uint(x.a1)) &
         __match_any_sync(act, __float_as_uint(x.a2)) & __match_any_sync(act, __float_as_uint(x.b)) &
         __match_any_sync(act, __float_as_uint(x.c)) & __match_any_sync(act, __float_as_uint(x.d));
}

__device__ __forceinline__ bool same_axis(const AxisF& x, const AxisF& y) {
  return __float_as_uint(x.a0) == __float_as_uint(y.a0) && __float_as_uint(x.a1) == __float_as_uint(y.a1) &&
         __float_as_uint(x.a2) == __float_as_uint(y.a2) && __float_as_uint(x.b) == __float_as_uint(y.b) &&
         __float_as_uint(x.c) == __float_as_uint(y.c) && __float_as_uint(x.d) == __float_as_uint(y.d);
}

// Builds the fp32 constants and the op classes (whole CTA; two __syncthreads).  Thread m < nmat
// composes N_m (B0) and its three axes' constants; warp 0 then groups the matrices whose class
// test constants are identical (warp match instructions, no serial loops): classes are numbered
// in order of their smallest member, members listed in increasing m.
__device__ void build_tables(const BinParams& p, const MatBlock& mb, BinTables& T) {
  const int nmat = mb.nmat;
  BIN_CLK(0);
  for (int m = threadIdx.x; m < nmat; m += blockDim.x) {
    double* N = T.sN + 9 * m;
    if (mb.compose) {
      if (!compose_binmd(mb.UB, mb.u.c.ops + 9 * m, mb.W, N))
        for (int i = 0; i < 9; ++i) N[i] = CUDART_NAN;
    } else {
      for (int i = 0; i < 9; ++i) N[i] = mb.u.M[9 * m + i];
    }
    T.mC0[m] = make_axis(p, N, 0, false);
    T.mCT[m] = make_axis(p, N, 0, true);
    T.sMA[2 * m] = make_axis(p, N, 1, false);
    T.sMA[2 * m + 1] = make_axis(p, N, 2, false);
  }
  BIN_CLK(1);
  __syncthreads();
  BIN_CLK(2);
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    const unsigned lt = (1u << lane) - 1u;
    // matrix m0 = lane (first half) and m1 = lane + 32 (second half)
    const int n0 = min(nmat, 32), n1 = max(nmat - 32, 0);
    const bool v0 = lane < n0, v1 = lane < n1;
    const unsigned act0 = n0 == 32 ? 0xffffffffu : (1u << n0) - 1u;
    const unsigned act1 = n1 == 32 ? 0xffffffffu : (1u << n1) - 1u;
    AxisF k0{}, k1{};
    if (v0) k0 = T.mCT[lane];
    if (v1) k1 = T.mCT[lane + 32];
    unsigned pe0 = 0, pe1 = 0;
    if (v0) pe0 = match_axis(act0, k0);
    if (v1) pe1 = match_axis(act1, k1);
    int rep0 = v0 ? __ffs(pe0) - 1 : -1;  // smallest equal first-half matrix
    // a second-half matrix whose constants equal some first-half matrix's belongs to that class
    int rep1 = -1;
    if (n1 > 0) {
      for (int j = 0; j < n0; ++j) {
        AxisF y;
        y.a0 = __shfl_sync(kFull, k0.a0, j);
        y.a1 = __shfl_sync(kFull, k0.a1, j);
        y.a2 = __shfl_sync(kFull, k0.a2, j);
        y.b = __shfl_sync(kFull, k0.b, j);
        y.c = __shfl_sync(kFull, k0.c, j);
        y.d = __shfl_sync(kFull, k0.d, j);
        if (v1 && rep1 < 0 && same_axis(k1, y)) rep1 = j;
      }
      if (v1 && rep1 < 0) rep1 = 32 + __ffs(pe1) - 1;
    }
    const bool r0 = v0 && rep0 == lane, r1 = v1 && rep1 == lane + 32;
    const unsigned b0 = __ballot_sync(kFull, r0), b1 = __ballot_sync(kFull, r1);
    const int nr0 = __popc(b0), ncls = nr0 + __popc(b1);
    // class ids in order of the smallest member (first-half reps, then second-half reps)
    const int id_r0 = __popc(b0 & lt), id_r1 = nr0 + __popc(b1 & lt);
    const int c0 = __shfl_sync(kFull, id_r0, max(rep0, 0));
    const int c1f = __shfl_sync(kFull, id_r0, rep1 >= 0 && rep1 < 32 ? rep1 : 0);
    const int c1s = __shfl_sync(kFull, id_r1, rep1 >= 32 ? rep1 - 32 : 0);
    const int cid0 = v0 ? c0 : -1;
    const int cid1 = v1 ? (rep1 < 32 ? c1f : c1s) : -1;
    if (v0) T.sCid[lane] = cid0;
    if (v1) T.sCid[lane + 32] = cid1;
    // class sizes per half, then starts (exclusive scan over the <= 64 classes, two per lane)
    for (int c = lane; c < kMaxMats; c += 32) T.sCnt[0][c] = T.sCnt[1][c] = 0;
    __syncwarp();
    unsigned q0 = 0, q1 = 0;
    if (v0) q0 = __match_any_sync(act0, cid0);
    if (v1) q1 = __match_any_sync(act1, cid1);
    if (v0 && (q0 & lt) == 0) T.sCnt[0][cid0] = __popc(q0);
    if (v1 && (q1 & lt) == 0) T.sCnt[1][cid1] = __popc(q1);
    __syncwarp();
    const int ca = lane < ncls ? T.sCnt[0][lane] + T.sCnt[1][lane] : 0;
    const int cb = lane + 32 < ncls ? T.sCnt[0][lane + 32] + T.sCnt[1][lane + 32] : 0;
    int ia = ca, ib = cb;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int ya = __shfl_up_sync(kFull, ia, o), yb = __shfl_up_sync(kFull, ib, o);
      if (lane >= o) {
        ia += ya;
        ib += yb;
      }
    }
    const int tota = __shfl_sync(kFull, ia, 31);
    if (lane < ncls) T.sCls[lane] = ia - ca;
    if (lane + 32 < ncls) T.sCls[lane + 32] = tota + ib - cb;
    if (lane == 0) {
      T.sCls[ncls] = nmat;
      T.ncls = ncls;
    }
    __syncwarp();
    // members in increasing m: first-half members of a class precede its second-half members
    if (v0) T.sMem[T.sCls[cid0] + __popc(q0 & lt)] = lane;
    if (v1) T.sMem[T.sCls[cid1] + T.sCnt[0][cid1] + __popc(q1 & lt)] = lane + 32;
    // class-indexed constants from each class's smallest member
    if (r0) {
      T.sC0[id_r0] = T.mC0[lane];
      T.sCT[id_r0] = k0;
    }
    if (r1) {
      T.sC0[id_r1] = T.mC0[lane + 32];
      T.sCT[id_r1] = k1;
    }
  }
  BIN_CLK(3);
  __syncthreads();
  BIN_CLK(4);
}

// First test-order axis of a queued (event, class): t, band, floor, near flag; false if the
// pair is definitely outside on that axis.
struct Axis0 {
  int i0;
  bool near;
};

__device__ __forceinline__ bool class_axis0(const AxisF& x, float q0, float q1, float q2, float qm, Axis0& r) {
  const float t = axis_t(x, q0, q1, q2);
  const float dl = fmaf(x.c, qm, x.d);
  if (t < -dl || t >= x.n + dl) return false;
  const float fl = floorf(t);
  const float fr = t - fl;
  r.near = t < dl || t > x.n - dl || fr < dl || fr > 1.0f - dl;
  r.i0 = (int)fl;
  return true;
}

// Bin of member m of a class whose first axis passed (r0), or -1: the remaining two axes in fp32
// with the band, the exact fp64 definition when any axis is within its band of a decision point.
__device__ __forceinline__ int member_bin(const BinParams& p, const BinTables& T, int m, float q0, float q1,
                                          float q2, float qm, const Axis0& r0) {
  const AxisF x1 = T.sMA[2 * m], x2 = T.sMA[2 * m + 1];
  const float t1 = axis_t(x1, q0, q1, q2), t2 = axis_t(x2, q0, q1, q2);
  const float d1 = fmaf(x1.c, qm, x1.d), d2 = fmaf(x2.c, qm, x2.d);
  if (t1 < -d1 || t1 >= x1.n + d1 || t2 < -d2 || t2 >= x2.n + d2) return -1;
  const float f1 = floorf(t1), f2 = floorf(t2);
  const float r1 = t1 - f1, r2 = t2 - f2;
  const bool near = r0.near || t1 < d1 || t1 > x1.n - d1 || r1 < d1 || r1 > 1.0f - d1 || t2 < d2 ||
                    t2 > x2.n - d2 || r2 < d2 || r2 > 1.0f - d2;
  if (!near) return r0.i0 * p.st[0] + (int)f1 * p.st[1] + (int)f2 * p.st[2];
  const int64_t be = event_bin(p.g, T.sN + 9 * m, (double)q0, (double)q1, (double)q2);
  return (int)be;  // -1 outside
}

// The class test of one event for kNC classes held in registers (kNC = 0: ncls classes read from
// shared memory).  Returns the mask of passing classes.
template <int kNC>
struct ClassTest {
  float a0[kNC > 0 ? kNC : 1], a1[kNC > 0 ? kNC : 1], a2[kNC > 0 ? kNC : 1], b[kNC > 0 ? kNC : 1];
  float c[kNC > 0 ? kNC : 1], d[kNC > 0 ? kNC : 1];
  __device__ __forceinline__ void load(const BinTables& T) {
    if constexpr (kNC > 0) {
#pragma unroll
      for (int k = 0; k < kNC; ++k) {
        if (k < T.ncls) {
          const AxisF& x = T.sCT[k];
          a0[k] = x.a0; a1[k] = x.a1; a2[k] = x.a2; b[k] = x.b; c[k] = x.c; d[k] = x.d;
        } else {  // padding class: never passes
          a0[k] = a1[k] = a2[k] = b[k] = c[k] = 0.f;
          d[k] = -1.f;
        }
      }
    }
  }
  __device__ __forceinline__ unsigned operator()(const BinTables& T, float q0, float q1, float q2, float qm) const {
    unsigned mask = 0;
    if constexpr (kNC > 0) {
#pragma unroll
      for (int k = 0; k < kNC; ++k) {
        const float u = fmaf(a2[k], q2, fmaf(a1[k], q1, fmaf(a0[k], q0, -b[k])));
        if (fabsf(u) < fmaf(c[k], qm, d[k])) mask |= 1u << k;
      }
    } else {
      for (int k = 0; k < T.ncls; ++k) {
        const AxisF x = T.sCT[k];
        const float u = axis_t(x, q0, q1, q2);
        if (fabsf(u) < fmaf(x.c, qm, x.d)) mask |= 1u << (k < 31 ? k : 31);  // bit 31: classes 31 ..
      }
    }
    return mask;
  }
};

// Decide the queued (event, class mask) entries [qhead, qhead + n) of this warp, one per lane:
// every member of every passing class (member_bin) and its reduction.  Returns this lane's
// (event, op) pairs inside.
template <int kPriv>
__device__ __forceinline__ unsigned drain_queue(const BinParams& p, const BinTables& T, const float4* qv,
                                             const unsigned* qk, const float* qe, int qhead, int n,
                                             bool has_err, priv_t<kPriv>* hb, priv_t<kPriv>* he) {
  using PT = priv_t<kPriv>;
  const int lane = threadIdx.x & 31;
  unsigned inside = 0;
  if (lane < n) {
    const int slot = (qhead + lane) & (kBinQueue - 1);
    const float4 ev = qv[slot];
    const float e2 = has_err ? qe[slot] : 0.f;
    unsigned mask = qk[slot];
    const float qm = fmaxf(fabsf(ev.y), fmaxf(fabsf(ev.z), fabsf(ev.w)));
    // bit c < 31: class c passed; bit 31: some class >= 31 passed (each is re-tested below)
    int c = -1, cend = 0;
    for (;;) {
      if (c + 1 < cend) {
        ++c;
      } else {
        if (!mask) break;
        c = __ffs(mask) - 1;
        mask &= mask - 1u;
        cend = c == 31 ? T.ncls : c + 1;
      }
      Axis0 r0;
      if (!class_axis0(T.sC0[c], ev.y, ev.z, ev.w, qm, r0)) continue;
      for (int j = T.sCls[c]; j < T.sCls[c + 1]; ++j) {
        const int b = member_bin(p, T, T.sMem[j], ev.y, ev.z, ev.w, qm, r0);
        if (b < 0) continue;
#ifdef MDN_EXP_NORED
        if (ev.x == -12345.f) p.binmd[b] = ev.x;
#else
        if constexpr (kPriv != 0) hist_add<PT>(hb, he, b, (PT)ev.x, (PT)e2, has_err);
        else hist_add<double>(p.binmd, p.err2, b, (double)ev.x, (double)e2, has_err);
#endif
        ++inside;
      }
    }
  }
  return inside;
}

template <bool kPacked>
__device__ __forceinline__ float4 load_event(const BinParams& p, int64_t e) {
  if (kPacked) return __ldcs(reinterpret_cast<const float4*>(p.events) + e);
  const float* ev = p.events + e * p.stride;
  return make_float4(__ldcs(ev + p.col_w), __ldcs(ev + p.col_q), __ldcs(ev + p.col_q + 1), __ldcs(ev + p.col_q + 2));
}

// The event loop for kNC register classes: grid-stride over warp-contiguous 32-event blocks,
// two blocks prefetched ahead (three float4 per lane in flight: the event stream is the roof).
template <int kNC, bool kPacked, bool kStats, int kPriv>
__device__ __forceinline__ void binmd_loop(const BinParams& p, const MatBlock& mb, const BinTables& T,
                                           float4* qv, unsigned* qk, float* qe, priv_t<kPriv>* hb,
                                           priv_t<kPriv>* he, unsigned long long& c_pairs,
                                           unsigned long long& c_in) {
  ClassTest<kNC> ct;
  ct.load(T);
  const int lane = threadIdx.x & 31;
  const bool has_err = !kPacked && p.col_e >= 0;
  int qhead = 0, qcnt = 0;

  auto drain = [&](int n) {
    __syncwarp();
    const unsigned in = drain_queue<kPriv>(p, T, qv, qk, qe, qhead, n, has_err, hb, he);
    if (kStats) c_in += in;
    qhead = (qhead + n) & (kBinQueue - 1);
    qcnt -= n;
    __syncwarp();
  };

  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  // 32-event block of warp w of CTA c in round k: (k W + w) C + c (W warps per CTA, C CTAs), so
  // consecutive blocks go to different CTAs, i.e. different SMs: the in-grid events of the
  // Q-ordered stream (a Bragg peak, the slab) are spread over all SMs (measured: per-SM active
  // cycles max / mean 1.38 with CTA-contiguous blocks on the CORELLI slab).
  const int64_t base0 = ((int64_t)(threadIdx.x >> 5) * gridDim.x + blockIdx.x) * 32;  // warp-uniform
  // rounds of this warp, and of this lane (they differ only in the last, ragged block)
  const int64_t n = p.nevents;
  const int rounds = base0 < n ? (int)((n - 1 - base0) / stride) + 1 : 0;
  const int lrounds = base0 + lane < n ? (int)((n - 1 - base0 - lane) / stride) + 1 : 0;
  // event of this lane in round r: e0 + r stride (64-bit only in the address arithmetic)
  const int64_t e0 = base0 + lane;
  auto ld = [&](int r, float& e2) {
    if (r < lrounds) {
      const int64_t e = e0 + (int64_t)r * stride;
      if (has_err) e2 = __ldcs(p.events + e * p.stride + p.col_e);
      return load_event<kPacked>(p, e);
    }
    return make_float4(0.f, 0.f, 0.f, 0.f);
  };
  auto test = [&](const float4& ev, float e2, bool valid) {
    if (kStats && valid) c_pairs += mb.nmat;
    const float qm = fmaxf(fabsf(ev.y), fmaxf(fabsf(ev.z), fabsf(ev.w)));
    unsigned mask = ct(T, ev.y, ev.z, ev.w, qm);
    if (!valid) mask = 0;
#ifdef MDN_EXP_NODRAIN
    if (ev.x == -12345.f) mask = 1; else mask = 0;
#endif
    const unsigned bal = __ballot_sync(kFull, mask != 0);
    if (bal) {
      if (mask) {
        const int slot = (qhead + qcnt + __popc(bal & ((1u << lane) - 1u))) & (kBinQueue - 1);
        qv[slot] = ev;
        qk[slot] = mask;
        if (has_err) qe[slot] = e2;
      }
      qcnt += __popc(bal);
    }
  };
  // kDepth 32-event blocks in flight per warp, in fixed register sets: round r is tested and its
  // registers refilled with round r + kDepth (no register rotation -- a move out of a register
  // whose load is in flight would wait for that load).
  float4 ev[kDepth];
  float ex[kDepth] = {};
#pragma unroll
  for (int u = 0; u < kDepth; ++u) ev[u] = ld(u, ex[u]);
  for (int r = 0;;) {
#pragma unroll
    for (int u = 0; u < kDepth; ++u) {
      if (r >= rounds) goto done;
      test(ev[u], ex[u], r < lrounds);
      ev[u] = ld(r + kDepth, ex[u]);
      ++r;
    }
    // one drain site per kDepth blocks (the ring holds kDepth x 32 + 31 entries): the member code
    // is emitted once, not once per unrolled block
    while (qcnt >= 32) drain(32);
  }
done:
  BIN_CLK(5);
  while (qcnt > 0) drain(min(qcnt, 32));
  BIN_CLK(6);
}

// One thread per event (grid-stride).  kPriv: 0 = global fp64 red.add, 1 / 2 = a private fp64 /
// fp32 histogram per CTA in shared memory (binmd, then err2 when the error column is read),
// flushed into the global one at the end.
template <bool kPacked, bool kStats, int kPriv>
__global__ void __launch_bounds__(bin_threads(kPriv), kPriv ? 2 : kBinMinBlocks)
binmd_kernel(const __grid_constant__ BinParams p, const __grid_constant__ MatBlock mb) {
  constexpr int kBT = bin_threads(kPriv);
  using PT = priv_t<kPriv>;
  __shared__ BinTables T;
  // dynamic shared memory: private histograms (kPriv: binmd, then err2 when the error column is
  // read, 16-byte rounded) | per-warp queues: events | class masks | error-squared column
  extern __shared__ double4 bsm[];
  const size_t hbytes = priv_bytes(kPriv, p.g.nbins) * (kPriv && p.col_e >= 0 ? 2 : 1);
  PT* hb = reinterpret_cast<PT*>(bsm);
  PT* he = reinterpret_cast<PT*>(reinterpret_cast<char*>(bsm) + priv_bytes(kPriv, p.g.nbins));
  float4* sQv = reinterpret_cast<float4*>(reinterpret_cast<char*>(bsm) + hbytes);
  unsigned* sQk = reinterpret_cast<unsigned*>(sQv + (kBT / 32) * kBinQueue);
  float* sQe = reinterpret_cast<float*>(sQk + (kBT / 32) * kBinQueue);
  if (kPriv) {
    priv_zero(hb, p.g.nbins);
    if (p.col_e >= 0) priv_zero(he, p.g.nbins);
  }
  // the divide after BinMD (launch_cross_section, programmatic dependent launch) may launch now;
  // it waits for this grid to complete before reading either histogram
  asm volatile("griddepcontrol.launch_dependents;");
  build_tables(p, mb, T);
  const int w = threadIdx.x >> 5;
  float4* qv = sQv + w * kBinQueue;
  unsigned* qk = sQk + w * kBinQueue;
  float* qe = sQe + w * kBinQueue;
  unsigned long long c_pairs = 0, c_in = 0;
  const int ncls = T.ncls;
  if (ncls <= 1)
    binmd_loop<1, kPacked, kStats, kPriv>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
  else if (ncls <= 2)
    binmd_loop<2, kPacked, kStats, kPriv>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
  else
    binmd_loop<0, kPacked, kStats, kPriv>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
  if (kPriv) {
    __syncthreads();
    priv_flush(hb, p.binmd, p.g.nbins);
    if (p.col_e >= 0) priv_flush(he, p.err2, p.g.nbins);
  }
  if (kStats) {
    flush_counter(p.stats + 4, c_pairs);
    flush_counter(p.stats + 5, c_in);
  }
}

// Parity entry point: the bin of every (matrix, event) pair through the production decision
// (class test, first-axis band, member_bin with its fp64 fallback) -- the same device functions
// the production drain calls.
__global__ void __launch_bounds__(kThreads)
debug_bins_kernel(const __grid_constant__ BinParams p, const __grid_constant__ MatBlock mb, int64_t* bins) {
  __shared__ BinTables T;
  build_tables(p, mb, T);
  const int64_t total = p.nevents * mb.nmat;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    const int m = (int)(t / p.nevents);
    const int64_t e = t - (int64_t)m * p.nevents;
    const float* ev = p.events + e * p.stride;
    const float q0 = ev[p.col_q], q1 = ev[p.col_q + 1], q2 = ev[p.col_q + 2];
    const float qm = fmaxf(fabsf(q0), fmaxf(fabsf(q1), fabsf(q2)));
    const int c = T.sCid[m];
    const AxisF x = T.sCT[c];
    int64_t b = -1;
    Axis0 r0;
    if (fabsf(axis_t(x, q0, q1, q2)) < fmaf(x.c, qm, x.d) && class_axis0(T.sC0[c], q0, q1, q2, qm, r0))
      b = member_bin(p, T, m, q0, q1, q2, qm, r0);
    bins[t] = b;
  }
}

template <bool kPacked, bool kStats, int kPriv>
cudaError_t launch_binmd_t(const BinParams& p, const MatBlock& mb, int num_sms, size_t smem, cudaStream_t s) {
  constexpr int threads = bin_threads(kPriv);
  auto k = binmd_kernel<kPacked, kStats, kPriv>;
  smem += queue_bytes(threads);
  cudaError_t err = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, threads, smem);
  if (err != cudaSuccess) return err;
  k<<<grid_for(p.nevents, num_sms, std::max(per_sm, 1), threads), threads, smem, s>>>(p, mb);
  return cudaGetLastError();
}

template <int kPriv>
cudaError_t launch_binmd_p(const BinParams& p, const MatBlock& mb, bool packed, int num_sms, size_t smem,
                           cudaStream_t s) {
  if (packed) return p.stats ? launch_binmd_t<true, true, kPriv>(p, mb, num_sms, smem, s)
                             : launch_binmd_t<true, false, kPriv>(p, mb, num_sms, smem, s);
  return p.stats ? launch_binmd_t<false, true, kPriv>(p, mb, num_sms, smem, s)
                 : launch_binmd_t<false, false, kPriv>(p, mb, num_sms, smem, s);
}

thread_local int g_last_binmd_path = 0;

}  // namespace

cudaError_t launch_binmd(const BinParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.nevents <= 0 || mb.nmat <= 0) return cudaSuccess;
  const bool packed = p.stride == 4 && p.col_w == 0 && p.col_q == 1 && p.col_e < 0 &&
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
    const size_t per_cta = fa.sharedSizeBytes + hb + queue_bytes(bin_threads(1)) + 1024;  // + the per-CTA reservation
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

int last_binmd_path() { return g_last_binmd_path; }

#ifdef MDN_EXP_CLOCK
}  // namespace mdn
extern "C" int mdn_exp_bin_clock(long long* out) {
  return (int)cudaMemcpyFromSymbol(out, mdn::g_bin_clock, sizeof(long long) * 1024 * 8);
}
namespace mdn {
#endif

cudaError_t launch_debug_bins(const BinParams& p, const MatBlock& mb, int64_t* bins, cudaStream_t s) {
  if (p.nevents <= 0) return cudaSuccess;
  debug_bins_kernel<<<grid_for(p.nevents * mb.nmat, 148, 8), kThreads, 0, s>>>(p, mb, bins);
  return cudaGetLastError();
}

}  // namespace mdn
