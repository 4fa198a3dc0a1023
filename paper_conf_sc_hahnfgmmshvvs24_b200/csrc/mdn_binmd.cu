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
#include <cstddef>
#include <cstdint>

#include "mdn_common.cuh"

namespace mdn {

namespace {

using namespace common;

// resident 256-thread CTAs per SM (global path) and 32-event blocks in flight per warp: measured
// (4, 3) >= (4, 4), (3, 5), (2, 6), (2, 8) on the CORELLI slab (the stream alone reads 160 MB in
// 33 us at any depth 1-8, tools/stream_bench.cu)
constexpr int kBinMinBlocks = 4;
constexpr int kDepth = 3;
// per-warp ring of (event, class mask) entries: >= kDepth x 32 + 31, a power of two
constexpr float kMagic = 12582912.0f;  // 1.5 * 2^23: RD(x + kMagic) = floor(x) + kMagic for |x| < 2^22
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

// The tables of one launch: built once by binmd_plan_kernel from the composed N_s (B0), read by
// every CTA of binmd_kernel into shared memory.  Fields up to `ncls` are what the event loop and
// the member decisions use; the rest is the plan's scratch.
struct alignas(16) BinTables {
  double sN[kMaxMats * 9];   // N_s (fp64, the exact fallback)
  float4 sMF[kMaxMats * 2];  // member rows (a0, a1, a2, b) of test-order axes 1 and 2: two 16-byte loads
  float4 sCB[kMaxMats];      // per class: band slopes c (max over members) of test-order axes 0, 1, 2
  AxisF sC0[kMaxMats];       // per class: test-order axis 0 constants (bin index, band)
  AxisF sCT[kMaxMats];       // per class: class test constants, folded around n/2
  int sCid[kMaxMats];        // class of matrix m
  int sCls[kMaxMats + 1];    // members of class c: sMem[sCls[c] .. sCls[c+1])
  int sMem[kMaxMats];
  float bd[3], bn[3], bM[3]; // per test-order axis: band offset d, n, kMagic + n (fast path); bM[0]
                             // is kMagic + w1 (the end of the axis-0 window)
  float bL0;                 // kMagic + w0 (the start of the axis-0 window)
  int ncls;
  // plan scratch (not copied to the event kernel)
  AxisF sMA[kMaxMats * 2];   // member constants of test-order axes 1 and 2 (by matrix)
  AxisF mC0[kMaxMats];       // test-order axis 0 constants (by matrix)
  AxisF mCT[kMaxMats];       // class test constants (by matrix)
};
constexpr size_t kTablesUsed = (offsetof(BinTables, ncls) + sizeof(int) + 15) & ~(size_t)15;

__device__ __forceinline__ AxisF make_axis(const BinParams& p, const double* N, int k, bool fold) {
  const int a = p.ord[k];
  const double* row = N + 3 * a;
  const double s = p.g.s[a], lo = p.g.lo[a], n = (double)p.g.n[a];
  const double sum = fabs(row[0]) + fabs(row[1]) + fabs(row[2]);
  // the class test (fold, axis 0) is centred on the launch's window [w0, w1) of the axis
  const double wc = 0.5 * ((double)p.w0 + (double)p.w1), wh = 0.5 * ((double)p.w1 - (double)p.w0);
  AxisF x;
  x.a0 = (float)(row[0] * s);
  x.a1 = (float)(row[1] * s);
  x.a2 = (float)(row[2] * s);
  x.b = (float)(fold ? lo * s + wc : lo * s);
  x.c = (float)(1e-6 * s * sum);
  x.d = (float)(1e-6 * (fabs(lo * s) + n + 1.0) + (fold ? wh : 0.0));
  x.n = (float)n;
  x.pad = 0.f;
  return x;
}

// Builds the fp32 constants and the op classes (whole CTA).  The MatBlock inputs are first staged
// into shared memory by all threads (kernel-parameter reads with per-thread addresses are
// serialised); thread m < nmat then composes N_m (B0) and its three axes' constants, and the
// classes are formed from shared-memory broadcasts in unrolled loops: rep(m) = the smallest r with
// the same class-test row, classes numbered in order of their smallest member, members in
// increasing m.
__device__ void build_tables(const BinParams& p, const MatBlock& mb, BinTables& T) {
  const int nmat = mb.nmat;
  __shared__ double sIn[kMaxMats * 9 + 18];
  const int nin = mb.compose ? 9 * mb.nops + 18 : 9 * nmat;
  for (int i = threadIdx.x; i < nin; i += blockDim.x) {
    if (mb.compose)
      sIn[i] = i < 9 * mb.nops ? mb.u.c.ops[i] : (i < 9 * mb.nops + 9 ? mb.UB[i - 9 * mb.nops] : mb.W[i - 9 * mb.nops - 9]);
    else
      sIn[i] = mb.u.M[i];
  }
  __syncthreads();
  for (int m = threadIdx.x; m < nmat; m += blockDim.x) {
    double N[9];
    if (mb.compose) {
      if (!compose_binmd(sIn + 9 * mb.nops, sIn + 9 * m, sIn + 9 * mb.nops + 9, N))
        for (int i = 0; i < 9; ++i) N[i] = CUDART_NAN;
    } else {
      for (int i = 0; i < 9; ++i) N[i] = sIn[9 * m + i];
    }
    for (int i = 0; i < 9; ++i) T.sN[9 * m + i] = N[i];
    T.mC0[m] = make_axis(p, N, 0, false);
    T.mCT[m] = make_axis(p, N, 0, true);
    T.sMA[2 * m] = make_axis(p, N, 1, false);
    T.sMA[2 * m + 1] = make_axis(p, N, 2, false);
    T.sMF[2 * m] = make_float4(T.sMA[2 * m].a0, T.sMA[2 * m].a1, T.sMA[2 * m].a2, T.sMA[2 * m].b);
    T.sMF[2 * m + 1] = make_float4(T.sMA[2 * m + 1].a0, T.sMA[2 * m + 1].a1, T.sMA[2 * m + 1].a2, T.sMA[2 * m + 1].b);
  }
  if (threadIdx.x < 3) {
    const int k = threadIdx.x, a = p.ord[k];
    const double n = (double)p.g.n[a];
    // axes of 2^21 bins or more take the exact path always (the fast floor needs |t| < 2^22)
    T.bd[k] = n < 2097152.0 ? (float)(1e-6 * (fabs(p.g.lo[a] * p.g.s[a]) + n + 1.0)) : 1e30f;
    T.bn[k] = (float)n;
    T.bM[k] = kMagic + (float)(k == 0 ? p.w1 : n);
  }
  if (threadIdx.x == 0) T.bL0 = kMagic + (float)p.w0;
  __syncthreads();
  // classes: the class-test row (a0, a1, a2) decides (b and d are per axis; the band slope c is
  // taken as the class maximum below).  rep(m) = first r <= m with the same row.
  __shared__ unsigned sBal[2];
  const int m = threadIdx.x;
  int rep = m;
  if (m < nmat) {
    const float4 x = *reinterpret_cast<const float4*>(&T.mCT[m].a0);
    bool found = false;
#pragma unroll 4
    for (int r = 0; r < m; ++r) {
      const float4 y = *reinterpret_cast<const float4*>(&T.mCT[r].a0);
      const bool eq = __float_as_uint(x.x) == __float_as_uint(y.x) && __float_as_uint(x.y) == __float_as_uint(y.y) &&
                      __float_as_uint(x.z) == __float_as_uint(y.z);
      if (eq && !found) {
        rep = r;
        found = true;
      }
    }
  }
  if (m < 64) {
    const unsigned bal = __ballot_sync(0xffffffffu, m < nmat && rep == m);
    if ((m & 31) == 0) sBal[m >> 5] = bal;
  }
  __syncthreads();
  // class id of a representative: representatives before it; of another member: its rep's
  const unsigned b0 = sBal[0], b1 = nmat > 32 ? sBal[1] : 0u;
  const int ncls = __popc(b0) + __popc(b1);
  auto cid_of_rep = [&](int r) {
    return r < 32 ? __popc(b0 & ((1u << r) - 1u)) : __popc(b0) + __popc(b1 & ((1u << (r - 32)) - 1u));
  };
  if (m < nmat) T.sCid[m] = cid_of_rep(rep);
  if (m == 0) {
    T.ncls = ncls;
    T.sCls[ncls] = nmat;
  }
  __syncthreads();
  // class c (thread c): its first member position = members of classes < c; class of the smallest
  // members first, so count the matrices whose class is below c
  if (m < ncls) {
    int start = 0;
#pragma unroll 4
    for (int r = 0; r < nmat; ++r) start += T.sCid[r] < m;
    T.sCls[m] = start;
  }
  __syncthreads();
  if (m < nmat) {
    const int c = T.sCid[m];
    int before = 0;
#pragma unroll 4
    for (int r = 0; r < m; ++r) before += T.sCid[r] == c;
    T.sMem[T.sCls[c] + before] = m;
    if (rep == m) {  // class-indexed constants from the class's smallest member
      T.sC0[c] = T.mC0[m];
      T.sCT[c] = T.mCT[m];
    }
  }
  __syncthreads();
  // per class: the largest band slope over its members, per axis (the band only has to exceed
  // every member's bound); the class test uses it too
  if (m < ncls) {
    float4 cb = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int j = T.sCls[m]; j < T.sCls[m + 1]; ++j) {
      const int r = T.sMem[j];
      cb.x = fmaxf(cb.x, T.mC0[r].c);
      cb.y = fmaxf(cb.y, T.sMA[2 * r].c);
      cb.z = fmaxf(cb.z, T.sMA[2 * r + 1].c);
    }
    T.sCB[m] = cb;
    T.sCT[m].c = cb.x;
  }
  __syncthreads();
}

// One axis of one (event, op) pair: t is the fp32 coordinate, d >= its proven error bound.  With
// lo = RD(t - d) <= t64 <= hi = RU(t + d): floor(lo) and floor(hi) come from one directed add of
// kMagic each; equal floors inside [0, n) decide the bin, hi < 0 or lo >= n decide "outside",
// anything else is left to the exact fp64 formula (-2).
__device__ __forceinline__ int axis_decide(float t, float d, float Mn, float M0 = kMagic) {
  const float rl = __fadd_rd(__fsub_rd(t, d), kMagic);
  const float rh = __fadd_rd(__fadd_ru(t, d), kMagic);
  if (rh < M0 || rl >= Mn) return -1;
  if (rl == rh && rl >= M0) return __float_as_int(rl) - __float_as_int(kMagic);
  return -2;
}

// The definition on one axis (oracle step 9): t = ((N_a0 q0 + N_a1 q1) + N_a2 q2 - lo_a) s_a in
// fp64, inside iff 0 <= t < n_a, bin floor(t) -- the same expressions as event_bin.
__device__ __forceinline__ int axis_exact(const GridC& g, const double* N, int a, float q0, float q1, float q2) {
  const double x = row_dot(N + 3 * a, (double)q0, (double)q1, (double)q2);
  const double t = dmul(dsub(x, g.lo[a]), g.s[a]);
  if (!(0.0 <= t && t < g.nd[a])) return -1;
  return __double2int_rz(t);
}

// First test-order axis of a queued (event, class): -1 outside, -2 undecided, else the bin.
__device__ __forceinline__ int class_axis0(const BinTables& T, int c, float q0, float q1, float q2, float qm) {
  const AxisF x = T.sC0[c];
  return axis_decide(axis_t(x, q0, q1, q2), fmaf(T.sCB[c].x, qm, T.bd[0]), T.bM[0], T.bL0);
}

// The remaining two axes of one member after the fp32 pass could not decide them (rare; kept
// out of line): axis_decide's verdicts from the directed bounds (rl, rh), the exact fp64 formula
// for each axis left undecided (and for the first axis when i0 = -2).
__device__ __forceinline__ int member_bin_slow(const BinParams& p, const double* N, float q0, float q1, float q2,
                                            int i0, float rl1, float rh1, float rl2, float rh2) {
  int i1 = (rl1 == rh1 && rl1 >= kMagic) ? __float_as_int(rl1) - __float_as_int(kMagic) : -2;
  int i2 = (rl2 == rh2 && rl2 >= kMagic) ? __float_as_int(rl2) - __float_as_int(kMagic) : -2;
  if (i0 == -2 && ((i0 = axis_exact(p.g, N, p.ord[0], q0, q1, q2)) < p.w0 || i0 >= p.w1)) return -1;
  if (i1 == -2 && (i1 = axis_exact(p.g, N, p.ord[1], q0, q1, q2)) < 0) return -1;
  if (i2 == -2 && (i2 = axis_exact(p.g, N, p.ord[2], q0, q1, q2)) < 0) return -1;
  return i0 * p.st[0] + i1 * p.st[1] + i2 * p.st[2];
}

// Bin of member m of class c whose first axis gave i0 (>= 0, or -2 undecided), or -1: the
// remaining two axes in fp32 inside their bands (d1, d2: the class's, for this event), and the
// exact fp64 formula for each axis left undecided -- axis_decide's rules for both axes at once,
// with one branch on the common outcome (both decided, first axis decided) and the rest out of line.
__device__ __forceinline__ int member_bin(const BinParams& p, const BinTables& T, int m, float q0, float q1,
                                          float q2, int i0, float d1, float d2, float M1, float M2, int st0,
                                          int st1, int st2) {
  const float4 f1 = T.sMF[2 * m], f2 = T.sMF[2 * m + 1];
  const float t1 = fmaf(f1.z, q2, fmaf(f1.y, q1, fmaf(f1.x, q0, -f1.w)));
  const float t2 = fmaf(f2.z, q2, fmaf(f2.y, q1, fmaf(f2.x, q0, -f2.w)));
  const float rl1 = __fadd_rd(__fsub_rd(t1, d1), kMagic), rh1 = __fadd_rd(__fadd_ru(t1, d1), kMagic);
  const float rl2 = __fadd_rd(__fsub_rd(t2, d2), kMagic), rh2 = __fadd_rd(__fadd_ru(t2, d2), kMagic);
  // axis_decide's "outside" on either axis
  if (rh1 < kMagic || rl1 >= M1 || rh2 < kMagic || rl2 >= M2) return -1;
  // both decided (not outside, equal floors: rl >= kMagic follows from rh >= kMagic)
  if (rl1 == rh1 && rl2 == rh2 && i0 >= 0)
    return i0 * st0 + (__float_as_int(rl1) - __float_as_int(kMagic)) * st1 +
           (__float_as_int(rl2) - __float_as_int(kMagic)) * st2;
  return member_bin_slow(p, T.sN + 9 * m, q0, q1, q2, i0, rl1, rh1, rl2, rh2);
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

// Decide one queued (event, class mask) entry: every member of every passing class (member_bin)
// and its reduction.  Returns the (event, op) pairs inside the grid.
template <int kPriv>
__device__ __forceinline__ unsigned drain_entry(const BinParams& p, const BinTables& T, const float4 ev, float e2,
                                                unsigned mask, bool has_err, priv_t<kPriv>* hb, priv_t<kPriv>* he) {
  using PT = priv_t<kPriv>;
  unsigned inside = 0;
  const float qm = fmaxf(fabsf(ev.y), fmaxf(fabsf(ev.z), fabsf(ev.w)));
  const float M1 = T.bM[1], M2 = T.bM[2];
  const int st0 = p.st[0], st1 = p.st[1], st2 = p.st[2];
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
    const int i0 = class_axis0(T, c, ev.y, ev.z, ev.w, qm);
    if (i0 == -1) continue;
    const float4 cb = T.sCB[c];
    const float d1 = fmaf(cb.y, qm, T.bd[1]), d2 = fmaf(cb.z, qm, T.bd[2]);
    const int j1 = T.sCls[c + 1];
#pragma unroll 2
    for (int j = T.sCls[c]; j < j1; ++j) {
      const int b = member_bin(p, T, T.sMem[j], ev.y, ev.z, ev.w, i0, d1, d2, M1, M2, st0, st1, st2);
      if (b < 0) continue;
      if constexpr (kPriv != 0) hist_add<PT>(hb, he, b, (PT)ev.x, (PT)e2, has_err);
      else hist_add(p.binmd, p.err2, b, (double)ev.x, (double)e2, has_err);
      ++inside;
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
template <int kNC, bool kPacked, bool kStats, int kPriv, bool kBoxes>
__device__ __forceinline__ void binmd_loop(const BinParams& p, const MatBlock& mb, const BinTables& T,
                                           float4* qv, unsigned* qk, float* qe, priv_t<kPriv>* hb,
                                           priv_t<kPriv>* he, unsigned long long& c_pairs,
                                           unsigned long long& c_in) {
  ClassTest<kNC> ct;
  ct.load(T);
  const int lane = threadIdx.x & 31;
  const bool has_err = !kPacked && p.col_e >= 0;
  int qhead = 0, qcnt = 0;

  // ring entries [qhead, qhead + n) (n <= 32) are decided, one per lane
  auto drain = [&](int n) {
    __syncwarp();
    if (lane < n) {
      const int slot = (qhead + lane) & (kBinQueue - 1);
      const unsigned in = drain_entry<kPriv>(p, T, qv[slot], has_err ? qe[slot] : 0.f, qk[slot], has_err, hb, he);
      if (kStats) c_in += in;
    }
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
  const int64_t n = p.nevents;
  // MDBox mode: the same interleave over the 32-event blocks of the listed boxes only
  const int64_t nvb = kBoxes ? ((int64_t)*p.box_count << p.box_log2) * 32 : n;
  // rounds of this warp, and of this lane (they differ only in the last, ragged block)
  const int rounds = base0 < nvb ? (int)((nvb - 1 - base0) / stride) + 1 : 0;
  const int lrounds = base0 + lane < n ? (int)((n - 1 - base0 - lane) / stride) + 1 : 0;
  // event of this lane in round r: e0 + r stride (64-bit only in the address arithmetic)
  const int64_t e0 = base0 + lane;
  auto ld = [&](int r, float& e2, bool& valid) {
    int64_t e;
    if constexpr (kBoxes) {
      const int64_t vb = (base0 >> 5) + (int64_t)r * (stride >> 5);  // virtual block of round r
      const int64_t bpb_mask = ((int64_t)1 << p.box_log2) - 1;
      e = r < rounds ? (((int64_t)__ldg(p.box_list + (vb >> p.box_log2)) << p.box_log2) + (vb & bpb_mask)) * 32 + lane
                     : n;
      valid = e < n;
    } else {
      e = e0 + (int64_t)r * stride;
      valid = r < lrounds;
    }
    if (valid) {
      if (has_err) e2 = __ldcs(p.events + e * p.stride + p.col_e);
      return load_event<kPacked>(p, e);
    }
    return make_float4(0.f, 0.f, 0.f, 0.f);
  };
  auto test = [&](const float4& ev, float e2, bool valid) {
    if (kStats && valid && p.w0 == 0) c_pairs += mb.nmat;  // once per event over the L2 slabs
    const float qm = fmaxf(fabsf(ev.y), fmaxf(fabsf(ev.z), fabsf(ev.w)));
    unsigned mask = ct(T, ev.y, ev.z, ev.w, qm);
    if (!valid) mask = 0;
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
  bool vd[kDepth];
#pragma unroll
  for (int u = 0; u < kDepth; ++u) ev[u] = ld(u, ex[u], vd[u]);
  for (int r = 0;;) {
#pragma unroll
    for (int u = 0; u < kDepth; ++u) {
      if (r >= rounds) goto done;
      test(ev[u], ex[u], vd[u]);
      ev[u] = ld(r + kDepth, ex[u], vd[u]);
      ++r;
    }
    // one drain site per kDepth blocks (the ring holds kDepth x 32 + 31 entries): the member code
    // is emitted once, not once per unrolled block
    while (qcnt >= 32) drain(32);
  }
done:
  while (qcnt > 0) drain(min(qcnt, 32));
}

// B0 once per launch: compose N_s and build the tables (one CTA), into global memory.
__global__ void __launch_bounds__(kThreads) binmd_plan_kernel(const __grid_constant__ BinParams p,
                                                              const __grid_constant__ MatBlock mb, BinTables* out) {
  __shared__ BinTables T;
  build_tables(p, mb, T);
  const float4* src = reinterpret_cast<const float4*>(&T);
  float4* dst = reinterpret_cast<float4*>(out);
  for (int i = threadIdx.x; i < (int)(kTablesUsed / 16); i += blockDim.x) dst[i] = src[i];
}

// The launch's tables from global memory (L2-resident, written by the plan kernel) into shared
// memory: 16-byte coalesced loads by the whole CTA.
__device__ __forceinline__ void load_tables(const void* g, BinTables& T) {
  const float4* src = static_cast<const float4*>(g);
  float4* dst = reinterpret_cast<float4*>(&T);
  for (int i = threadIdx.x; i < (int)(kTablesUsed / 16); i += blockDim.x) dst[i] = __ldcg(src + i);
  __syncthreads();
}

// One thread per event (grid-stride).  kPriv: 0 = global fp64 red.add, 1 / 2 = a private fp64 /
// fp32 histogram per CTA in shared memory (binmd, then err2 when the error column is read),
// flushed into the global one at the end.
template <bool kPacked, bool kStats, int kPriv, bool kBoxes = false>
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
  // a kernel launched after BinMD with programmatic dependent launch (the MDNorm cull in the
  // bench step order, or the divide) may start its CTAs on the SMs this grid's CTAs leave; it
  // executes griddepcontrol.wait before anything that depends on this grid (the divide before
  // reading the histograms, the cull at its very end) -- this trigger only allows the early start
  asm volatile("griddepcontrol.launch_dependents;");
  load_tables(p.tables, T);
  const int w = threadIdx.x >> 5;
  float4* qv = sQv + w * kBinQueue;
  unsigned* qk = sQk + w * kBinQueue;
  float* qe = sQe + w * kBinQueue;
  unsigned long long c_pairs = 0, c_in = 0;
  const int ncls = T.ncls;
  if (ncls <= 1)
    binmd_loop<1, kPacked, kStats, kPriv, kBoxes>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
  else if (ncls <= 2)
    binmd_loop<2, kPacked, kStats, kPriv, kBoxes>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
  else
    binmd_loop<0, kPacked, kStats, kPriv, kBoxes>(p, mb, T, qv, qk, qe, hb, he, c_pairs, c_in);
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
    if (fabsf(axis_t(x, q0, q1, q2)) < fmaf(x.c, qm, x.d)) {
      const int i0 = class_axis0(T, c, q0, q1, q2, qm);
      const float4 cb = T.sCB[c];
      if (i0 != -1)
        b = member_bin(p, T, m, q0, q1, q2, i0, fmaf(cb.y, qm, T.bd[1]), fmaf(cb.z, qm, T.bd[2]), T.bM[1], T.bM[2],
                       p.st[0], p.st[1], p.st[2]);
    }
    bins[t] = b;
  }
}

// ---------------------------------------------------------------- NEXT #4: MDBox extents
// Q extents of boxes of box_events consecutive packed events (the last box may be shorter): one
// warp per box, coalesced float4 loads, warp min / max.  bounds[6 b ..] = (min q0, q1, q2, max q0,
// q1, q2).
__global__ void __launch_bounds__(kThreads) binmd_box_bounds_kernel(const float4* __restrict__ ev, int64_t n,
                                                                    int32_t box_events, float* __restrict__ bounds,
                                                                    int64_t nboxes) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t b = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); b < nboxes; b += nw) {
    float lo0 = CUDART_INF_F, lo1 = CUDART_INF_F, lo2 = CUDART_INF_F;
    float hi0 = -CUDART_INF_F, hi1 = -CUDART_INF_F, hi2 = -CUDART_INF_F;
    const int64_t e1 = min(n, (b + 1) * (int64_t)box_events);
    for (int64_t e = b * (int64_t)box_events + lane; e < e1; e += 32) {
      const float4 v = __ldcs(ev + e);
      lo0 = fminf(lo0, v.y); lo1 = fminf(lo1, v.z); lo2 = fminf(lo2, v.w);
      hi0 = fmaxf(hi0, v.y); hi1 = fmaxf(hi1, v.z); hi2 = fmaxf(hi2, v.w);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      lo0 = fminf(lo0, __shfl_xor_sync(kFull, lo0, o)); lo1 = fminf(lo1, __shfl_xor_sync(kFull, lo1, o));
      lo2 = fminf(lo2, __shfl_xor_sync(kFull, lo2, o)); hi0 = fmaxf(hi0, __shfl_xor_sync(kFull, hi0, o));
      hi1 = fmaxf(hi1, __shfl_xor_sync(kFull, hi1, o)); hi2 = fmaxf(hi2, __shfl_xor_sync(kFull, hi2, o));
    }
    if (lane < 6) bounds[6 * b + lane] = lane == 0 ? lo0 : lane == 1 ? lo1 : lane == 2 ? lo2 : lane == 3 ? hi0 : lane == 4 ? hi1 : hi2;
  }
}

// The boxes whose extent can reach the grid under some matrix of the launch (thread per box):
// x_a = N_a . q over the box is enclosed by [sum_i min(N_ai lo_i, N_ai hi_i), sum_i max(..)] in
// fp64; the box is dropped only when, for every matrix, some axis has t = (x - lo) s entirely
// below -eps or at or above n + eps (eps = 1e-6 (n + |lo s| + 1): far beyond the rounding of the
// fp64 enclosure and of the definition's own t).  Survivors are appended in any order.
__global__ void __launch_bounds__(kThreads) binmd_box_cull_kernel(const __grid_constant__ BinParams p,
                                                                  const float* __restrict__ bounds, int64_t nboxes,
                                                                  int32_t* __restrict__ list,
                                                                  unsigned* __restrict__ count) {
  __shared__ double sN[kMaxMats * 9];
  __shared__ int snmat;
  const BinTables* gt = static_cast<const BinTables*>(p.tables);
  if (threadIdx.x == 0) snmat = gt->sCls[gt->ncls];  // number of matrices (sCls[ncls] = nmat)
  __syncthreads();
  const int nmat = snmat;
  for (int i = threadIdx.x; i < 9 * nmat; i += blockDim.x) sN[i] = gt->sN[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t b0 = (int64_t)blockIdx.x * blockDim.x; b0 < nboxes; b0 += stride) {
    const int64_t b = b0 + threadIdx.x;
    bool keep = false;
    if (b < nboxes) {
      double lo[3], hi[3];
      for (int i = 0; i < 3; ++i) {
        lo[i] = (double)bounds[6 * b + i];
        hi[i] = (double)bounds[6 * b + 3 + i];
      }
      // no finite-Q event (fminf / fmaxf skip NaN): every event of the box is outside by definition
      const bool empty = !(lo[0] <= hi[0]);
      if (!empty) {
        for (int m = 0; m < nmat && !keep; ++m) {
          bool miss = false;
          for (int a = 0; a < 3 && !miss; ++a) {
            const double* r = sN + 9 * m + 3 * a;
            double xl = 0.0, xh = 0.0;
            for (int i = 0; i < 3; ++i) {
              const double u = r[i] * lo[i], v = r[i] * hi[i];
              xl += fmin(u, v);
              xh += fmax(u, v);
            }
            const double s = p.g.s[a], l = p.g.lo[a], nb = p.g.nd[a];
            const double eps = 1e-6 * (nb + fabs(l * s) + 1.0);
            const double tl = (xl - l) * s, th = (xh - l) * s;
            miss = th < -eps || tl >= nb + eps;  // NaN compares false: kept
          }
          keep = !miss;
        }
      }
    }
    const unsigned bal = __ballot_sync(kFull, keep);
    unsigned at = 0;
    if (lane == 0 && bal) at = atomicAdd(count, (unsigned)__popc(bal));
    at = __shfl_sync(kFull, at, 0);
    if (keep) list[at + __popc(bal & ((1u << lane) - 1u))] = (int32_t)b;
  }
}

template <bool kPacked, bool kStats, int kPriv, bool kBoxes = false>
cudaError_t launch_binmd_t(const BinParams& p, const MatBlock& mb, int num_sms, size_t smem, cudaStream_t s) {
  constexpr int threads = bin_threads(kPriv);
  auto k = binmd_kernel<kPacked, kStats, kPriv, kBoxes>;
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
  if (p.box_list)  // MDBox mode: packed float4 events only (checked by the API)
    return p.stats ? launch_binmd_t<true, true, kPriv, true>(p, mb, num_sms, smem, s)
                   : launch_binmd_t<true, false, kPriv, true>(p, mb, num_sms, smem, s);
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


size_t binmd_tables_bytes() { return sizeof(BinTables); }

cudaError_t launch_binmd_box_bounds(const float4* events, int64_t nevents, int32_t box_events, float* bounds,
                                    int num_sms, cudaStream_t s) {
  const int64_t nboxes = (nevents + box_events - 1) / box_events;
  if (nboxes <= 0) return cudaSuccess;
  binmd_box_bounds_kernel<<<grid_for(nboxes * 32, num_sms, 8), kThreads, 0, s>>>(events, nevents, box_events,
                                                                                 bounds, nboxes);
  return cudaGetLastError();
}

cudaError_t launch_binmd_box_cull(const BinParams& p, const float* bounds, int64_t nboxes, int32_t* list,
                                  unsigned* count, int num_sms, cudaStream_t s) {
  if (nboxes <= 0) return cudaSuccess;
  binmd_box_cull_kernel<<<grid_for(nboxes, num_sms, 4), kThreads, 0, s>>>(p, bounds, nboxes, list, count);
  return cudaGetLastError();
}

cudaError_t launch_binmd_plan(const BinParams& p, const MatBlock& mb, void* tables, cudaStream_t s) {
  binmd_plan_kernel<<<1, kThreads, 0, s>>>(p, mb, static_cast<BinTables*>(tables));
  return cudaGetLastError();
}

cudaError_t launch_debug_bins(const BinParams& p, const MatBlock& mb, int64_t* bins, cudaStream_t s) {
  if (p.nevents <= 0) return cudaSuccess;
  debug_bins_kernel<<<grid_for(p.nevents * mb.nmat, 148, 8), kThreads, 0, s>>>(p, mb, bins);
  return cudaGetLastError();
}

}  // namespace mdn
