// mdn_device.cuh -- device-side building blocks of the MDNorm / BinMD hot path (sm_100a).
//
// Every value that decides a crossing, a clip, a midpoint, a bin index or a flux value is IEEE
// fp64 with explicit round-to-nearest intrinsics (__dmul_rn, __dadd_rn, __ddiv_rn), so no
// multiply-add is ever contracted into an FMA and the results are bit-identical to the paper's
// definition as DESIGN.md §3 fixes it.  The translation unit is
// also compiled with --fmad=false as a guard.
//
// Citations: PAPER.md P:n.  M0-M7, B0-B3, X2 = the rows of SURVEY.md §8(a).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <math_constants.h>

namespace mdn {

// ------------------------------------------------------------------------------ grid constants
// w_a = (hi_a - lo_a) / n_a, s_a = 1 / w_a, computed once on the host in IEEE double (x86-64
// SSE2: the same bits the device would produce).  Edge e_{a,j} = lo_a + j * w_a.
struct GridC {
  double lo[3], hi[3], w[3], s[3];
  double nd[3];  // n_a as double (the "t < n_a" tests)
  int32_t n[3];
  int32_t pad;
  int64_t nbins;
};

__device__ __forceinline__ double dmul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ double dadd(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ double dsub(double a, double b) { return __dadd_rn(a, -b); }
__device__ __forceinline__ double ddiv(double a, double b) { return __ddiv_rn(a, b); }

// ((r0 q0 + r1 q1) + r2 q2): M1 / B2 row product, fixed order, no FMA.
__device__ __forceinline__ double row_dot(const double* r, double q0, double q1, double q2) {
  return dadd(dadd(dmul(r[0], q0), dmul(r[1], q1)), dmul(r[2], q2));
}

__device__ __forceinline__ double edge(const GridC& g, int a, int j) {
  return dadd(g.lo[a], dmul((double)j, g.w[a]));
}

// ------------------------------------------------------------------------------ M0 / B0
// C = A * B (row-major 3x3), element ((a0 b0 + a1 b1) + a2 b2).
__device__ __forceinline__ void matmul3(const double* A, const double* B, double* C) {
#pragma unroll
  for (int i = 0; i < 3; ++i)
#pragma unroll
    for (int j = 0; j < 3; ++j)
      C[3 * i + j] = dadd(dadd(dmul(A[3 * i + 0], B[j]), dmul(A[3 * i + 1], B[3 + j])),
                          dmul(A[3 * i + 2], B[6 + j]));
}

// RN(a / b) from y = RN(1 / b) by Markstein's correction: q = RN(a y) is within one ulp of a / b,
// r = a - q b is exact (one FMA) and RN(q + r y) is the correctly rounded quotient -- the same
// argument as the flux interpolation below (tests/test_flux_division.py pins it).  Valid when a,
// b and a / b are normal and far from overflow; callers check the range and otherwise divide.  A
// zero numerator gives the quotient's signed zero directly.
__device__ __forceinline__ double div_rn_recip(double a, double b, double y) {
  if (a == 0.0) return dmul(a, y);
  const double q = dmul(a, y);
  const double r = __fma_rn(-q, b, a);
  return __fma_rn(r, y, q);
}

__device__ __forceinline__ bool recip_range(double x) {
  const double ax = fabs(x);
  return ax == 0.0 || (ax > 0x1p-400 && ax < 0x1p400);
}

// out = adj(C)/det * scale, out_ij = (cof_ji / det) * scale.  Returns false if singular.  The nine
// quotients share one IEEE reciprocal of det (div_rn_recip; bit-identical to nine divisions).
__device__ __forceinline__ bool inv3_scaled(const double* C, double scale, double* out) {
  double cof[9];
  cof[0] = dsub(dmul(C[4], C[8]), dmul(C[5], C[7]));
  cof[1] = dsub(dmul(C[5], C[6]), dmul(C[3], C[8]));
  cof[2] = dsub(dmul(C[3], C[7]), dmul(C[4], C[6]));
  cof[3] = dsub(dmul(C[2], C[7]), dmul(C[1], C[8]));
  cof[4] = dsub(dmul(C[0], C[8]), dmul(C[2], C[6]));
  cof[5] = dsub(dmul(C[1], C[6]), dmul(C[0], C[7]));
  cof[6] = dsub(dmul(C[1], C[5]), dmul(C[2], C[4]));
  cof[7] = dsub(dmul(C[2], C[3]), dmul(C[0], C[5]));
  cof[8] = dsub(dmul(C[0], C[4]), dmul(C[1], C[3]));
  double det = dadd(dadd(dmul(C[0], cof[0]), dmul(C[1], cof[1])), dmul(C[2], cof[2]));
  if (det == 0.0 || !isfinite(det)) return false;
  const double y = ddiv(1.0, det);
  bool fast = recip_range(det);
#pragma unroll
  for (int i = 0; i < 9; ++i) fast = fast && recip_range(cof[i]);
  if (fast) {
#pragma unroll
    for (int i = 0; i < 3; ++i)
#pragma unroll
      for (int j = 0; j < 3; ++j) out[3 * i + j] = dmul(div_rn_recip(cof[3 * j + i], det, y), scale);
  } else {
    for (int i = 0; i < 3; ++i)
      for (int j = 0; j < 3; ++j) out[3 * i + j] = dmul(ddiv(cof[3 * j + i], det), scale);
  }
  return true;
}

// RN(1 / RN(2 pi)) (0x3fc45f306dc9c883), the constant the oracle's 1.0 / (2.0 * pi) evaluates to
__device__ __forceinline__ double inv_two_pi() { return __hiloint2double(0x3fc45f30, 0x6dc9c883); }

// M_{r,s} = (R UB S W)^-1 / (2 pi)   (reading #1-#2; rotations P:80, per-op 3x3 P:143/148)
__device__ __forceinline__ bool compose_mdnorm(const double* R, const double* UB, const double* S,
                                               const double* W, double* M) {
  double A[9], B[9], C[9];
  matmul3(R, UB, A);
  matmul3(A, S, B);
  matmul3(B, W, C);
  return inv3_scaled(C, inv_two_pi(), M);
}

// N_s = (UB S W)^-1 / (2 pi)   (events already in Q_sample)
__device__ __forceinline__ bool compose_binmd(const double* UB, const double* S, const double* W,
                                              double* N) {
  double B[9], C[9];
  matmul3(UB, S, B);
  matmul3(B, W, C);
  return inv3_scaled(C, inv_two_pi(), N);
}

// ------------------------------------------------------------------------------ M5 flux
// F(x): clamp outside, else i = max{i : kappa_i <= x} and
//   Phi_i + (Phi_{i+1} - Phi_i) * ((x - kappa_i) / (kappa_{i+1} - kappa_i)).
//
// Per interval the table stores ka_i = (kappa_i, Phi_i) and kb_i = (dPhi_i, y_i) with dPhi_i =
// RN(Phi_{i+1} - Phi_i) and y_i = RN(1 / dk_i), dk_i = RN(kappa_{i+1} - kappa_i) (the same
// roundings as the formula; dk_i is recomputed from the knots).  The correctly rounded quotient
// a / dk_i (a = RN(x - kappa_i)) is then
//   q = RN(a y_i);  r = a - q dk_i (exact, one FMA);  q' = RN(q + r y_i)   (one FMA)
// -- Markstein's theorem: y within half an ulp of 1/b and q within one ulp of a/b make r exact
// and q' = RN(a/b) (no overflow / underflow here: 0 <= a < dk, both normal or zero).  Three
// fp64 instructions instead of an IEEE division; tests/test_flux_division.py pins the claim on
// 2e7 random and adversarial operands against IEEE division.
//
// Search: U(x) = RN(RN(x - kappa_0) * inv_cell) is monotone non-decreasing in x, and the host
// evaluates the same expression U_i = U(kappa_i).  For x with floor(U(x)) = c:
//   every knot with U_i < c is < x, and every knot with U_i >= c + 1 is > x,
// so with s_c = max{i : U_i < c}, i is s_c plus the number of knots of cell c that are <= x:
// probe kappa_{s_c+1}, kappa_{s_c+2}, ... until the first knot > x (which is kappa_{i+1}, the
// knot dk_i needs).  The common case -- no knot of cell c at or below x -- needs one probe, and
// the interval records are loaded alongside it; cells are MDN_FLUX_CELLS (8) per knot (or
// narrower), so a probe finds a knot <= x for a small fraction of the look-ups.  Cells with more
// than three knots (and c = 0, x outside the table, or c + 1 > U_{n-1}) are flagged and take the
// general path: clamps and a bisection.  A fast cell lies below U_{n-1}, so its probes stop at
// kappa_{n-1} at the latest: they read kappa_{i+1} from the next interval record (ka[n-1] holds
// kappa_{n-1}), and the shared-memory copy needs no separate knot array (the freed 32 KB pay for
// the 8 cells per knot: measured 1-2% faster walk than 4 cells + knots).
// The general path bisects the global knot array (two +inf pads).
//
// Shared-memory layout (bank conflicts of random look-ups, measured: profiles/): the two records as separate
// 16-byte-strided double2 arrays (all 8 sixteen-byte bank groups), instead of one 32-byte record
// per interval (which uses only 4 of the 8 groups).
#ifndef MDN_FLUX_CELLS
#define MDN_FLUX_CELLS 8  // cell-table cells per knot (at least); measured 8 > 6 > 4 with MDN_FLUX_NOKN
#endif
constexpr unsigned kFluxDense32 = 1u << 30;  // flag bit in an int32 table entry
constexpr unsigned kFluxDense16 = 1u << 15;  // flag bit in a uint16 (shared-memory) entry

struct FluxView {
  const double* kn;    // kappa_i: n knots + 2 (+inf) pads
  const double2* ka;   // per interval i < n - 1: (kappa_i, Phi_i); n entries
  const double2* kb;   // per interval i < n - 1: (dPhi_i, y_i); n entries
  const void* tab;     // ntab cell entries: int32 (global) or uint16 (shared-memory copy)
  double k_first, F_first, k_last, F_last, inv_cell;
  int n, ntab;
  // interval guess (0: none; 1: knots near-uniform in k; 2: near-uniform in 1/k, i.e. in
  // wavelength): i ~ floor(fma(T(x), ga, gb)) in fp32, T(x) = x or 1/x
  float ga, gb;
  int gmode;
  // shared-window addresses of ka and kb (shared-memory copy only): the look-up adds 16 i instead
  // of converting a generic pointer on every call
  unsigned ska, skb;
  // the cell table as the uint16 entries of the shared-memory copy (zero padded to a multiple of
  // 8 entries), or nullptr when an entry does not fit 15 bits
  const uint16_t* tab16;
};

template <typename TabT>
__device__ __forceinline__ unsigned tab_entry(const FluxView& f, int c) {
  return (unsigned)static_cast<const TabT*>(f.tab)[c];
}

// Phi_i + dPhi_i * RN((x - kappa_i) / dk_i) for kappa_i <= x < kappa_{i+1} = kn1
__device__ __forceinline__ double flux_interp(double x, double2 a, double2 b, double kn1) {
  const double d = dsub(x, a.x);
  const double dk = dsub(kn1, a.x);
  const double q = dmul(d, b.y);
  const double r = __fma_rn(-q, dk, d);
  const double t = __fma_rn(r, b.y, q);
  return dadd(a.y, dmul(b.x, t));
}

__device__ __forceinline__ double flux_general(const FluxView& f, double x) {
  if (x <= f.k_first) return f.F_first;
  if (x >= f.k_last) return f.F_last;
  // largest i in [0, n - 2] with kappa_i <= x (kappa_0 < x < kappa_{n-1})
  int lo = 0, len = f.n - 1;
  while (len > 1) {
    const int half = len >> 1;
    if (f.kn[lo + half] <= x) lo += half;
    len -= half;
  }
  return flux_interp(x, f.ka[lo], f.kb[lo], f.kn[lo + 1]);
}

// Guessed interval (set_flux picks the mode when the guess is right for most of the k range):
// the guess is only a candidate -- it is accepted iff kappa_i <= x < kappa_{i+1} (and x >
// kappa_0), which identifies the same unique interval the search finds (knots strictly
// increase), so the value is the search path's bit for bit.  It replaces the cell-table load
// and its dependent record loads with three independent loads (ka_i, kb_i, kappa_{i+1}).
template <typename TabT>
__device__ __forceinline__ bool flux_guess(const FluxView& f, double x, double& F) {
  const float xf = __double2float_rn(x);
  float u = xf;
  if (f.gmode == 2) asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(u) : "f"(xf));
  int i = __float2int_rd(__fmaf_rn(u, f.ga, f.gb));
  i = min(max(i, 0), f.n - 2);
  double2 a, b;
  double kn1;
  if constexpr (sizeof(TabT) == 2) {
    // shared-memory records: the three loads are issued together, before the acceptance test
    // (left to itself the compiler sinks the kb load behind it: one more dependent round trip)
    const unsigned sa = f.ska + 16u * (unsigned)i;
    const unsigned sb = f.skb + 16u * (unsigned)i;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(a.x), "=d"(a.y) : "r"(sa));
    asm volatile("ld.shared.f64 %0, [%1+16];" : "=d"(kn1) : "r"(sa));
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(b.x), "=d"(b.y) : "r"(sb));
  } else {
    a = f.ka[i];
    b = f.kb[i];
    kn1 = f.ka[i + 1].x;
  }
  if (a.x <= x && x < kn1 && x > f.k_first) {
    F = flux_interp(x, a, b, kn1);
    return true;
  }
  return false;
}

template <typename TabT = int>
__device__ __forceinline__ double flux_at(const FluxView& f, double x) {
  constexpr unsigned flag = sizeof(TabT) == 2 ? kFluxDense16 : kFluxDense32;
  if (f.gmode != 0) {
    double F;
    if (flux_guess<TabT>(f, x, F)) return F;
  }
  const int c = __double2int_rd(dmul(dsub(x, f.k_first), f.inv_cell));
  const unsigned e = (unsigned)c < (unsigned)f.ntab ? tab_entry<TabT>(f, c) : flag;
  if (e & flag) return flux_general(f, x);
  int i = (int)e;
  // kappa_{i+1} from the next interval record: the fast path never looks past kappa_{n-1} (its
  // cells end below U_{n-1})
  double kn1 = f.ka[i + 1].x;
  double2 a = f.ka[i], b = f.kb[i];
  if (kn1 <= x) {  // a knot of cell c lies at or below x (at most three)
    do {
      ++i;
      kn1 = f.ka[i + 1].x;
    } while (kn1 <= x);
    a = f.ka[i];
    b = f.kb[i];
  }
  return flux_interp(x, a, b, kn1);
}

// ------------------------------------------------------------------------------ M1-M2
// v = M q (q = z - d precomputed per pixel), clip [k_min, k_max] to the box slab by slab.
// r[a] = RN(1 / v[a]) for v[a] != 0 (any value for v[a] == 0)
__device__ __forceinline__ bool traj_clip_r(const GridC& g, const double v[3], const double r[3], double kmin,
                                            double kmax, double& kin, double& kout) {
  kin = kmin;
  kout = kmax;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    double lk, hk;
    if (v[a] > 0.0) {
      lk = dmul(g.lo[a], r[a]);
      hk = dmul(g.hi[a], r[a]);
    } else if (v[a] < 0.0) {
      lk = dmul(g.hi[a], r[a]);
      hk = dmul(g.lo[a], r[a]);
    } else {
      if (g.lo[a] <= 0.0 && 0.0 < g.hi[a]) continue;
      return false;
    }
    if (lk > kin) kin = lk;
    if (hk < kout) kout = hk;
  }
  return kin < kout;
}

__device__ __forceinline__ bool traj_clip(const GridC& g, const double v[3], double kmin,
                                          double kmax, double& kin, double& kout) {
  const double r[3] = {v[0] != 0.0 ? ddiv(1.0, v[0]) : 0.0, v[1] != 0.0 ? ddiv(1.0, v[1]) : 0.0,
                       v[2] != 0.0 ? ddiv(1.0, v[2]) : 0.0};
  return traj_clip_r(g, v, r, kmin, kmax, kin, kout);
}

// ------------------------------------------------------------------------------ M3
// Plane crossings of axis a: J = {j in [1, n-1] : lo_k < e_j * r < hi_k} with r = 1/v.
// f(j) = e_j * r is monotone in j (rounding is monotone), so J is one contiguous index range:
// the region-of-interest replacement of the paper's linear plane loops.
// The range is estimated from the continuous grid coordinate and fixed up by exact tests of
// f(j) itself, so J is exactly the oracle's set.  The stream yields J in increasing k:
// first index j, count cnt, step +1 (v > 0) or -1 (v < 0).
struct AxisStream {
  int j, cnt, step;
};

__device__ __forceinline__ double plane_k(const GridC& g, int a, int j, double r) {
  return dmul(edge(g, a, j), r);
}

__device__ __forceinline__ int clamp_floor(double u, int lo, int hi) {
  double f = floor(u);
  f = fmax(f, (double)lo - 1.0);
  f = fmin(f, (double)hi + 1.0);
  int x = (int)f;
  return x < lo ? lo : (x > hi ? hi : x);
}

__device__ __forceinline__ AxisStream axis_stream(const GridC& g, int a, double v, double r,
                                                  double kin, double kout) {
  AxisStream s{0, 0, 1};
  const int n = g.n[a];
  if (v == 0.0 || n < 2) return s;
  // approximate continuous coordinates (any rounding; only used as a starting guess)
  double u_in = (kin * v - g.lo[a]) * g.s[a];
  double u_out = (kout * v - g.lo[a]) * g.s[a];
  if (v > 0.0) {
    // jlo = first j with f(j) > kin (f increasing)
    int j = clamp_floor(u_in + 1.0, 1, n);
    while (j > 1 && plane_k(g, a, j - 1, r) > kin) --j;
    while (j <= n - 1 && !(plane_k(g, a, j, r) > kin)) ++j;
    int jlo = j;
    // jhi = last j with f(j) < kout
    j = clamp_floor(u_out, 0, n - 1);
    while (j < n - 1 && plane_k(g, a, j + 1, r) < kout) ++j;
    while (j >= 1 && !(plane_k(g, a, j, r) < kout)) --j;
    s.j = jlo;
    s.cnt = j >= jlo ? j - jlo + 1 : 0;
    s.step = 1;
  } else {
    // f decreasing: increasing k visits descending j.  jA = last j with f(j) > kin.
    int j = clamp_floor(u_in, 0, n - 1);
    while (j < n - 1 && plane_k(g, a, j + 1, r) > kin) ++j;
    while (j >= 1 && !(plane_k(g, a, j, r) > kin)) --j;
    int jA = j;
    // jB = first j with f(j) < kout
    j = clamp_floor(u_out + 1.0, 1, n);
    while (j > 1 && plane_k(g, a, j - 1, r) < kout) --j;
    while (j <= n - 1 && !(plane_k(g, a, j, r) < kout)) ++j;
    s.j = jA;
    s.cnt = jA >= j ? jA - j + 1 : 0;
    s.step = -1;
  }
  return s;
}

// The starting guesses of axis_stream without its exact fix-up (within one plane of the exact
// range at either end; the cull's piece plan only needs that).
__device__ __forceinline__ AxisStream axis_estimate(const GridC& g, int a, double v, double kin, double kout) {
  AxisStream s{0, 0, 1};
  const int n = g.n[a];
  if (v == 0.0 || n < 2) return s;
  const double u_in = (kin * v - g.lo[a]) * g.s[a];
  const double u_out = (kout * v - g.lo[a]) * g.s[a];
  if (v > 0.0) {
    const int jlo = clamp_floor(u_in + 1.0, 1, n), jhi = clamp_floor(u_out, 0, n - 1);
    s.j = jlo;
    s.cnt = jhi >= jlo ? jhi - jlo + 1 : 0;
  } else {
    const int jA = clamp_floor(u_in, 0, n - 1), jB = clamp_floor(u_out + 1.0, 1, n);
    s.j = jA;
    s.cnt = jA >= jB ? jA - jB + 1 : 0;
    s.step = -1;
  }
  return s;
}

// One axis of the merge: reciprocal, position (j kept as an exact double so that the edge
// lo + j * w needs no int->double conversion), remaining count, next crossing value.
struct AxisCursor {
  double r, nk, jd, stepd;
  int cnt;
};

__device__ __forceinline__ void cursor_init(AxisCursor& c, const GridC& g, int a, double v, double lo_k,
                                            double hi_k) {
  c.r = v != 0.0 ? ddiv(1.0, v) : 0.0;
  const AxisStream s = axis_stream(g, a, v, c.r, lo_k, hi_k);
  c.jd = (double)s.j;
  c.stepd = (double)s.step;
  c.cnt = s.cnt;
  c.nk = s.cnt > 0 ? dmul(dadd(g.lo[a], dmul(c.jd, g.w[a])), c.r) : CUDART_INF;
}

// ------------------------------------------------------------------------------ B2-B3
// Bin of event Q (fp32 input widened to fp64) under N: x_a = ((N_a0 q0 + N_a1 q1) + N_a2 q2),
// t_a = (x_a - lo_a) s_a, inside iff 0 <= t_a < n_a for every a.  -1 = outside.
__device__ __forceinline__ int64_t event_bin(const GridC& g, const double* N, double q0, double q1,
                                             double q2) {
  int idx[3];
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    double x = row_dot(N + 3 * a, q0, q1, q2);
    double t = dmul(dsub(x, g.lo[a]), g.s[a]);
    if (!(0.0 <= t && t < g.nd[a])) return -1;
    idx[a] = __double2int_rz(t);
  }
  return (int64_t)idx[0] + (int64_t)g.n[0] * ((int64_t)idx[1] + (int64_t)g.n[1] * idx[2]);
}

}  // namespace mdn
