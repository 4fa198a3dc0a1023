// mdn_device.cuh -- device-side building blocks of the MDNorm / BinMD hot path (sm_100a).
//
// Every function here is IEEE fp64 with explicit round-to-nearest intrinsics (__dmul_rn,
// __dadd_rn, __dsub_rn, __ddiv_rn), so no multiply-add is ever contracted into an FMA and the
// crossing values, midpoints, bin indices and flux values are bit-identical to the paper's
// definition as DESIGN.md §3 fixes it.  The translation unit is
// additionally compiled with --fmad=false as a guard.
//
// Citations: PAPER.md P:n.  M0-M7, B0-B3, X2 = the rows of SURVEY.md §8(a).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <math_constants.h>

namespace mdn {

// ------------------------------------------------------------------------------ grid constants
// w_a = (hi_a - lo_a) / n_a, s_a = 1 / w_a, computed once on the host in IEEE double (identical
// to the device result; x86-64 SSE2).  Edge e_{a,j} = lo_a + j * w_a (product, then sum).
struct GridC {
  double lo[3], hi[3], w[3], s[3];
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

// out = adj(C)/det * scale, out_ij = (cof_ji / det) * scale.  Returns false if singular.
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
#pragma unroll
  for (int i = 0; i < 3; ++i)
#pragma unroll
    for (int j = 0; j < 3; ++j) out[3 * i + j] = dmul(ddiv(cof[3 * j + i], det), scale);
  return true;
}

__device__ __forceinline__ double inv_two_pi() { return ddiv(1.0, dmul(2.0, CUDART_PI)); }

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
// F(x): clamp outside, else i = max{i : k_i <= x} (unique, so any search order gives the same i)
// and Phi_i + (Phi_{i+1} - Phi_i) * ((x - k_i) / (k_{i+1} - k_i)).
struct FluxView {
  const double* k;
  const double* F;
  int n;
};

__device__ __forceinline__ double flux_at(const FluxView& f, double x) {
  if (x <= f.k[0]) return f.F[0];
  if (x >= f.k[f.n - 1]) return f.F[f.n - 1];
  int lo = 0, hi = f.n - 1;  // invariant k[lo] <= x < k[hi]
  while (hi - lo > 1) {
    int mid = (lo + hi) >> 1;
    if (f.k[mid] <= x)
      lo = mid;
    else
      hi = mid;
  }
  double k0 = f.k[lo], k1 = f.k[lo + 1], F0 = f.F[lo], F1 = f.F[lo + 1];
  return dadd(F0, dmul(dsub(F1, F0), ddiv(dsub(x, k0), dsub(k1, k0))));
}

// ------------------------------------------------------------------------------ M1-M2
// v = M q (q = z - d precomputed per pixel), clip [k_min, k_max] to the box slab by slab.
__device__ __forceinline__ bool traj_clip(const GridC& g, const double v[3], double kmin,
                                          double kmax, double& kin, double& kout) {
  kin = kmin;
  kout = kmax;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    double lk, hk;
    if (v[a] > 0.0) {
      double r = ddiv(1.0, v[a]);
      lk = dmul(g.lo[a], r);
      hk = dmul(g.hi[a], r);
    } else if (v[a] < 0.0) {
      double r = ddiv(1.0, v[a]);
      lk = dmul(g.hi[a], r);
      hk = dmul(g.lo[a], r);
    } else {
      if (g.lo[a] <= 0.0 && 0.0 < g.hi[a]) continue;
      return false;
    }
    if (lk > kin) kin = lk;
    if (hk < kout) kout = hk;
  }
  return kin < kout;
}

// ------------------------------------------------------------------------------ M3
// Plane crossings of axis a: J = {j in [1, n-1] : kin < e_j * r < kout} with r = 1/v.
// f(j) = e_j * r is monotone in j (rounding is monotone), so J is one contiguous index range:
// the region-of-interest replacement of the paper's linear plane loops.
// The range is estimated from the continuous grid coordinate and fixed up by exact tests of
// f(j) itself, so J is exactly the oracle's set.  Output: first index in increasing-k order,
// count, and step (+1 if v > 0, -1 if v < 0).
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
    int jhi = j;
    s.j = jlo;
    s.cnt = jhi >= jlo ? jhi - jlo + 1 : 0;
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
    int jB = j;
    s.j = jA;
    s.cnt = jA >= jB ? jA - jB + 1 : 0;
    s.step = -1;
  }
  return s;
}

// ------------------------------------------------------------------------------ M4-M7
// Walk one clipped trajectory: a 3-way streaming merge of the per-axis monotone crossing
// sequences (replaces the paper's sort, and the GPU comb sort, with no buffer),
// flux at each list entry (M5), midpoint bin of every positive-length segment (M6) and
// emit(b, (F(k2) - F(k1)) * omega_c) (M7).  Returns n_seg; *ncross = |L| = 2 + crossings.
template <class Emit>
__device__ __forceinline__ int traj_walk(const GridC& g, const FluxView& fx, const double v[3],
                                         double kin, double kout, double omega_c, Emit& emit,
                                         int* ncross) {
  double r[3], nk[3];
  AxisStream st[3];
  int total = 0;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    r[a] = v[a] != 0.0 ? ddiv(1.0, v[a]) : 0.0;
    st[a] = axis_stream(g, a, v[a], r[a], kin, kout);
    total += st[a].cnt;
    nk[a] = st[a].cnt > 0 ? plane_k(g, a, st[a].j, r[a]) : CUDART_INF;
  }
  *ncross = total + 2;
  double k1 = kin, F1 = flux_at(fx, kin);
  int nseg = 0;
  for (int left = total;; --left) {
    double k2;
    if (left > 0) {
      int a = 0;
      k2 = nk[0];
      if (nk[1] < k2) { a = 1; k2 = nk[1]; }
      if (nk[2] < k2) { a = 2; k2 = nk[2]; }
      st[a].cnt -= 1;
      st[a].j += st[a].step;
      nk[a] = st[a].cnt > 0 ? plane_k(g, a, st[a].j, r[a]) : CUDART_INF;
    } else {
      k2 = kout;
    }
    if (k2 > k1) {
      double F2 = flux_at(fx, k2);
      double km = dmul(0.5, dadd(k1, k2));
      bool inside = true;
      int idx[3];
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        double t = dmul(dsub(dmul(km, v[a]), g.lo[a]), g.s[a]);
        inside = inside && (0.0 <= t && t < (double)g.n[a]);
        idx[a] = __double2int_rz(t);
      }
      if (inside) {
        int64_t b = (int64_t)idx[0] + (int64_t)g.n[0] * ((int64_t)idx[1] + (int64_t)g.n[1] * idx[2]);
        emit(b, dmul(dsub(F2, F1), omega_c));
        ++nseg;
      }
      k1 = k2;
      F1 = F2;
    }
    if (left == 0) break;
  }
  return nseg;
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
    if (!(0.0 <= t && t < (double)g.n[a])) return -1;
    idx[a] = __double2int_rz(t);
  }
  return (int64_t)idx[0] + (int64_t)g.n[0] * ((int64_t)idx[1] + (int64_t)g.n[1] * idx[2]);
}

}  // namespace mdn
