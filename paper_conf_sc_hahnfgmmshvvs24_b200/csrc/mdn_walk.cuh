// mdn_walk.cuh -- M4-M7: the streaming walk of one piece of a clipped trajectory (sm_100a).
//
// A piece is the part [lo_k, hi_k] of a trajectory's list L, where lo_k and hi_k are members of
// L (its clip endpoints or plane crossings).  The walk is a 3-way streaming merge of the per-axis
// monotone crossing sequences strictly inside (lo_k, hi_k) (replaces the paper's sort, and
// the GPU comb sort, with no buffer), the flux at each list entry (M5), the midpoint bin of
// every positive-length segment (M6) and emit(b, (F(k2) - F(k1)) * omega_c) (M7).  Splitting L at
// any of its members leaves the set of segments unchanged, which is what lets the production
// kernel cut long trajectories into balanced pieces and hand them to lanes in any order.
//
// The walk is a resumable state (WalkState): init() sets a piece up, step() consumes one entry of
// L.  The production kernel keeps one state per lane and refills idle lanes with new pieces while
// the others continue (mdnorm_walk_kernel); the parity entry point runs one piece to completion
// (traj_walk).  Both execute the same device code.
#pragma once
#include "mdn_device.cuh"

namespace mdn {

template <bool k3D>
struct WalkState {
  // k3D = false: the last axis has a single bin (2-D slice), so it never has a crossing
  AxisCursor c0, c1, c2;
  double v0, v1, v2, oc;  // direction and Omega * c
  double k1, F1, hi_k;    // last list entry and its flux; end of the piece
  int left;               // crossings not yet merged
  int rem;                // list entries not yet consumed (0: idle)

  template <typename TabT>
  __device__ __forceinline__ void init(const GridC& g, const FluxView& fx, double v0_, double v1_, double v2_,
                                       double lo_k, double hi_k_, double oc_) {
    v0 = v0_;
    v1 = v1_;
    v2 = v2_;
    oc = oc_;
    hi_k = hi_k_;
    cursor_init(c0, g, 0, v0, lo_k, hi_k);
    cursor_init(c1, g, 1, v1, lo_k, hi_k);
    if (k3D) {
      cursor_init(c2, g, 2, v2, lo_k, hi_k);
    } else {
      c2.cnt = 0;
      c2.nk = CUDART_INF;
      c2.jd = c2.stepd = c2.r = 0.0;
    }
    left = c0.cnt + c1.cnt + c2.cnt;
    rem = left + 1;
    k1 = lo_k;
    F1 = flux_at<TabT>(fx, lo_k);
  }

  // next entry of L: the smallest pending crossing (ties: lowest axis first; equal values give
  // a skipped zero-length segment, so the order among ties never matters), then hi_k
  __device__ __forceinline__ double next(const GridC& g) {
    if (left == 0) return hi_k;
    --left;
    if (!k3D) {  // 2-D slice: two streams
      if (c0.nk <= c1.nk) {
        const double k = c0.nk;
        c0.jd += c0.stepd;
        --c0.cnt;
        c0.nk = c0.cnt > 0 ? dmul(dadd(g.lo[0], dmul(c0.jd, g.w[0])), c0.r) : CUDART_INF;
        return k;
      }
      const double k = c1.nk;
      c1.jd += c1.stepd;
      --c1.cnt;
      c1.nk = c1.cnt > 0 ? dmul(dadd(g.lo[1], dmul(c1.jd, g.w[1])), c1.r) : CUDART_INF;
      return k;
    }
    // three streams, selects only: advance the chosen axis with one plane evaluation
    const bool s01 = c1.nk < c0.nk;
    const double m01 = s01 ? c1.nk : c0.nk;
    const bool s2 = c2.nk < m01;
    const bool p0 = !s2 && !s01, p1 = !s2 && s01;
    const double k = s2 ? c2.nk : m01;
    const double jd = (p0 ? c0.jd + c0.stepd : (p1 ? c1.jd + c1.stepd : c2.jd + c2.stepd));
    const int cnt = (p0 ? c0.cnt : (p1 ? c1.cnt : c2.cnt)) - 1;
    const double lo = p0 ? g.lo[0] : (p1 ? g.lo[1] : g.lo[2]);
    const double w = p0 ? g.w[0] : (p1 ? g.w[1] : g.w[2]);
    const double r = p0 ? c0.r : (p1 ? c1.r : c2.r);
    const double nk = cnt > 0 ? dmul(dadd(lo, dmul(jd, w)), r) : CUDART_INF;
    if (p0) { c0.jd = jd; c0.cnt = cnt; c0.nk = nk; }
    if (p1) { c1.jd = jd; c1.cnt = cnt; c1.nk = nk; }
    if (s2) { c2.jd = jd; c2.cnt = cnt; c2.nk = nk; }
    return k;
  }

  // segment (k1, k2) if it has positive length: midpoint bin (M6) and value (M7).  Returns 1
  // if a segment was emitted.
  template <class Emit>
  __device__ __forceinline__ int segment(const GridC& g, double k2, double F2, Emit& emit) {
    int emitted = 0;
    if (k2 > k1) {
      const double km = dmul(0.5, dadd(k1, k2));
      const double t0 = dmul(dsub(dmul(km, v0), g.lo[0]), g.s[0]);
      const double t1 = dmul(dsub(dmul(km, v1), g.lo[1]), g.s[1]);
      const double t2 = dmul(dsub(dmul(km, v2), g.lo[2]), g.s[2]);
      // for finite t, (0 <= t < n) <=> (unsigned)floor(t) < n (floor saturates, -0 -> 0); the
      // walk only sees finite v (the cull drops non-finite directions)
      const int i0 = __double2int_rd(t0), i1 = __double2int_rd(t1), i2 = __double2int_rd(t2);
      if ((unsigned)i0 < (unsigned)g.n[0] && (unsigned)i1 < (unsigned)g.n[1] && (unsigned)i2 < (unsigned)g.n[2]) {
        emit(i0 + g.n[0] * (i1 + g.n[1] * i2), dmul(dsub(F2, F1), oc));
        emitted = 1;
      }
      k1 = k2;
      F1 = F2;
    }
    return emitted;
  }

  // consume one entry of L (rem >= 1); returns the number of segments emitted
  template <typename TabT, class Emit>
  __device__ __forceinline__ int step1(const GridC& g, const FluxView& fx, Emit& emit) {
    const double ka = next(g);
    --rem;
    return segment(g, ka, flux_at<TabT>(fx, ka), emit);
  }

  // consume two entries of L (rem >= 2): their flux look-ups (the longest dependency chain) are
  // independent and overlap
  template <typename TabT, class Emit>
  __device__ __forceinline__ int step2(const GridC& g, const FluxView& fx, Emit& emit) {
    const double ka = next(g);
    const double kb = next(g);
    rem -= 2;
    const double Fa = flux_at<TabT>(fx, ka);
    const double Fb = flux_at<TabT>(fx, kb);
    const int n = segment(g, ka, Fa, emit);
    return n + segment(g, kb, Fb, emit);
  }
};

// Walk one piece to completion.  Returns n_seg; *ncross receives the number of crossings
// strictly inside (lo_k, hi_k).
template <bool k3D, typename TabT = int, class Emit>
__device__ __forceinline__ int traj_walk(const GridC& g, const FluxView& fx, double v0, double v1,
                                         double v2, double lo_k, double hi_k, double omega_c,
                                         Emit& emit, int* ncross) {
  WalkState<k3D> ws;
  ws.template init<TabT>(g, fx, v0, v1, v2, lo_k, hi_k, omega_c);
  *ncross = ws.left;
  int nseg = 0;
  // (2-D slices too: measured no faster with the interval guess, r02)
  if (k3D)
    while (ws.rem >= 2) nseg += ws.template step2<TabT>(g, fx, emit);
  while (ws.rem >= 1) nseg += ws.template step1<TabT>(g, fx, emit);
  return nseg;
}

}  // namespace mdn
