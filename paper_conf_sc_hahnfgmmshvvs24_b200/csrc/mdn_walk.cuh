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
// The walk is a state (WalkState): init() sets a piece up, step1/step2() consume one or two
// crossings of L, segment() closes the piece at hi_k.  The production kernel hands every lane of
// a warp one piece per round and the parity entry point runs single pieces; both call traj_walk.
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
  // 2-D: every midpoint of the piece lies in the slab's single axis-2 bin.  t_2(k) =
  // RN(RN(RN(k v2) - lo_2) s_2) is monotone in k (each rounding is), and every midpoint
  // RN(0.5 RN(k1 + k2)) of two list entries lies in [lo_k, hi_k], so floor(t_2) = 0 at both
  // ends of the piece decides it for every segment -- the definition's own test otherwise.
  bool t2ok;

  __device__ __forceinline__ static bool axis2_in(const GridC& g, double k, double v) {
    const double t2 = dmul(dsub(dmul(k, v), g.lo[2]), g.s[2]);
    return __double2int_rd(t2) == 0;
  }

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
      t2ok = false;
    } else {
      c2.cnt = 0;
      c2.nk = CUDART_INF;
      c2.jd = c2.stepd = c2.r = 0.0;
      t2ok = axis2_in(g, lo_k, v2) && axis2_in(g, hi_k, v2);
    }
    left = c0.cnt + c1.cnt + c2.cnt;
    k1 = lo_k;
    F1 = flux_at<TabT>(fx, lo_k);
  }

  // next crossing of L (left >= 1): the smallest pending one (ties: lowest axis first; equal
  // values give a skipped zero-length segment, so the order among ties never matters)
  __device__ __forceinline__ double next(const GridC& g) {
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
  // if a segment was emitted.  L is non-decreasing (k2 >= k1), and equal k gives an equal F,
  // so the last entry is taken unconditionally.
  template <class Emit>
  __device__ __forceinline__ int segment(const GridC& g, double k2, double F2, Emit& emit) {
    int emitted = 0;
    if (k2 > k1) {
      const double km = dmul(0.5, dadd(k1, k2));
      const double t0 = dmul(dsub(dmul(km, v0), g.lo[0]), g.s[0]);
      const double t1 = dmul(dsub(dmul(km, v1), g.lo[1]), g.s[1]);
      // for finite t, (0 <= t < n) <=> (unsigned)floor(t) < n (floor saturates, -0 -> 0); the
      // walk only sees finite v (the cull drops non-finite directions)
      const int i0 = __double2int_rd(t0), i1 = __double2int_rd(t1);
      bool in = (unsigned)i0 < (unsigned)g.n[0] && (unsigned)i1 < (unsigned)g.n[1];
      int b;
      if (k3D) {
        const double t2 = dmul(dsub(dmul(km, v2), g.lo[2]), g.s[2]);
        const int i2 = __double2int_rd(t2);
        in = in && (unsigned)i2 < (unsigned)g.n[2];
        b = i0 + g.n[0] * (i1 + g.n[1] * i2);
      } else {
        if (!t2ok) in = in && axis2_in(g, km, v2);
        b = i0 + g.n[0] * i1;
      }
      if (in) {
        emit(b, dmul(dsub(F2, F1), oc));
        emitted = 1;
      }
    }
    k1 = k2;
    F1 = F2;
    return emitted;
  }

  // consume the next crossing (left >= 1); returns the number of segments emitted
  template <typename TabT, class Emit>
  __device__ __forceinline__ int step1(const GridC& g, const FluxView& fx, Emit& emit) {
    const double ka = next(g);
    return segment(g, ka, flux_at<TabT>(fx, ka), emit);
  }

  // consume the next two crossings (left >= 2): their flux look-ups (the longest dependency
  // chain) are independent and overlap
  template <typename TabT, class Emit>
  __device__ __forceinline__ int step2(const GridC& g, const FluxView& fx, Emit& emit) {
    const double ka = next(g);
    const double kb = next(g);
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
    while (ws.left >= 2) nseg += ws.template step2<TabT>(g, fx, emit);
  while (ws.left >= 1) nseg += ws.template step1<TabT>(g, fx, emit);
  // the last entry of L: the end of the piece
  return nseg + ws.segment(g, hi_k, flux_at<TabT>(fx, hi_k), emit);
}

}  // namespace mdn
