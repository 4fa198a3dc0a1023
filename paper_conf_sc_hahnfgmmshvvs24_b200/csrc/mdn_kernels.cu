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
//   B0-B3             mdn_binmd.cu
//   X2                xs_kernel
// The parity entry points (debug_*) run the very same device functions (mdn_device.cuh).
#include <algorithm>
#include <type_traits>

#include "mdn_common.cuh"
#include "mdn_walk.cuh"

namespace mdn {

namespace {

using namespace common;

// One persistent walk CTA per SM (the shared-memory flux table takes up to 196 KB): 1024
// threads for 2-D slices (64 registers: measured 1024 > 896 > 768 on the CORELLI slab), 768 for
// 3-D grids (the unrolled walk needs more registers).
#ifndef MDN_WALK_THREADS_2D
#define MDN_WALK_THREADS_2D 1024
#endif
#ifndef MDN_WALK_THREADS_3D
#define MDN_WALK_THREADS_3D 768
#endif
constexpr int kWalkThreads2D = MDN_WALK_THREADS_2D;
constexpr int kWalkThreads3D = MDN_WALK_THREADS_3D;
// walk warps claim hitters kWalkChunk at a time (near the end of a launch) into a per-warp ring
constexpr int kWalkChunk = 8;
// the last kWalkSplitTail hitters per warp are cut into kWalkSplit x more pieces (measured: 4 > 8
// > 16 > 32, -1% CORELLI walk at 4; a split of 4 is slower)
constexpr int kWalkSplit = 2;
constexpr int kWalkSplitTail = 4;
// % of a launch's hitters in static per-CTA blocks, claimed kStaticChunk at a time
constexpr int kWalkStaticPct = 60;
constexpr int kStaticChunk = 32;
// claims shrink to kWalkChunk hitters once fewer than kWalkTail x 32 hitters per warp remain
constexpr int kWalkTail = 4;
// auto privatisation of the walk: trajectories per (bin x CTA) of the flush (3-D grids; x16 for 2-D)
constexpr int kPrivTrajPerBin = 1;
constexpr int kWalkRing = 64;  // >= 31 + the largest claim (32), a power of two
static_assert(kWalkChunk >= 1 && kWalkChunk <= 32, "walk claim size");
constexpr int walk_threads(bool k3D) { return k3D ? kWalkThreads3D : kWalkThreads2D; }

// Shared-memory privatised histogram (S§2.8 G2/G3): T = double (MDN_ACC_F64) or float
// (MDN_ACC_F32 partials); flushed into the fp64 global histogram at the end of the kernel.
template <typename T>
struct SmemEmit {
  T* h;
  __device__ __forceinline__ void operator()(int b, double val) const {
    hist_add<T>(h, nullptr, b, (T)val, T(0), false);
  }
};

// red.global.add.f64 stated explicitly (red_add): with a fence anywhere in the kernel (the
// counters' reset at its end) the compiler otherwise turns atomicAdd into an atomic with a
// discarded return (ATOMG), and every segment waits for its L2 round trip -- measured 2x slower.
struct AtomicEmit {
  double* h;
  __device__ __forceinline__ void operator()(int b, double val) const { red_add(h + b, val); }
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

// bytes of the cull's per-launch tables: M (9 doubles), charge (1 double), CullMat per matrix
__host__ __device__ constexpr size_t cull_mat_bytes(int nmat) {
  return (sizeof(double) * 10 + sizeof(CullMat)) * (size_t)nmat;
}
// per-warp cull ring: 64 pixel offsets + 64 matrix indices
constexpr size_t kCullRingBytes = sizeof(uint32_t) * 128;

// M0 and the fp32 test constants (whole CTA; ends with a barrier)
__device__ __forceinline__ void cull_prepare(const MdnParams& p, const MatBlock& mb, double* sM, double* sC,
                                             CullMat* sF) {
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
      // |q_i| <= qmax (2 for unit directions); fp32 v and x = k v are within 0.5e-6 qmax kmax
      // sum|M_a| of the exact values: the window is widened by >= 4x that
      const double delta = 2e-6 * p.qmax * p.kmax * sum + 1e-6 * (fabs(p.g.lo[a]) + fabs(p.g.hi[a])) + 1e-30;
      sF[m].a[k] = make_float4((float)row[0], (float)row[1], (float)row[2], (float)p.g.lo[a] - (float)delta);
      hi[k] = (float)p.g.hi[a] + (float)delta;
    }
    sF[m].hi = make_float4(hi[0], hi[1], hi[2], 0.f);
  }
  __syncthreads();
}

// One warp's cull: a ring of fp32 survivors (pixel offset, matrix); the exact fp64 path runs when
// 32 of them are queued, so it executes with the whole warp converged.
template <bool kStats>
struct CullWarp {
  uint32_t* qoff;
  uint32_t* qmat;
  int qhead, qcnt;
  unsigned long long c_traj, c_hit, c_cross;

  __device__ __forceinline__ void init(uint32_t* ring) {
    qoff = ring;
    qmat = ring + 64;
    qhead = qcnt = 0;
    c_traj = c_hit = c_cross = 0;
  }

  // exact M1-M3 for queued candidates [qhead, qhead + n) (n <= 32), hitters appended
  __device__ __forceinline__ void drain(const MdnParams& p, const double* sM, const double* sC, int n, int lane) {
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
        // The piece plan needs only approximate crossing ranges: the walk clamps every cut to
        // [kin, kout] and finds each piece's crossings exactly (a cut strictly inside (kin, kout)
        // is a plane crossing, i.e. a member of L, and a clamped one is kin or kout): measured
        // CORELLI MDNorm -1.8%, the 120-run scan -2.8% per step.  3-D grids take the exact range
        // of the cut axis (their pieces end on the box faces, where an estimate one plane off
        // leaves a short first or last piece: TOPAZ 48 ops +1.8% with every range estimated);
        // the work counters keep every range exact.
        const bool exact = kStats;
        const AxisStream s0 = exact ? axis_stream(p.g, 0, v0, rr[0], kin, kout) : axis_estimate(p.g, 0, v0, kin, kout);
        const AxisStream s1 = exact ? axis_stream(p.g, 1, v1, rr[1], kin, kout) : axis_estimate(p.g, 1, v1, kin, kout);
        const AxisStream s2 = exact ? axis_stream(p.g, 2, v2, rr[2], kin, kout) : axis_estimate(p.g, 2, v2, kin, kout);
        const int total = s0.cnt + s1.cnt + s2.cnt;
        // piece plan: cut at crossings of the busiest axis A, ~kPieceSegs segments per piece
        const bool a1 = s1.cnt > s0.cnt;
        const bool a2 = s2.cnt > (a1 ? s1.cnt : s0.cnt);
        const int A = a2 ? 2 : (a1 ? 1 : 0);
        // 3-D grids: the exact range of the cut axis (an estimate one plane off at the box faces
        // leaves short end pieces), the others estimated
        AxisStream sa = a2 ? s2 : (a1 ? s1 : s0);
        if (!exact && p.g.n[2] > 1)
          sa = axis_stream(p.g, A, A == 0 ? v0 : (A == 1 ? v1 : v2), A == 0 ? rr[0] : (A == 1 ? rr[1] : rr[2]), kin, kout);
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
        // cuts at crossings floor(p cA / P) of axis A (p = 1 .. P-1): the crossings of every axis
        // are equally spaced in k, so the P pieces get equal segment counts (no short remainder)
        h.jA = sa.j; h.stepG = sa.step * sa.cnt; h.P = P;
        if (kStats) {
          c_hit += 1;
          c_cross += total;
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
  }

  // the fp32 pre-test of slab pixels [base, base + 32) x every matrix of the launch; candidates
  // are queued and decided 32 at a time
  __device__ __forceinline__ void claim(const MdnParams& p, const MatBlock& mb, const CullMat* sF, const double* sM,
                                        const double* sC, uint32_t base, int lane) {
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
    if (!__any_sync(kFull, live)) return;
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
        if (qcnt >= 32) drain(p, sM, sC, 32, lane);
      }
    }
  }

  __device__ __forceinline__ void flush_stats(const MdnParams& p) {
    if (kStats) {
      flush_counter(p.stats + 0, c_traj);
      flush_counter(p.stats + 1, c_hit);
      flush_counter(p.stats + 2, c_cross);
    }
  }
};

template <bool kStats>
__global__ void __launch_bounds__(kThreads, 4)  // 64 registers: four resident CTAs per SM
mdnorm_cull_kernel(const __grid_constant__ MdnParams p, const __grid_constant__ MatBlock mb) {
  extern __shared__ double smem[];
  double* sM = smem;
  double* sC = sM + 9 * mb.nmat;
  CullMat* sF = reinterpret_cast<CullMat*>(sC + mb.nmat);
  // the walk (launched with programmatic stream serialisation) may start its
  // prologue on SMs this one-wave grid leaves; it waits for this grid before reading hitters
  asm volatile("griddepcontrol.launch_dependents;");
  cull_prepare(p, mb, sM, sC, sF);
  const int lane = threadIdx.x & 31;
  CullWarp<kStats> cw;
  cw.init(reinterpret_cast<uint32_t*>(sF + mb.nmat) + (threadIdx.x >> 5) * 128);
  // warps claim 32 pixels at a time from a global cursor (the hit fraction varies strongly over
  // the detector, so a static split leaves a tail of busy warps); loops are warp-uniform so the
  // ballots always have the full warp
  for (;;) {
    uint32_t base = 0;
    if (lane == 0) base = atomicAdd(&p.ctr->pclaim, 32u);
    base = __shfl_sync(kFull, base, 0);
    if (base >= p.plen) break;
    cw.claim(p, mb, sF, sM, sC, base, lane);
  }
  if (cw.qcnt > 0) cw.drain(p, sM, sC, cw.qcnt, lane);
  cw.flush_stats(p);
  // launched with programmatic dependent launch: the cull may run while the kernel before it
  // (e.g. the run's BinMD, which it does not depend on) finishes, but it completes only after that
  // kernel has, so everything after the walk sees both (no-op without the attribute)
  asm volatile("griddepcontrol.wait;" ::: "memory");
}

// ---------------------------------------------------------------- M3-M7: balanced piece walk
// A warp's queue of hitters (ring of kWalkRing indices; the head hitter may be partly consumed:
// `skip` of its pieces are done) holding `qpieces` pieces.  Each round hands the next 32 pieces
// of the queue to the 32 lanes, which walk them to completion together (so the piece set-up --
// divisions, per-axis ranges, first flux look-up -- runs converged).
struct WalkQ {
  unsigned* ring;  // hitter indices
  int* ringP;      // their piece counts
  int* pre;        // 32 ints of scan scratch
  unsigned head, nq;
  int skip, qpieces;

  __device__ __forceinline__ void init(unsigned* r, int* pr) {
    ring = r;
    ringP = reinterpret_cast<int*>(r + kWalkRing);
    pre = pr;
    head = nq = 0;
    skip = qpieces = 0;
  }

  // Enqueue hitters [b, b + nnew) (nnew <= 32, warp-uniform), longest pieces first (warp bitonic
  // sort on the piece length the cull stored: a round's 32 pieces then have similar lengths and
  // its lanes finish together).  split: cut them into up to kWalkSplit x more pieces at crossings
  // of the same axis (the last hitters of a launch, so that the final rounds end sooner).
  __device__ __forceinline__ void insert(const MdnParams& p, unsigned b, unsigned nnew, bool split, int lane) {
    int P = 0, A = 0;
    if ((unsigned)lane < nnew) {
      const int4 t = *reinterpret_cast<const int4*>(&p.hit[b + lane].A);  // (A, jA, stepG, P)
      A = t.x;
      P = t.w;
      if (split) P = max(P, min(abs(t.z), P * kWalkSplit));
    }
    // key = length << 5 | lane: unique, invalid lanes (0) last
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
    nq += nnew;
    qpieces += __reduce_add_sync(kFull, P);
    __syncwarp();
  }

  // one round: the next min(qpieces, 32) pieces, one per lane, walked to completion
  template <int kFlux, bool kStats, bool k3D, class Emit>
  __device__ __forceinline__ void round(const MdnParams& p, const FluxView& fx, Emit& emit, int lane,
                                        unsigned long long& c_seg) {
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
        const int cA = abs(h.stepG), st = h.stepG < 0 ? -1 : 1;
        if (mypi > 0) lo_k = fmax(h.kin, plane_k(p.g, A, h.jA + st * ((mypi * cA) / myP), rA));
        if (mypi < myP - 1) hi_k = fmin(h.kout, plane_k(p.g, A, h.jA + st * (((mypi + 1) * cA) / myP), rA));
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
};

// kFlux 1: the flux records and the uint16 cell table into shared memory, and the view the walk
// uses (other modes: the global view).  Every 16-byte load of the copy is issued before the first
// store, so the prologue costs about one L2 round trip (the cell table arrives pre-converted to
// uint16; a per-element loop over the int32 table took a round trip per element: 3.7% of the
// walk's stall samples on CORELLI).
constexpr int kStageBatch = 8;  // 16-byte loads per thread in flight
template <int kFlux>
__device__ __forceinline__ FluxView stage_flux(const MdnParams& p, double2* sKa, uint16_t* sTab) {
  FluxView fx = p.flux;
  if (kFlux == 1) {
    double2* sKb = sKa + p.flux.n;
    const int n = p.flux.n, nt = (p.flux.ntab + 7) >> 3;  // records, 16-byte groups of 8 cells
    if (p.flux.tab16) {
      // items [ka | kb | cells] of 16 bytes; a batch = kStageBatch items per thread, all loads
      // issued before the stores (4096 knots at 1024 threads: two batches)
      const int total = 2 * n + nt;
      for (int base = 0; base < total; base += kStageBatch * (int)blockDim.x) {
        uint4 v[kStageBatch];
#pragma unroll
        for (int j = 0; j < kStageBatch; ++j) {
          const int i = base + threadIdx.x + j * blockDim.x;
          if (i < n) v[j] = __ldg(reinterpret_cast<const uint4*>(p.flux.ka) + i);
          else if (i < 2 * n) v[j] = __ldg(reinterpret_cast<const uint4*>(p.flux.kb) + (i - n));
          else if (i < total) v[j] = __ldg(reinterpret_cast<const uint4*>(p.flux.tab16) + (i - 2 * n));
        }
#pragma unroll
        for (int j = 0; j < kStageBatch; ++j) {
          const int i = base + threadIdx.x + j * blockDim.x;
          if (i < 2 * n) reinterpret_cast<uint4*>(sKa)[i] = v[j];  // sKb = sKa + n
          else if (i < total) reinterpret_cast<uint4*>(sTab)[i - 2 * n] = v[j];
        }
      }
    } else {
      for (int i = threadIdx.x; i < n; i += blockDim.x) {
        sKa[i] = p.flux.ka[i];
        sKb[i] = p.flux.kb[i];
      }
      const int* gtab = static_cast<const int*>(p.flux.tab);
      for (int i = threadIdx.x; i < p.flux.ntab; i += blockDim.x) {
        const unsigned e = (unsigned)gtab[i];
        sTab[i] = (uint16_t)((e & (kFluxDense32 - 1)) | ((e & kFluxDense32) ? kFluxDense16 : 0u));
      }
    }
    fx.tab = sTab;
    // the rare general path bisects the global knots (fx.kn)
    fx.ka = sKa;
    fx.kb = sKb;
    fx.ska = (unsigned)__cvta_generic_to_shared(sKa);
    fx.skb = (unsigned)__cvta_generic_to_shared(sKb);
  }
  return fx;
}
__host__ __device__ constexpr size_t flux_smem_bytes(int kFlux, int n, int ntab) {
  return kFlux == 1 ? 2 * sizeof(double2) * (size_t)n + 16 * (size_t)((ntab + 7) >> 3) : 0;
}
// per warp: scan scratch (32 int) and the hitter ring (kWalkRing indices + piece counts)
constexpr size_t kWalkWarpBytes = sizeof(int) * 32 + 2 * sizeof(unsigned) * kWalkRing;

// the last CTA out returns the counters to zero for the next slab's cull
__device__ __forceinline__ void release_counters(const MdnParams& p) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&p.ctr->done, 1u) == gridDim.x - 1) {
      p.ctr->last_nhit = *(volatile unsigned*)&p.ctr->nhit;
      p.ctr->nhit = 0;
      p.ctr->claimed = 0;
      p.ctr->pclaim = 0;
      p.ctr->done = 0;
      __threadfence();
    }
  }
}

// kFlux: 0 = one flux table read from global memory, 1 = one table staged in shared memory,
// 2 = per-bank tables (pixel -> table map, NEXT #1) read from global memory, 3 = records in
// shared memory, cell table in global memory
template <int kFlux, bool kStats, bool k3D, int kPriv>
__global__ void __launch_bounds__(walk_threads(k3D), 1)
mdnorm_walk_kernel(const __grid_constant__ MdnParams p) {
  using PT = priv_t<kPriv>;
  extern __shared__ double4 wsm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  // shared layout: private histogram (kPriv, 16-byte rounded) | interval records ka, kb (n
  // double2 each) | cell table (uint16, even) | per-warp prefix sums (32 int) | per-warp hitter
  // rings (kWalkRing unsigned)
  PT* sHist = reinterpret_cast<PT*>(wsm);
  if (kPriv) priv_zero(sHist, p.g.nbins);
  double2* sKa = reinterpret_cast<double2*>(reinterpret_cast<char*>(wsm) + priv_bytes(kPriv, p.g.nbins));
  uint16_t* sTab = reinterpret_cast<uint16_t*>(sKa + 2 * (kFlux == 1 ? p.flux.n : 0));
  char* sW = reinterpret_cast<char*>(sKa) + flux_smem_bytes(kFlux, p.flux.n, p.flux.ntab);
  const FluxView fx = stage_flux<kFlux>(p, sKa, sTab);
  __shared__ unsigned sCur;  // claims taken from this CTA's static block of hitters
  if (threadIdx.x == 0) sCur = 0;
  __syncthreads();
  WalkQ q;
  q.init(reinterpret_cast<unsigned*>(sW + sizeof(int) * 32 * nwarps) + 2 * kWalkRing * warp,
         reinterpret_cast<int*>(sW) + 32 * warp);
  typename std::conditional<kPriv != 0, SmemEmit<PT>, AtomicEmit>::type emit;
  if constexpr (kPriv != 0) emit.h = sHist;
  else emit.h = p.norm;
  // everything above (flux staging, private histogram zeroing) overlaps the cull's tail under
  // programmatic dependent launch; the hitter list and count are read only after the cull
  // grid has completed.  No-op without the attribute.
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const unsigned nhit = *(volatile unsigned*)&p.ctr->nhit;
  unsigned long long c_seg = 0;
  // The queue is topped up by claiming hitters from the global cursor, so rounds are full across
  // hitter boundaries and the end-of-kernel imbalance is one small chunk.
  bool more = true;
  const unsigned tail = (unsigned)kWalkTail * 32u * gridDim.x * (unsigned)nwarps;
  unsigned chunk = nhit > tail ? 32u : (unsigned)kWalkChunk;
  // static per-CTA blocks of hitters cover kWalkStaticPct % of them; [rest, nhit) is dynamic
  // (only for launches small enough to claim in small chunks from the start: with 32-hitter
  // claims the global counter is not contended, and static blocks unbalance 3-D walks)
  const unsigned blk_n =
      nhit > tail ? 0u : (unsigned)(((unsigned long long)nhit * kWalkStaticPct / 100) / gridDim.x);
  const unsigned blk = blockIdx.x * blk_n, rest = blk_n * gridDim.x;
  bool sdone = false;  // lane 0: this CTA's block is used up
  const unsigned split_tail = (unsigned)kWalkSplitTail * gridDim.x * (unsigned)nwarps;
  for (;;) {
    while (q.qpieces < 32 && more) {
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
        // no early launch_dependents here: a cull launched after this walk (the next slab or run
        // block) reuses the hitter buffer and counters, so it may start only when the walk is
        // done (the implicit trigger at grid completion)
        break;
      }
      const unsigned nnew = min(n, nhit - b);
      // large claims (hitter locality, fewer atomics) until the last few claims per warp, then
      // small ones so that the warps finish together
      if (b >= rest) chunk = nhit - b > tail ? 32u : (unsigned)kWalkChunk;
      q.insert(p, b, nnew, nhit - b <= split_tail, lane);
    }
    if (q.qpieces == 0) break;
    q.round<kFlux, kStats, k3D>(p, fx, emit, lane, c_seg);
  }
  if (kPriv) {
    __syncthreads();
    priv_flush(sHist, p.norm, p.g.nbins);
  }
  if (kStats) flush_counter(p.stats + 3, c_seg);
  release_counters(p);
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

// dynamic shared memory of the walk kernel (layout in mdnorm_walk_kernel)
size_t walk_smem(const MdnParams& p, int kflux, int threads) {
  return flux_smem_bytes(kflux, p.flux.n, p.flux.ntab) + kWalkWarpBytes * (threads / 32);
}
template <int kFlux, bool kStats, bool k3D, int kPriv>
cudaError_t launch_walk(const MdnParams& p, int num_sms, cudaStream_t s) {
  constexpr int threads = walk_threads(k3D);
  const size_t smem = walk_smem(p, kFlux, threads) + priv_bytes(kPriv, p.g.nbins);
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
  // vs 0.372, step 0.481 vs 0.490.
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
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

template <bool kStats>
cudaError_t launch_cull(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  const size_t smem = cull_mat_bytes(mb.nmat) + kCullRingBytes * (kThreads / 32);
  auto k = mdnorm_cull_kernel<kStats>;
  cudaError_t err = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  // one wave of resident CTAs (grid-stride): no tail wave of unevenly loaded blocks
  int per_sm = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kThreads, smem);
  if (err != cudaSuccess) return err;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid_for(p.plen, num_sms, std::max(per_sm, 1)));
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  // programmatic dependent launch: cull CTAs take the SMs that the previous kernel's CTAs leave
  // (a BinMD launched before MDNorm ends unevenly: its in-grid events are clustered)
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, p, mb);
}

}  // namespace

cudaError_t launch_pixels_prepare(const double* dir, const double* solid, double4* pix, int64_t npix,
                                  cudaStream_t s) {
  pixels_prepare_kernel<<<grid_for(npix, 148, 8), kThreads, 0, s>>>(dir, solid, pix, npix);
  return cudaGetLastError();
}

uint32_t walk_big_claim_threshold(bool d3, int num_sms) {
  return (uint32_t)kWalkTail * 32u * (uint32_t)num_sms * (uint32_t)(walk_threads(d3) / 32);
}

cudaError_t launch_mdnorm(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s) {
  if (p.plen == 0 || mb.nmat <= 0) return cudaSuccess;
  cudaError_t err = cudaSuccess;
  // 2-D slices (a single bin on the last axis, "lBins=1") merge two crossing streams
  const bool d3 = p.g.n[2] > 1;
  const int smem_max = smem_optin(&err);
  if (err != cudaSuccess) return err;
  const int threads = walk_threads(d3);
  // the flux table goes to shared memory when it fits one CTA (uint16 cell entries)
  const bool flux_fits = p.flux.n <= kFluxSmemMax && walk_smem(p, 1, threads) <= (size_t)smem_max;
  // Private shared-memory histogram (S§2.8 G2) when the grid fits next to the walk's other shared
  // data: with the flux table in shared memory if both fit, else with the flux read through L1.
  // priv = 1 takes it whenever it fits; auto (-1) when the launch's trajectories outnumber the
  // bins the flush touches (one CTA per SM flushes every bin) by kPrivTrajPerBin (3-D
  // grids: every trajectory crosses the box) or 16x that (2-D slices: a few % hit the slab).
  // Measured (tools/priv_sweep.sh): TOPAZ 8 ops on 16^3 - 25^3 grids 2.1-3.2x faster; CORELLI
  // 24 ops on 16^2 / 60^2 slabs 2.7x / 1.2x faster, on 100^2 equal, on 150^2 1.35x slower.
  const int kind = p.acc_f32 ? 2 : 1;
  const size_t hb = priv_bytes(kind, p.g.nbins);
  const bool priv_ok = p.priv != 0 && !p.fviews;
  const uint64_t per_bin = (uint64_t)kPrivTrajPerBin * (d3 ? 1u : 16u);
  const bool worth = p.priv == 1 ||
                     (uint64_t)p.plen * (uint64_t)mb.nmat >= (uint64_t)p.g.nbins * (uint64_t)num_sms * per_bin;
  const bool with_sflux = priv_ok && worth && flux_fits && walk_smem(p, 1, threads) + hb <= (size_t)smem_max;
  const bool with_gflux = priv_ok && worth && !with_sflux && walk_smem(p, 0, threads) + hb <= (size_t)smem_max;
  if (with_sflux || with_gflux) {
    g_last_mdnorm_path = kind;
    err = p.stats ? launch_cull<true>(p, mb, num_sms, s) : launch_cull<false>(p, mb, num_sms, s);
    if (err != cudaSuccess) return err;
    if (with_sflux) return kind == 2 ? launch_walk_d<1, 2>(p, d3, num_sms, s) : launch_walk_d<1, 1>(p, d3, num_sms, s);
    return kind == 2 ? launch_walk_d<0, 2>(p, d3, num_sms, s) : launch_walk_d<0, 1>(p, d3, num_sms, s);
  }
  g_last_mdnorm_path = 0;
  err = p.stats ? launch_cull<true>(p, mb, num_sms, s) : launch_cull<false>(p, mb, num_sms, s);
  if (err != cudaSuccess) return err;
  if (p.fviews) return launch_walk_d<2, 0>(p, d3, num_sms, s);
  if (flux_fits) return launch_walk_d<1, 0>(p, d3, num_sms, s);
  return launch_walk_d<0, 0>(p, d3, num_sms, s);
}

int last_mdnorm_path() { return g_last_mdnorm_path; }

cudaError_t launch_cross_section(const double* norm, const double* binmd, double* xs, int64_t nbins,
                                 int num_sms, cudaStream_t s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid_for(nbins, num_sms, 8));
  cfg.blockDim = dim3(kThreads);
  cfg.stream = s;
  // programmatic dependent launch after the preceding kernel (the walk in the bench step order,
  // or BinMD): xs_kernel executes griddepcontrol.wait before reading the histograms
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
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


cudaError_t launch_debug_compose(const MatBlock& mdn, const MatBlock& bin, double* M, double* N,
                                 int32_t* ok, cudaStream_t s) {
  debug_compose_kernel<<<1, kThreads, 0, s>>>(mdn, bin, M, N, ok);
  return cudaGetLastError();
}

}  // namespace mdn
