// mdn_kernels.cuh -- launch parameter blocks and launcher declarations (internal, not the ABI).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "mdn_device.cuh"

namespace mdn {

constexpr int kMaxOps = 48;           // MDN_MAX_OPS
constexpr int kMaxMats = 64;          // MDN_MAX_MATS
constexpr int kRunsPerLaunch = 16;    // runs composed per MDNorm launch (batched API)
constexpr int kFluxSmemMax = 4096;    // flux knots staged in shared memory (32 B records + 8 x 2 B cells per knot: 192 KB)
#ifndef MDN_PIECE_BALANCED
#define MDN_PIECE_BALANCED 1  // equal-length pieces (cuts at floor(p cA / P)); 0: every G-th crossing
#endif
#ifndef MDN_PIECE_SEGS
#define MDN_PIECE_SEGS 40  // 2-D slices; measured (balanced pieces): 40 > 32 > 48 on the CORELLI slab
#endif
#ifndef MDN_PIECE_SEGS_3D
#define MDN_PIECE_SEGS_3D 56  // 3-D grids; measured (balanced pieces): 56 > 48 > 40 > 32 on TOPAZ 200^3
#endif
constexpr int kPieceSegs = MDN_PIECE_SEGS;  // target segments per work piece (load balance, M4-M7)
constexpr int kPieceSegs3D = MDN_PIECE_SEGS_3D;

// Matrices for one launch, passed by value as a __grid_constant__ kernel parameter (sm_70+
// kernels accept up to 32 KB of parameters; CUDA >= 12.1).  Either compose (UB, W, ops, R) on
// the device (API mode, M0/B0) or take final matrices (parity mode).
struct MatBlock {
  int32_t compose;   // 1: compose from UB/W/ops/R; 0: use M
  int32_t nops;      // compose mode
  int32_t nruns;     // compose mode (MDNorm); 0 for BinMD
  int32_t nmat;      // = nruns * nops (MDNorm), nops (BinMD), or the parity count
  double UB[9];
  double W[9];
  double charge[kMaxMats > kRunsPerLaunch ? kMaxMats : kRunsPerLaunch];  // per run / per matrix
  union {
    struct {
      double ops[kMaxOps * 9];
      double R[kRunsPerLaunch * 9];
    } c;
    double M[kMaxMats * 9];
  } u;
};

// A trajectory that hits the grid (output of the cull kernel, input of the walk kernel): its
// direction v, clip [kin, kout], weight Omega_p c_r, and how it is cut into P pieces at
// crossings of axis A: with MDN_PIECE_BALANCED, stepG = step * cA (signed crossing count of A)
// and cut p (p = 1 .. P-1) is the crossing with index j_A + step * floor(p cA / P); otherwise
// the crossing with index j_A + p * stepG.
struct alignas(16) Hitter {
  double v0, v1, v2, kin;
  double kout, oc;
  int32_t A;               // busiest axis (bits 0-1) | flux table index << 2
  int32_t jA, stepG, P;
};

// Zero at the start of every cull: the walk's last CTA returns them to zero (so no memset sits
// between a preceding kernel and the cull, which is launched with programmatic dependent launch)
// and keeps the slab's hitter count in last_nhit (tracing).
struct DevCounters {
  unsigned int nhit;      // hitters written by the cull kernel
  unsigned int claimed;   // hitters claimed by the walk kernel's warps
  unsigned int pclaim;    // slab pixels claimed by the cull kernel's warps
  unsigned int done;      // walk CTAs finished
  unsigned int last_nhit; // hitters of the last slab walked
  unsigned int pad[3];
};

struct MdnParams {
  GridC g;
  const double4* pix;      // (q0, q1, q2, Omega) per pixel, q = z - d  (M1)
  const double2* pkr;      // per-pixel (k_lo, k_hi) limits, or nullptr (NEXT #1)
  int64_t pix_begin, pix_stride, nshard;
  FluxView flux;           // table 0 (device pointers, global)
  const FluxView* fviews;  // per-bank tables (several tables), or nullptr
  const int32_t* ptab;     // pixel -> flux table (with fviews), or nullptr
  int32_t acc_f32;         // privatised partial sums in fp32 (MDN_ACC_F32) instead of fp64
  int32_t priv;            // shared-memory privatised histogram: -1 auto, 0 never, 1 whenever it fits
  double kmin, kmax;
  double qmax;             // max(2, max_p max_i |q_p,i|): scales the cull's fp32 error band
  double* norm;            // fp64 histogram (nbins)
  unsigned long long* stats;  // nullptr, or [traj, hits, crossings, segments] (+= per launch)
  // cull -> walk hand-off (production path)
  Hitter* hit;             // capacity >= slab length
  DevCounters* ctr;
  uint32_t p0, plen;       // slab: shard pixels [p0, p0 + plen), all matrices of the launch
};

struct BinParams {
  GridC g;
  const float* events;
  int64_t nevents, stride;
  int32_t col_w, col_q;
  int32_t col_e;           // error-squared column, or -1
  int32_t ord[3];          // axis test order of the fp32 fast path (fewest bins first)
  int32_t st[3];           // linear-index stride of axis ord[k] (1, n0, n0 n1)
  int32_t w0, w1;          // bins [w0, w1) of test-order axis 0 are scattered (an L2-sized slab of a
                           // grid larger than L2, one launch per slab); [0, n) otherwise
  int32_t acc_f32;         // privatised partial sums in fp32 (MDN_ACC_F32) instead of fp64
  int32_t priv;            // shared-memory privatised histogram: -1 auto, 0 never, 1 whenever it fits
  double* binmd;           // fp64 histogram (nbins)
  double* err2;            // fp64 error-squared histogram (nbins), used when col_e >= 0
  unsigned long long* stats;  // nullptr, or [.., .., .., .., pairs, inside] (+= per launch)
  const void* tables;      // the launch's BinTables in global memory (launch_binmd_plan)
  // MDBox mode (NEXT #4, binmd_accumulate_boxes): only the boxes listed in box_list (box_count of
  // them, written by launch_binmd_box_cull) are read; box b = events [b box_events, (b+1) box_events)
  const int32_t* box_list;
  const unsigned* box_count;
  int32_t box_log2;        // log2(box_events / 32)
};

// launchers (return the launch's cudaError_t)
cudaError_t launch_pixels_prepare(const double* dir, const double* solid, double4* pix, int64_t npix,
                                  cudaStream_t s);
// MDNorm for shard pixels [p.p0, p.p0 + p.plen) x all matrices: cull (M1-M3) + piece walk (M3-M7).
cudaError_t launch_mdnorm(const MdnParams& p, const MatBlock& mb, int num_sms, cudaStream_t s);
// Hitters per walk launch above which warps claim 32 hitters at a time from the start (no static
// per-CTA blocks): the walk's large-launch regime (tests assert they cover it).
uint32_t walk_big_claim_threshold(bool d3, int num_sms);
cudaError_t launch_binmd(const BinParams& p, const MatBlock& mb, int num_sms, cudaStream_t s);
// B0 for one BinMD launch: compose N_s and build the decision tables into `tables` (device memory
// of binmd_tables_bytes()), one CTA; binmd_kernel reads them (BinParams::tables).
size_t binmd_tables_bytes();
cudaError_t launch_binmd_plan(const BinParams& p, const MatBlock& mb, void* tables, cudaStream_t s);
// NEXT #4: Q extents of boxes of box_events consecutive packed events (one pass), and the list of
// boxes that can reach the grid under some op of the launch's tables (conservative fp64 interval
// arithmetic); count must be zero before the cull.
cudaError_t launch_binmd_box_bounds(const float4* events, int64_t nevents, int32_t box_events, float* bounds,
                                    int num_sms, cudaStream_t s);
cudaError_t launch_binmd_box_cull(const BinParams& p, const float* bounds, int64_t nboxes, int32_t* list,
                                  unsigned* count, int num_sms, cudaStream_t s);
// Accumulation path chosen for the last launch_mdnorm / launch_binmd on this thread (tracing and
// tests): 0 = global fp64 red.add, 1 = shared-memory fp64 partials, 2 = shared-memory fp32 partials.
int last_mdnorm_path();
int last_binmd_path();
cudaError_t launch_cross_section(const double* norm, const double* binmd, double* xs, int64_t nbins,
                                 int num_sms, cudaStream_t s);
cudaError_t launch_cross_section_err(const double* norm, const double* binmd, const double* err2, double* xs,
                                     double* xs_err, int64_t nbins, int num_sms, cudaStream_t s);
cudaError_t launch_debug_traj(const MdnParams& p, const MatBlock& mb, int64_t ntraj,
                              const int64_t* ids, int64_t npix, int32_t* n_cross, int32_t* n_seg,
                              int64_t* seg_bins, double* seg_vals, int64_t max_segs, cudaStream_t s);
cudaError_t launch_debug_bins(const BinParams& p, const MatBlock& mb, int64_t* bins, cudaStream_t s);
cudaError_t launch_debug_compose(const MatBlock& mdn, const MatBlock& bin, double* M, double* N,
                                 int32_t* ok, cudaStream_t s);

}  // namespace mdn
