// mdn_api.cu -- the extern "C" boundary declared in include/mdnorm.h.
//
// Host side only: argument validation (before any side effect), device-memory ownership,
// stream ordering and launch marshalling.  Every step of the hot path itself (matrix
// composition, trajectories, scatter, divide) runs in the kernels of mdn_kernels.cu.
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "mdn_kernels.cuh"
#include "mdnorm.h"

using mdn::GridC;
using mdn::MatBlock;

struct mdn_grid {
  int device = 0;
  int num_sms = 148;
  GridC g{};
  double W[9]{};
  mdn_acc acc = MDN_ACC_F64;
  int32_t priv = -1;          // shared-memory privatisation: -1 auto, 0 never, 1 whenever it fits
  int32_t path[2] = {0, 0};   // accumulation path of the last MDNorm / BinMD launch
  double* d_hist = nullptr;  // [norm | binmd | err2], 3 * nbins doubles
  double2* d_pkr = nullptr;  // per-pixel (k_lo, k_hi) limits, or nullptr
  double4* d_pix = nullptr;
  int64_t npix = 0;
  double* d_flux = nullptr;   // every flux table: knots (+2 pads each), then interval records
  int* d_ftab = nullptr;      // cell tables of every flux table
  uint16_t* d_ftab16 = nullptr;  // table 0's cell table as uint16 entries (the walk's shared-memory copy)
  mdn::FluxView* d_fviews = nullptr;  // one view per flux table (device)
  int32_t* d_ptab = nullptr;  // pixel -> flux table (several tables only)
  int32_t nftables = 0;
  mdn::FluxView flux0{};      // view of table 0 (device pointers)
  std::vector<double> fguess_hit;  // per flux table: fraction of the k range the interval guess names
  mdn::Hitter* d_hit = nullptr;       // cull -> walk hand-off buffer
  uint32_t hit_cap = 0;
  uint32_t hit_cap_max = 0;  // kMaxSlab, lowered if the device cannot hold that buffer
  uint32_t slab_limit = 0;   // trajectories per cull/walk slab (kMaxSlab; lowered by a test entry)
  uint32_t last_nslab = 0;   // slabs of the last MDNorm launch block (tracing)
  double qmax = 2.0;         // max(2, largest |q_p,i| of the instrument)
  mdn::DevCounters* d_ctr = nullptr;
  double* d_xs = nullptr;    // scratch for host xs
  unsigned long long* d_stats = nullptr;  // 6 work counters (mdnorm_stats)
  bool stats_on = false;
  // host-event streaming (binmd_accumulate with a host pointer)
  float* d_stage[2] = {nullptr, nullptr};
  size_t stage_floats = 0;
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_ready[2] = {nullptr, nullptr};
  cudaEvent_t ev_free[2] = {nullptr, nullptr};
  cudaEvent_t ev_epoch = nullptr;  // recorded by mdnorm_reset: host-event copies start after it
  // BinMD decision tables (B0, launch_binmd_plan): two buffers used in turn; the plan of a call
  // runs on plan_stream (it depends on no device data, so it overlaps the MDNorm kernels before
  // it) and the BinMD kernels wait for it
  void* d_btab[2] = {nullptr, nullptr};
  int32_t* d_blist[2] = {nullptr, nullptr};  // surviving boxes (binmd_accumulate_boxes), count first
  int64_t blist_cap[2] = {0, 0};
  int btab_i = 0;
  cudaStream_t plan_stream = nullptr;
  cudaEvent_t ev_tab_ready[2] = {nullptr, nullptr};
  cudaEvent_t ev_tab_free[2] = {nullptr, nullptr};
};

namespace {

thread_local std::string g_err;

mdn_status fail(mdn_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

mdn_status cuda_fail(cudaError_t e, const char* where) {
  cudaGetLastError();  // clear sticky-free errors
  return fail(e == cudaErrorMemoryAllocation ? MDN_ENOMEM : MDN_ECUDA, "%s: %s", where,
              cudaGetErrorString(e));
}

#define MDN_CUDA(call, where)                   \
  do {                                          \
    cudaError_t e_ = (call);                    \
    if (e_ != cudaSuccess) return cuda_fail(e_, where); \
  } while (0)

mdn_status ok() {
  g_err.clear();
  return MDN_OK;
}

// Restores the caller's current device on scope exit.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

bool finite_all(const double* x, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (!std::isfinite(x[i])) return false;
  return true;
}

double det3(const double* m) {
  return m[0] * (m[4] * m[8] - m[5] * m[7]) - m[1] * (m[3] * m[8] - m[5] * m[6]) +
         m[2] * (m[3] * m[7] - m[4] * m[6]);
}

bool nonsingular(const double* m) {
  double d = det3(m);
  return std::isfinite(d) && d != 0.0;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// copy n elements from a host or device pointer into a host vector
template <class T>
cudaError_t to_host(const T* src, int64_t n, std::vector<T>& dst) {
  dst.resize((size_t)n);
  if (n == 0) return cudaSuccess;
  if (is_device_ptr(src)) return cudaMemcpy(dst.data(), src, sizeof(T) * n, cudaMemcpyDeviceToHost);
  std::memcpy(dst.data(), src, sizeof(T) * n);
  return cudaSuccess;
}

mdn_status check_ops(int32_t nops, const double* ops) {
  if (nops < 1 || nops > MDN_MAX_OPS) return fail(MDN_EINVAL, "nops = %d outside [1, %d]", nops, MDN_MAX_OPS);
  if (!ops) return fail(MDN_EINVAL, "ops is NULL");
  if (!finite_all(ops, 9 * (int64_t)nops)) return fail(MDN_EINVAL, "ops contain non-finite values");
  for (int s = 0; s < nops; ++s)
    if (!nonsingular(ops + 9 * s)) return fail(MDN_EINVAL, "symmetry op %d is singular", s);
  return MDN_OK;
}

mdn_status check_matrix(const double* m, const char* name) {
  if (!m) return fail(MDN_EINVAL, "%s is NULL", name);
  if (!finite_all(m, 9)) return fail(MDN_EINVAL, "%s has non-finite values", name);
  if (!nonsingular(m)) return fail(MDN_EINVAL, "%s is singular", name);
  return MDN_OK;
}

mdn_status check_krange(double k_min, double k_max) {
  if (!(std::isfinite(k_min) && std::isfinite(k_max) && k_min > 0.0 && k_min < k_max))
    return fail(MDN_EINVAL, "need 0 < k_min < k_max (got %g, %g)", k_min, k_max);
  return MDN_OK;
}

mdn_status check_ready(mdn_grid* g) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (!g->d_pix) return fail(MDN_ESTATE, "mdnorm_set_instrument has not been called");
  if (!g->d_flux) return fail(MDN_ESTATE, "mdnorm_set_flux has not been called");
  return MDN_OK;
}

mdn_status shard(mdn_grid* g, int64_t pix_begin, int64_t pix_end, int64_t pix_stride, int64_t* nshard) {
  if (pix_end < 0) pix_end = g->npix;
  if (pix_begin < 0 || pix_end > g->npix || pix_stride < 1)
    return fail(MDN_EINVAL, "bad pixel shard [%lld, %lld) stride %lld for npix %lld", (long long)pix_begin,
                (long long)pix_end, (long long)pix_stride, (long long)g->npix);
  *nshard = pix_begin < pix_end ? (pix_end - pix_begin + pix_stride - 1) / pix_stride : 0;
  return MDN_OK;
}

mdn::MdnParams mdn_params(mdn_grid* g, double k_min, double k_max, int64_t pix_begin, int64_t pix_stride,
                          int64_t nshard) {
  mdn::MdnParams p{};
  p.g = g->g;
  p.pix = g->d_pix;
  p.pkr = g->d_pkr;
  p.pix_begin = pix_begin;
  p.pix_stride = pix_stride;
  p.nshard = nshard;
  p.flux = g->flux0;
  p.fviews = g->nftables > 1 ? g->d_fviews : nullptr;
  p.ptab = g->nftables > 1 ? g->d_ptab : nullptr;
  p.acc_f32 = g->acc == MDN_ACC_F32;
  p.priv = g->priv;
  p.kmin = k_min;
  p.kmax = k_max;
  p.qmax = g->qmax;
  p.norm = g->d_hist;
  p.stats = g->stats_on ? g->d_stats : nullptr;
  p.hit = g->d_hit;
  p.ctr = g->d_ctr;
  return p;
}

#ifndef MDN_MAX_SLAB_LOG2
#define MDN_MAX_SLAB_LOG2 27
#endif
// Trajectories per cull/walk pair.  The hitter buffer holds a slab's worst case (every trajectory
// hits, 64 B each: up to 8 GiB of the 180 GB).  Large slabs pay: the walk of one CORELLI run
// (342K hitters) runs at 1.07e11 segments/s, a batch of 16 runs in one slab at ~1.4e11
// (measured: the 120-run scan 64 ms with 2^24-trajectory slabs, 38 ms with 2^27).
constexpr uint32_t kMaxSlab = 1u << MDN_MAX_SLAB_LOG2;

// MDNorm over all nmat x nshard trajectories of one launch block: slabs of at most kMaxSlab
// trajectories, each a cull kernel (compacting hitters into g->d_hit) and a walk kernel.  The
// hitter buffer holds one slab's worst case (every trajectory hits), so no count ever has to
// come back to the host (the MiniVATES host round trip of P:139 is avoided).
mdn_status run_mdnorm(mdn_grid* g, mdn::MdnParams p, const MatBlock& mb, cudaStream_t s) {
  const uint64_t ntraj = (uint64_t)mb.nmat * (uint64_t)p.nshard;
  if (ntraj == 0) return MDN_OK;
  const uint32_t want = (uint32_t)std::min<uint64_t>(ntraj, std::min(g->hit_cap_max, g->slab_limit));
  if (g->hit_cap < want) {
    if (g->d_hit) {
      cudaStreamSynchronize(s);
      cudaFree(g->d_hit);
    }
    g->d_hit = nullptr;
    g->hit_cap = 0;
    // largest buffer the device grants, halving down to 2^20 trajectories (smaller slabs)
    uint32_t cap = want;
    cudaError_t e = cudaMalloc(&g->d_hit, sizeof(mdn::Hitter) * (size_t)cap);
    while (e == cudaErrorMemoryAllocation && cap > (1u << 20)) {
      cudaGetLastError();
      cap /= 2;
      e = cudaMalloc(&g->d_hit, sizeof(mdn::Hitter) * (size_t)cap);
    }
    MDN_CUDA(e, "hitter buffer");
    g->hit_cap = cap;
    if (cap < want) g->hit_cap_max = cap;  // do not retry the larger size on every call
  }
  if (!g->d_ctr) {
    MDN_CUDA(cudaMalloc(&g->d_ctr, sizeof(mdn::DevCounters)), "counters");
    MDN_CUDA(cudaMemset(g->d_ctr, 0, sizeof(mdn::DevCounters)), "counters");  // the walk keeps them zero
  }
  p.hit = g->d_hit;
  p.ctr = g->d_ctr;
  // pixels per slab so that every trajectory of the slab can be a hitter, split evenly
  const uint64_t cap_px = std::max<uint64_t>(1, std::min(g->hit_cap, g->slab_limit) / (uint64_t)mb.nmat);
  const uint64_t nslab = ((uint64_t)p.nshard + cap_px - 1) / cap_px;
  g->last_nslab = (uint32_t)nslab;
  const uint64_t per = ((uint64_t)p.nshard + nslab - 1) / nslab;
  for (uint64_t p0 = 0; p0 < (uint64_t)p.nshard; p0 += per) {
    p.p0 = (uint32_t)p0;
    p.plen = (uint32_t)std::min<uint64_t>(per, (uint64_t)p.nshard - p0);
    MDN_CUDA(mdn::launch_mdnorm(p, mb, g->num_sms, s), "mdnorm kernels");
    g->path[0] = mdn::last_mdnorm_path();
  }
  return MDN_OK;
}

// Event row layout: stride floats per event; weight, error-squared (-1 = none) and Q columns.
struct EvLayout {
  int64_t stride;
  int32_t col_w, col_e, col_q;
};

mdn_status check_events(int64_t nevents, const float* events, const EvLayout& L) {
  if (nevents < 0) return fail(MDN_EINVAL, "nevents < 0");
  if (nevents > 0 && !events) return fail(MDN_EINVAL, "events is NULL");
  const bool bad_e = L.col_e >= 0 && (L.col_e >= L.stride || L.col_e == L.col_w ||
                                      (L.col_e >= L.col_q && L.col_e < L.col_q + 3));
  if (L.stride < 4 || L.col_w < 0 || L.col_q < 0 || L.col_e < -1 || L.col_w >= L.stride ||
      L.col_q + 3 > L.stride || (L.col_w >= L.col_q && L.col_w < L.col_q + 3) || bad_e)
    return fail(MDN_EINVAL, "bad event layout: stride %lld, col_w %d, col_e %d, col_q %d", (long long)L.stride,
                L.col_w, L.col_e, L.col_q);
  return MDN_OK;
}

mdn::BinParams bin_params(mdn_grid* g, const float* ev, int64_t n, const EvLayout& L, int32_t w0 = 0,
                          int32_t w1 = 0) {
  mdn::BinParams p{};
  p.g = g->g;
  p.events = ev;
  p.nevents = n;
  p.stride = L.stride;
  p.col_w = L.col_w;
  p.col_q = L.col_q;
  p.col_e = L.col_e;
  // fp32 fast-path axis order: fewest bins first (stable), so a thin slab axis rejects early; an
  // L2 slab launch (w1 > 0) tests the last axis first, with the slab as its window
  int ord[3] = {0, 1, 2};
  if (w1 > 0) {
    ord[0] = 2;
    ord[1] = 0;
    ord[2] = 1;
  } else {
    std::stable_sort(ord, ord + 3, [&](int a, int b) { return g->g.n[a] < g->g.n[b]; });
  }
  const int32_t stride[3] = {1, g->g.n[0], g->g.n[0] * g->g.n[1]};
  for (int a = 0; a < 3; ++a) {
    p.ord[a] = ord[a];
    p.st[a] = stride[ord[a]];
  }
  p.w0 = w1 > 0 ? w0 : 0;
  p.w1 = w1 > 0 ? w1 : g->g.n[ord[0]];
  p.acc_f32 = g->acc == MDN_ACC_F32;
  p.priv = g->priv;
  p.binmd = g->d_hist + g->g.nbins;
  p.err2 = g->d_hist + 2 * g->g.nbins;
  p.stats = g->stats_on ? g->d_stats : nullptr;
  return p;
}

// Run the BinMD kernel over host events through a two-slot staging ring: the H2D copy of chunk
// c+1 (copy stream) overlaps the scatter of chunk c (caller's stream).
mdn_status binmd_host_stream(mdn_grid* g, const MatBlock& mb, int64_t nevents, const float* events,
                             const EvLayout& L, cudaStream_t s, const void* tables) {
  const int64_t stride = L.stride;
  const int64_t chunk = std::max<int64_t>(1, (int64_t)(64ll << 20) / (int64_t)(4 * stride));  // 64 MB
  const size_t need = (size_t)(chunk * stride);
  if (g->stage_floats < need) {
    for (int i = 0; i < 2; ++i) {
      if (g->d_stage[i]) {
        cudaStreamSynchronize(s);
        cudaFree(g->d_stage[i]);
      }
      g->d_stage[i] = nullptr;
    }
    g->stage_floats = 0;
    for (int i = 0; i < 2; ++i) MDN_CUDA(cudaMalloc(&g->d_stage[i], need * sizeof(float)), "staging alloc");
    g->stage_floats = need;
  }
  if (!g->copy_stream) {
    MDN_CUDA(cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking), "copy stream");
    for (int i = 0; i < 2; ++i) {
      MDN_CUDA(cudaEventCreateWithFlags(&g->ev_ready[i], cudaEventDisableTiming), "event");
      MDN_CUDA(cudaEventCreateWithFlags(&g->ev_free[i], cudaEventDisableTiming), "event");
    }
  }
  // A slot may be refilled once the last kernel that read it is done: ev_free[slot] is recorded
  // after every scatter launch (never-recorded events are complete).  Nothing else orders the
  // copies after earlier work on the caller's stream, so the first chunks' H2D overlaps the
  // MDNorm kernels enqueued before this call.
  // The copies are ordered after the caller's last mdnorm_reset (the start of an accumulation
  // epoch), not after its MDNorm kernels, so they overlap MDNorm without starting before the
  // epoch the events belong to.
  if (g->ev_epoch) MDN_CUDA(cudaStreamWaitEvent(g->copy_stream, g->ev_epoch, 0), "wait");
  int64_t c = 0;
  for (int64_t off = 0; off < nevents; off += chunk, ++c) {
    const int slot = (int)(c & 1);
    const int64_t n = std::min(chunk, nevents - off);
    MDN_CUDA(cudaStreamWaitEvent(g->copy_stream, g->ev_free[slot], 0), "wait");
    MDN_CUDA(cudaMemcpyAsync(g->d_stage[slot], events + off * stride, sizeof(float) * n * stride,
                             cudaMemcpyHostToDevice, g->copy_stream), "H2D events");
    MDN_CUDA(cudaEventRecord(g->ev_ready[slot], g->copy_stream), "event record");
    MDN_CUDA(cudaStreamWaitEvent(s, g->ev_ready[slot], 0), "wait");
    mdn::BinParams p = bin_params(g, g->d_stage[slot], n, L);
    p.tables = tables;
    MDN_CUDA(mdn::launch_binmd(p, mb, g->num_sms, s), "binmd kernel");
    g->path[1] = mdn::last_binmd_path();
    MDN_CUDA(cudaEventRecord(g->ev_free[slot], s), "event record");
  }
  return MDN_OK;
}

// B0 of one BinMD call: the plan kernel on plan_stream into the next table buffer, ordered after
// the last kernels that read that buffer; returns the buffer (the caller's kernels wait on
// ev_tab_ready and record ev_tab_free after them).
mdn_status binmd_plan(mdn_grid* g, const MatBlock& mb, const EvLayout& L, cudaStream_t s, int* slot,
                      const float* box_bounds = nullptr, int64_t nboxes = 0, int32_t w0 = 0, int32_t w1 = 0) {
  if (!g->plan_stream) {
    MDN_CUDA(cudaStreamCreateWithFlags(&g->plan_stream, cudaStreamNonBlocking), "plan stream");
    for (int i = 0; i < 2; ++i) {
      MDN_CUDA(cudaEventCreateWithFlags(&g->ev_tab_ready[i], cudaEventDisableTiming), "event");
      MDN_CUDA(cudaEventCreateWithFlags(&g->ev_tab_free[i], cudaEventDisableTiming), "event");
    }
  }
  const int i = g->btab_i ^ 1;
  if (!g->d_btab[i]) MDN_CUDA(cudaMalloc(&g->d_btab[i], mdn::binmd_tables_bytes()), "binmd tables");

  // the plan reads only host-side parameters: it waits for nothing but the last kernels that read
  // this buffer (two calls back), so it runs as soon as the host enqueues it -- typically during
  // the previous call's kernels -- and is off the critical path
  MDN_CUDA(cudaStreamWaitEvent(g->plan_stream, g->ev_tab_free[i], 0), "wait");
  MDN_CUDA(mdn::launch_binmd_plan(bin_params(g, nullptr, 0, L, w0, w1), mb, g->d_btab[i], g->plan_stream),
           "binmd plan");
  if (box_bounds) {  // NEXT #4: the boxes that can reach the grid, after the plan's tables
    if (g->blist_cap[i] < nboxes + 1) {
      MDN_CUDA(cudaEventSynchronize(g->ev_tab_free[i]), "sync");
      cudaFree(g->d_blist[i]);
      g->d_blist[i] = nullptr;
      g->blist_cap[i] = 0;
      MDN_CUDA(cudaMalloc(&g->d_blist[i], sizeof(int32_t) * (size_t)(nboxes + 1)), "box list");
      g->blist_cap[i] = nboxes + 1;
    }
    MDN_CUDA(cudaMemsetAsync(g->d_blist[i], 0, sizeof(int32_t), g->plan_stream), "box count");
    mdn::BinParams bp = bin_params(g, nullptr, 0, L);
    bp.tables = g->d_btab[i];
    MDN_CUDA(mdn::launch_binmd_box_cull(bp, box_bounds, nboxes, g->d_blist[i] + 1,
                                        reinterpret_cast<unsigned*>(g->d_blist[i]), g->num_sms, g->plan_stream),
             "box cull");
  }
  MDN_CUDA(cudaEventRecord(g->ev_tab_ready[i], g->plan_stream), "event record");
  MDN_CUDA(cudaStreamWaitEvent(s, g->ev_tab_ready[i], 0), "wait");
  g->btab_i = i;
  *slot = i;
  return MDN_OK;
}

#ifndef MDN_BIN_SLAB_MB
#define MDN_BIN_SLAB_MB 80
#endif
// Slabs of the last axis for device-resident events when the fp64 binmd histogram is larger than
// the L2 (126 MB) can hold next to the event stream: each slab (at most MDN_BIN_SLAB_MB of bins,
// contiguous in memory) gets its own launch over all events, whose reductions then stay in L2.
// Without slabs every grid line is fetched from HBM once per op whose image passes over it (the
// Q-ordered stream visits a bin's 48 preimages at 48 unrelated times): on the 500^3 stress grid,
// 10^8 events x 48 ops, 27% of the reductions hit L2 and BinMD moved 90 GB of DRAM traffic.
// Measured (10^8 events): no slabs 36.6 ms; 20 / 40 / 60 / 80 / 100 / 120 / 160 MB slabs 32.4 /
// 20.7 / 16.8 / 14.8 / 15.3 / 17.6 / 20.4 ms.  Each slab re-reads the events (12 x 1.6 GB here).
int binmd_l2_slabs(const mdn_grid* g) {
  const uint64_t bytes = sizeof(double) * (uint64_t)g->g.nbins;
  const uint64_t cap = (uint64_t)MDN_BIN_SLAB_MB << 20;
  if (bytes <= cap + cap / 2 || g->g.n[2] < 2) return 1;
  return (int)std::min<uint64_t>((bytes + cap - 1) / cap, (uint64_t)g->g.n[2]);
}

mdn_status binmd_run(mdn_grid* g, const MatBlock& mb, int64_t nevents, const float* events, const EvLayout& L,
                     cudaStream_t s) {
  if (nevents == 0) return ok();
  int slot = 0;
  mdn_status st;
  const int nslab = is_device_ptr(events) ? binmd_l2_slabs(g) : 1;
  if (nslab > 1) {
    for (int k = 0; k < nslab; ++k) {
      const int32_t z0 = (int32_t)((int64_t)k * g->g.n[2] / nslab);
      const int32_t z1 = (int32_t)((int64_t)(k + 1) * g->g.n[2] / nslab);
      st = binmd_plan(g, mb, L, s, &slot, nullptr, 0, z0, z1);
      if (st != MDN_OK) return st;
      mdn::BinParams p = bin_params(g, events, nevents, L, z0, z1);
      p.tables = g->d_btab[slot];
      MDN_CUDA(mdn::launch_binmd(p, mb, g->num_sms, s), "binmd kernel");
      g->path[1] = mdn::last_binmd_path();
      MDN_CUDA(cudaEventRecord(g->ev_tab_free[slot], s), "event record");
    }
    return ok();
  }
  st = binmd_plan(g, mb, L, s, &slot);
  if (st != MDN_OK) return st;
  if (is_device_ptr(events)) {
    mdn::BinParams p = bin_params(g, events, nevents, L);
    p.tables = g->d_btab[slot];
    MDN_CUDA(mdn::launch_binmd(p, mb, g->num_sms, s), "binmd kernel");
    g->path[1] = mdn::last_binmd_path();
  } else {
    st = binmd_host_stream(g, mb, nevents, events, L, s, g->d_btab[slot]);
    if (st != MDN_OK) return st;
  }
  MDN_CUDA(cudaEventRecord(g->ev_tab_free[slot], s), "event record");
  return ok();
}

}  // namespace

extern "C" {

const char* mdn_last_error(void) { return g_err.c_str(); }

const char* mdn_version(void) { return "mdnorm sm_100a 0.1.0"; }

mdn_status mdnorm_create_grid(int device, const double lo[3], const double hi[3], const int64_t nbins[3],
                              const double W[9], mdn_acc acc, mdn_grid** out) {
  if (!out) return fail(MDN_EINVAL, "out is NULL");
  *out = nullptr;
  if (!lo || !hi || !nbins || !W) return fail(MDN_EINVAL, "NULL argument");
  int64_t total = 1;
  for (int a = 0; a < 3; ++a) {
    if (!(std::isfinite(lo[a]) && std::isfinite(hi[a]) && lo[a] < hi[a]))
      return fail(MDN_EINVAL, "axis %d: need finite lo < hi (got %g, %g)", a, lo[a], hi[a]);
    if (nbins[a] < 1 || nbins[a] > (1ll << 30)) return fail(MDN_EINVAL, "axis %d: nbins %lld outside [1, 2^30]", a, (long long)nbins[a]);
    total *= nbins[a];
    if (total >= (1ll << 31)) return fail(MDN_EINVAL, "grid too large (at most 2^31 - 1 bins)");
  }
  if (!finite_all(W, 9) || !nonsingular(W)) return fail(MDN_EINVAL, "W is singular or non-finite");
  if (acc != MDN_ACC_F64 && acc != MDN_ACC_F32) return fail(MDN_EINVAL, "unknown accumulation mode %d", (int)acc);
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
  if (device < 0 || device >= ndev) return fail(MDN_EINVAL, "device %d outside [0, %d)", device, ndev);
  DeviceGuard dg(device);
  mdn_grid* g = new mdn_grid;
  g->device = device;
  g->acc = acc;
  g->hit_cap_max = kMaxSlab;
  g->slab_limit = kMaxSlab;
  cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, device);
  for (int a = 0; a < 3; ++a) {
    g->g.lo[a] = lo[a];
    g->g.hi[a] = hi[a];
    g->g.n[a] = (int32_t)nbins[a];
    g->g.w[a] = (hi[a] - lo[a]) / (double)nbins[a];  // IEEE double, same as the device would
    g->g.s[a] = 1.0 / g->g.w[a];
    g->g.nd[a] = (double)nbins[a];
  }
  g->g.nbins = total;
  std::memcpy(g->W, W, sizeof g->W);
  e = cudaMalloc(&g->d_hist, sizeof(double) * 3 * (size_t)total);  // [norm | binmd | err2]
  if (e == cudaSuccess) e = cudaMemset(g->d_hist, 0, sizeof(double) * 3 * (size_t)total);
  if (e != cudaSuccess) {
    if (g->d_hist) cudaFree(g->d_hist);
    delete g;
    return cuda_fail(e, "histogram allocation");
  }
  *out = g;
  return ok();
}

mdn_status mdnorm_destroy(mdn_grid* g) {
  if (!g) return ok();
  DeviceGuard dg(g->device);
  cudaDeviceSynchronize();
  cudaFree(g->d_hist);
  cudaFree(g->d_pix);
  cudaFree(g->d_pkr);
  cudaFree(g->d_flux);
  cudaFree(g->d_ftab);
  cudaFree(g->d_ftab16);
  cudaFree(g->d_fviews);
  cudaFree(g->d_ptab);
  cudaFree(g->d_hit);
  cudaFree(g->d_ctr);
  cudaFree(g->d_xs);
  cudaFree(g->d_stats);
  for (int i = 0; i < 2; ++i) {
    cudaFree(g->d_stage[i]);
    if (g->ev_ready[i]) cudaEventDestroy(g->ev_ready[i]);
    if (g->ev_free[i]) cudaEventDestroy(g->ev_free[i]);
  }
  if (g->ev_epoch) cudaEventDestroy(g->ev_epoch);
  if (g->copy_stream) cudaStreamDestroy(g->copy_stream);
  for (int i = 0; i < 2; ++i) {
    cudaFree(g->d_btab[i]);
    cudaFree(g->d_blist[i]);
    if (g->ev_tab_ready[i]) cudaEventDestroy(g->ev_tab_ready[i]);
    if (g->ev_tab_free[i]) cudaEventDestroy(g->ev_tab_free[i]);
  }
  if (g->plan_stream) cudaStreamDestroy(g->plan_stream);
  delete g;
  cudaGetLastError();
  return ok();
}

mdn_status mdnorm_set_instrument(mdn_grid* g, int64_t npix, const double* dir, const double* solid) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (npix < 1 || !dir || !solid) return fail(MDN_EINVAL, "need npix >= 1 and non-NULL dir, solid");
  DeviceGuard dg(g->device);
  std::vector<double> hd, hs;
  MDN_CUDA(to_host(dir, 3 * npix, hd), "read dir");
  MDN_CUDA(to_host(solid, npix, hs), "read solid");
  if (!finite_all(hd.data(), 3 * npix)) return fail(MDN_EINVAL, "dir has non-finite values");
  // the cull's fp32 pre-test band scales with the largest |q_i| = |(-d_x, -d_y, 1 - d_z)_i| (2 for
  // unit directions): any direction table is accepted and decided exactly as the definition does
  double qmax = 2.0;
  for (int64_t i = 0; i < npix; ++i)
    qmax = std::max(qmax, std::max(std::fabs(hd[3 * i]), std::max(std::fabs(hd[3 * i + 1]), std::fabs(1.0 - hd[3 * i + 2]))));
  for (int64_t i = 0; i < npix; ++i)
    if (!(std::isfinite(hs[i]) && hs[i] >= 0.0)) return fail(MDN_EINVAL, "solid[%lld] = %g is not >= 0", (long long)i, hs[i]);
  double *d_dir = nullptr, *d_sol = nullptr;
  double4* d_pix = nullptr;
  cudaError_t e = cudaMalloc(&d_pix, sizeof(double4) * npix);
  if (e == cudaSuccess) e = cudaMalloc(&d_dir, sizeof(double) * 3 * npix);
  if (e == cudaSuccess) e = cudaMalloc(&d_sol, sizeof(double) * npix);
  if (e == cudaSuccess) e = cudaMemcpy(d_dir, hd.data(), sizeof(double) * 3 * npix, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d_sol, hs.data(), sizeof(double) * npix, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = mdn::launch_pixels_prepare(d_dir, d_sol, d_pix, npix, nullptr);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaFree(d_dir);
  cudaFree(d_sol);
  if (e != cudaSuccess) {
    cudaFree(d_pix);
    return cuda_fail(e, "set_instrument");
  }
  cudaFree(g->d_pix);
  cudaFree(g->d_pkr);  // per-pixel limits belong to the previous instrument
  g->d_pkr = nullptr;
  if (g->nftables > 1) {  // so does a pixel -> flux-table map: the tables must be set again
    cudaFree(g->d_flux);
    cudaFree(g->d_ftab);
    cudaFree(g->d_ftab16);
    cudaFree(g->d_fviews);
    cudaFree(g->d_ptab);
    g->d_flux = nullptr;
    g->d_ftab = nullptr;
    g->d_ftab16 = nullptr;
    g->d_fviews = nullptr;
    g->d_ptab = nullptr;
    g->nftables = 0;
  }
  g->d_pix = d_pix;
  g->npix = npix;
  g->qmax = qmax;
  return ok();
}

namespace {

// Host image of one flux table (M5, see flux_at in mdn_device.cuh): knots kappa_i + two +inf
// pads; per interval ka_i = (kappa_i, Phi_i), kb_i = (dPhi_i, y_i) with dPhi_i = Phi_{i+1} -
// Phi_i, y_i = 1 / (kappa_{i+1} - kappa_i) (IEEE double, the same roundings as the device); and
// the cell table over U(x) = (x - kappa_0) * inv_cell: entry c = s_c = max{i : U_i < c}, flagged
// when cell c holds more than three knots, when s_c does not exist (c = 0) or when c + 1 >
// U_{n-1}.  max(4n, range / (2.9 min spacing)) cells, at most 2^22.  This file is compiled with
// -ffp-contract=off, so U_i is exactly the device's dmul(dsub(x, kappa_0), inv_cell).
struct HostFluxTable {
  std::vector<double> kn;
  std::vector<double2> ka, kb;
  std::vector<int> tab;
  double k_first, F_first, k_last, F_last, inv_cell;
  int n, ntab;
  float ga = 0.f, gb = 0.f;
  int gmode = 0;
  double ghit = 0.0;
};

// Interval guess for flux_guess (mdn_device.cuh): fit i ~ (T(x) - T(kappa_0)) / dT for T(x) = x
// and T(x) = 1/x (knots uniform in wavelength), measure on 64 points per interval spread evenly
// over [kappa_0, kappa_{n-1}] how often the fp32 guess names x's interval, and keep the better
// transform if it is right at least kFluxGuessMin of the time (the guess never decides a value:
// a wrong one falls back to the cell-table search).
constexpr double kFluxGuessMin = 0.9;
void fit_flux_guess(const double* hk, int64_t n, HostFluxTable& t) {
  if (n > (1 << 24)) return;
  double best = 0.0;
  for (int mode = 1; mode <= 2; ++mode) {
    const double T0 = mode == 1 ? hk[0] : 1.0 / hk[0], T1 = mode == 1 ? hk[n - 1] : 1.0 / hk[n - 1];
    const double dT = (T1 - T0) / (double)(n - 1);
    if (!std::isfinite(dT) || dT == 0.0) continue;
    const float ga = (float)(1.0 / dT), gb = (float)(-T0 / dT);
    const int64_t npts = std::min<int64_t>(64 * (n - 1), 1 << 22);
    int64_t hit = 0, j = 0;
    for (int64_t s = 0; s < npts; ++s) {
      const double x = hk[0] + (hk[n - 1] - hk[0]) * ((double)s + 0.5) / (double)npts;
      while (j + 2 < n && hk[j + 1] <= x) ++j;  // x's interval
      const float xf = (float)x;
      const float u = mode == 1 ? xf : 1.0f / xf;
      const int64_t g = std::min<int64_t>(std::max<int64_t>((int64_t)std::floor(std::fma(u, ga, gb)), 0), n - 2);
      hit += g == j;
    }
    const double frac = (double)hit / (double)npts;
    if (frac >= kFluxGuessMin && frac > best) {
      best = frac;
      t.ghit = frac;
      t.gmode = mode;
      t.ga = ga;
      t.gb = gb;
    }
  }
}

mdn_status build_flux_table(const double* hk, const double* hF, int64_t n, HostFluxTable& t) {
  if (n < 2 || n > (1 << 28)) return fail(MDN_EINVAL, "a flux table needs 2 .. 2^28 knots (got %lld)", (long long)n);
  if (!finite_all(hk, n) || !finite_all(hF, n)) return fail(MDN_EINVAL, "flux table has non-finite values");
  for (int64_t i = 1; i < n; ++i) {
    if (!(hk[i] > hk[i - 1])) return fail(MDN_EINVAL, "flux k not strictly increasing at %lld", (long long)i);
    if (hF[i] < hF[i - 1]) return fail(MDN_EINVAL, "cumulative flux F decreases at %lld", (long long)i);
  }
  t.kn.assign(hk, hk + n);
  t.kn.push_back(HUGE_VAL);
  t.kn.push_back(HUGE_VAL);
  t.ka.assign((size_t)n, make_double2(0.0, 0.0));
  t.kb.assign((size_t)n, make_double2(0.0, 0.0));
  for (int64_t i = 0; i + 1 < n; ++i) {
    const double dk = hk[i + 1] - hk[i];
    const double dF = hF[i + 1] - hF[i];
    if (!std::isfinite(dk) || !std::isfinite(dF) || !std::isfinite(1.0 / dk))
      return fail(MDN_EINVAL, "flux table interval %lld overflows", (long long)i);
    t.ka[i] = make_double2(hk[i], hF[i]);
    t.kb[i] = make_double2(dF, 1.0 / dk);
  }
  t.ka[n - 1] = make_double2(hk[n - 1], hF[n - 1]);  // kappa_{n-1} for probes (MDN_FLUX_NOKN)
  // cells narrower than 3 x the smallest knot spacing hold at most 3 knots (all fast); eight cells
  // per knot (MDN_FLUX_CELLS) make a knot at or below x in x's own cell rare (one-probe look-up)
  double hmin = HUGE_VAL;
  for (int64_t i = 0; i + 1 < n; ++i) hmin = std::min(hmin, hk[i + 1] - hk[i]);
  const double want = std::ceil((hk[n - 1] - hk[0]) / (2.9 * hmin));
  const int ntab = (int)std::min<double>(std::max<double>((double)MDN_FLUX_CELLS * (double)n, want), (double)(1 << 22));
  t.inv_cell = (double)ntab / (hk[n - 1] - hk[0]);
  if (!std::isfinite(t.inv_cell)) return fail(MDN_EINVAL, "flux table k range too small");
  std::vector<double> U((size_t)n);
  for (int64_t i = 0; i < n; ++i) U[i] = (hk[i] - hk[0]) * t.inv_cell;
  t.tab.assign((size_t)ntab, 0);
  int64_t s = -1, j = 0;  // s = max{i : U_i < c}; j = first i with U_i >= c
  for (int c = 0; c < ntab; ++c) {
    while (j < n && U[j] < (double)c) s = j++;
    int64_t cnt = 0;
    while (j + cnt < n && U[j + cnt] < (double)c + 1.0) ++cnt;
    const bool fast = s >= 0 && cnt <= 3 && (double)c + 1.0 <= U[n - 1];
    t.tab[c] = (int)std::max<int64_t>(s, 0) | (fast ? 0 : (int)mdn::kFluxDense32);
  }
  t.k_first = hk[0];
  t.F_first = hF[0];
  t.k_last = hk[n - 1];
  t.F_last = hF[n - 1];
  t.n = (int)n;
  t.ntab = ntab;
  fit_flux_guess(hk, n, t);
  return MDN_OK;
}

}  // namespace

mdn_status mdnorm_set_flux_tables(mdn_grid* g, int32_t ntables, const int64_t* offsets, const double* k,
                                  const double* F, int64_t npix, const int32_t* pixel_table) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (ntables < 1 || ntables > (1 << 20) || !offsets || !k || !F)
    return fail(MDN_EINVAL, "need ntables >= 1 and non-NULL offsets, k, F");
  if (ntables > 1 && !pixel_table) return fail(MDN_EINVAL, "several flux tables need a pixel -> table map");
  if (pixel_table && (!g->d_pix || npix != g->npix))
    return fail(MDN_EINVAL, "the pixel -> table map needs npix == the instrument's (%lld)", (long long)g->npix);
  if (offsets[0] != 0) return fail(MDN_EINVAL, "offsets[0] must be 0");
  for (int t = 0; t < ntables; ++t)
    if (offsets[t + 1] - offsets[t] < 2) return fail(MDN_EINVAL, "flux table %d has fewer than 2 knots", t);
  const int64_t total = offsets[ntables];
  DeviceGuard dg(g->device);
  std::vector<double> hk, hF;
  MDN_CUDA(to_host(k, total, hk), "read k");
  MDN_CUDA(to_host(F, total, hF), "read F");
  std::vector<int32_t> hpt;
  if (pixel_table) {
    MDN_CUDA(to_host(pixel_table, npix, hpt), "read pixel table");
    for (int64_t i = 0; i < npix; ++i)
      if (hpt[i] < 0 || hpt[i] >= ntables) return fail(MDN_EINVAL, "pixel_table[%lld] = %d outside [0, %d)", (long long)i, hpt[i], ntables);
  }
  std::vector<HostFluxTable> tabs((size_t)ntables);
  mdn_status st;
  for (int t = 0; t < ntables; ++t)
    if ((st = build_flux_table(hk.data() + offsets[t], hF.data() + offsets[t], offsets[t + 1] - offsets[t],
                               tabs[t])) != MDN_OK)
      return st;
  // concatenate into one allocation: every table's knots (padded to an even count, so the
  // interval records stay 16-byte aligned), then every table's ka records, then every table's kb
  // records; the cell tables in a second allocation; one FluxView per table
  size_t nkn = 0, nrec = 0, ntb = 0;
  for (auto& t : tabs) {
    nkn += (t.kn.size() + 1) & ~size_t(1);
    nrec += t.ka.size();
    ntb += t.tab.size();
  }
  std::vector<double> all(nkn + 4 * nrec, 0.0);
  std::vector<int> all_tab;
  all_tab.reserve(ntb);
  std::vector<size_t> kn_off, ka_off, kb_off, tb_off;
  size_t o = 0, ao = nkn, bo = nkn + 2 * nrec;
  for (auto& t : tabs) {
    kn_off.push_back(o);
    ka_off.push_back(ao);
    kb_off.push_back(bo);
    tb_off.push_back(all_tab.size());
    std::copy(t.kn.begin(), t.kn.end(), all.begin() + o);
    std::memcpy(all.data() + ao, t.ka.data(), sizeof(double2) * t.ka.size());
    std::memcpy(all.data() + bo, t.kb.data(), sizeof(double2) * t.kb.size());
    o += (t.kn.size() + 1) & ~size_t(1);
    ao += 2 * t.ka.size();
    bo += 2 * t.kb.size();
    all_tab.insert(all_tab.end(), t.tab.begin(), t.tab.end());
  }
  double* d = nullptr;
  int* tab = nullptr;
  mdn::FluxView* views = nullptr;
  int32_t* ptab = nullptr;
  cudaError_t e = cudaMalloc(&d, sizeof(double) * all.size());
  if (e == cudaSuccess) e = cudaMalloc(&tab, sizeof(int) * ntb);
  if (e == cudaSuccess) e = cudaMalloc(&views, sizeof(mdn::FluxView) * ntables);
  if (e == cudaSuccess && pixel_table && ntables > 1) e = cudaMalloc(&ptab, sizeof(int32_t) * npix);
  std::vector<mdn::FluxView> hv((size_t)ntables);
  for (int t = 0; t < ntables; ++t) {
    mdn::FluxView& v = hv[t];
    v = mdn::FluxView{};
    v.kn = d + kn_off[t];
    v.ka = reinterpret_cast<const double2*>(d + ka_off[t]);
    v.kb = reinterpret_cast<const double2*>(d + kb_off[t]);
    v.tab = tab + tb_off[t];
    v.k_first = tabs[t].k_first;
    v.F_first = tabs[t].F_first;
    v.k_last = tabs[t].k_last;
    v.F_last = tabs[t].F_last;
    v.inv_cell = tabs[t].inv_cell;
    v.n = tabs[t].n;
    v.ntab = tabs[t].ntab;
    v.ga = tabs[t].ga;
    v.gb = tabs[t].gb;
    v.gmode = tabs[t].gmode;
  }
  if (e == cudaSuccess) e = cudaMemcpy(d, all.data(), sizeof(double) * all.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(tab, all_tab.data(), sizeof(int) * ntb, cudaMemcpyHostToDevice);
  // table 0's cells as the uint16 entries the walk stages into shared memory (flag bit 15), zero
  // padded to whole 16-byte groups; only when every interval index fits 15 bits
  uint16_t* tab16 = nullptr;
  if (e == cudaSuccess && tabs[0].n <= (1 << 15) - 1) {
    std::vector<uint16_t> t16((size_t)((tabs[0].ntab + 7) & ~7), 0);
    for (int i = 0; i < tabs[0].ntab; ++i) {
      const unsigned c = (unsigned)tabs[0].tab[(size_t)i];
      t16[(size_t)i] = (uint16_t)((c & (mdn::kFluxDense32 - 1)) | ((c & mdn::kFluxDense32) ? mdn::kFluxDense16 : 0u));
    }
    e = cudaMalloc(&tab16, sizeof(uint16_t) * t16.size());
    if (e == cudaSuccess) e = cudaMemcpy(tab16, t16.data(), sizeof(uint16_t) * t16.size(), cudaMemcpyHostToDevice);
    hv[0].tab16 = tab16;
  }
  if (e == cudaSuccess) e = cudaMemcpy(views, hv.data(), sizeof(mdn::FluxView) * ntables, cudaMemcpyHostToDevice);
  if (e == cudaSuccess && ptab) e = cudaMemcpy(ptab, hpt.data(), sizeof(int32_t) * npix, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    cudaFree(d);
    cudaFree(tab);
    cudaFree(views);
    cudaFree(ptab);
    cudaFree(tab16);
    return cuda_fail(e, "set_flux");
  }
  cudaDeviceSynchronize();
  cudaFree(g->d_flux);
  cudaFree(g->d_ftab);
  cudaFree(g->d_ftab16);
  g->d_ftab16 = tab16;
  cudaFree(g->d_fviews);
  cudaFree(g->d_ptab);
  g->d_flux = d;
  g->d_ftab = tab;
  g->d_fviews = views;
  g->d_ptab = ptab;
  g->nftables = ntables;
  g->fguess_hit.assign((size_t)ntables, 0.0);
  for (int t = 0; t < ntables; ++t) g->fguess_hit[(size_t)t] = tabs[t].gmode ? tabs[t].ghit : 0.0;
  g->flux0 = hv[0];
  return ok();
}

mdn_status mdnorm_set_flux(mdn_grid* g, int64_t n, const double* k, const double* F) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (n < 2 || !k || !F) return fail(MDN_EINVAL, "need n >= 2 and non-NULL k, F");
  const int64_t offsets[2] = {0, n};
  return mdnorm_set_flux_tables(g, 1, offsets, k, F, 0, nullptr);
}

mdn_status mdnorm_accumulate_runs(mdn_grid* g, const double UB[9], int32_t nruns, const double* R,
                                  const double* charge, int32_t nops, const double* ops, double k_min,
                                  double k_max, int64_t pix_begin, int64_t pix_end, int64_t pix_stride,
                                  void* stream) {
  mdn_status st;
  if ((st = check_ready(g)) != MDN_OK) return st;
  if ((st = check_matrix(UB, "UB")) != MDN_OK) return st;
  if ((st = check_ops(nops, ops)) != MDN_OK) return st;
  if ((st = check_krange(k_min, k_max)) != MDN_OK) return st;
  if (nruns < 0 || (nruns > 0 && (!R || !charge))) return fail(MDN_EINVAL, "bad runs (nruns %d)", nruns);
  for (int r = 0; r < nruns; ++r) {
    if ((st = check_matrix(R + 9 * r, "R")) != MDN_OK) return st;
    if (!(std::isfinite(charge[r]) && charge[r] >= 0.0)) return fail(MDN_EINVAL, "charge[%d] = %g is not >= 0", r, charge[r]);
  }
  int64_t nshard = 0;
  if ((st = shard(g, pix_begin, pix_end, pix_stride, &nshard)) != MDN_OK) return st;
  DeviceGuard dg(g->device);
  cudaStream_t s = (cudaStream_t)stream;
  const mdn::MdnParams p = mdn_params(g, k_min, k_max, pix_begin, pix_stride, nshard);
  const int per_launch = std::max(1, std::min(mdn::kRunsPerLaunch, 384 / nops));
  for (int r0 = 0; r0 < nruns; r0 += per_launch) {
    const int nr = std::min(per_launch, nruns - r0);
    MatBlock mb{};
    mb.compose = 1;
    mb.nops = nops;
    mb.nruns = nr;
    mb.nmat = nr * nops;
    std::memcpy(mb.UB, UB, sizeof mb.UB);
    std::memcpy(mb.W, g->W, sizeof mb.W);
    std::memcpy(mb.u.c.ops, ops, sizeof(double) * 9 * nops);
    std::memcpy(mb.u.c.R, R + 9 * r0, sizeof(double) * 9 * nr);
    std::memcpy(mb.charge, charge + r0, sizeof(double) * nr);
    if ((st = run_mdnorm(g, p, mb, s)) != MDN_OK) return st;
  }
  return ok();
}

mdn_status mdnorm_accumulate(mdn_grid* g, const double UB[9], const double R[9], int32_t nops, const double* ops,
                             double k_min, double k_max, double proton_charge, int64_t pix_begin, int64_t pix_end,
                             int64_t pix_stride, void* stream) {
  return mdnorm_accumulate_runs(g, UB, 1, R, &proton_charge, nops, ops, k_min, k_max, pix_begin, pix_end,
                                pix_stride, stream);
}

mdn_status binmd_accumulate_err(mdn_grid* g, const double UB[9], int32_t nops, const double* ops,
                                int64_t nevents, const float* events, int64_t stride_floats, int32_t col_w,
                                int32_t col_e, int32_t col_q, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  mdn_status st;
  const EvLayout L{stride_floats, col_w, col_e, col_q};
  if ((st = check_matrix(UB, "UB")) != MDN_OK) return st;
  if ((st = check_ops(nops, ops)) != MDN_OK) return st;
  if ((st = check_events(nevents, events, L)) != MDN_OK) return st;
  DeviceGuard dg(g->device);
  MatBlock mb{};
  mb.compose = 1;
  mb.nops = nops;
  mb.nmat = nops;
  std::memcpy(mb.UB, UB, sizeof mb.UB);
  std::memcpy(mb.W, g->W, sizeof mb.W);
  std::memcpy(mb.u.c.ops, ops, sizeof(double) * 9 * nops);
  return binmd_run(g, mb, nevents, events, L, (cudaStream_t)stream);
}

mdn_status binmd_accumulate(mdn_grid* g, const double UB[9], int32_t nops, const double* ops, int64_t nevents,
                            const float* events, int64_t stride_floats, int32_t col_w, int32_t col_q, void* stream) {
  return binmd_accumulate_err(g, UB, nops, ops, nevents, events, stride_floats, col_w, -1, col_q, stream);
}

mdn_status binmd_box_bounds(mdn_grid* g, int64_t nevents, const float* events, int32_t box_events, float* bounds,
                            void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (nevents < 0 || box_events < 32 || (box_events & (box_events - 1)))
    return fail(MDN_EINVAL, "need nevents >= 0 and box_events a power of two >= 32 (got %lld, %d)",
                (long long)nevents, box_events);
  if (nevents == 0) return ok();
  if (!events || !bounds) return fail(MDN_EINVAL, "events or bounds is NULL");
  DeviceGuard dg(g->device);
  if (!is_device_ptr(events) || !is_device_ptr(bounds)) return fail(MDN_EINVAL, "events and bounds must be device arrays");
  if (reinterpret_cast<uintptr_t>(events) & 15) return fail(MDN_EINVAL, "events must be 16-byte aligned float4 rows");
  MDN_CUDA(mdn::launch_binmd_box_bounds(reinterpret_cast<const float4*>(events), nevents, box_events, bounds,
                                        g->num_sms, (cudaStream_t)stream), "box bounds");
  return ok();
}

mdn_status binmd_accumulate_boxes(mdn_grid* g, const double UB[9], int32_t nops, const double* ops, int64_t nevents,
                                  const float* events, int32_t box_events, const float* bounds, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  mdn_status st;
  const EvLayout L{4, 0, -1, 1};
  if ((st = check_matrix(UB, "UB")) != MDN_OK) return st;
  if ((st = check_ops(nops, ops)) != MDN_OK) return st;
  if ((st = check_events(nevents, events, L)) != MDN_OK) return st;
  if (box_events < 32 || (box_events & (box_events - 1)))
    return fail(MDN_EINVAL, "box_events must be a power of two >= 32 (got %d)", box_events);
  if (nevents == 0) return ok();
  if (!bounds) return fail(MDN_EINVAL, "bounds is NULL");
  DeviceGuard dg(g->device);
  if (!is_device_ptr(events) || !is_device_ptr(bounds)) return fail(MDN_EINVAL, "events and bounds must be device arrays");
  if (reinterpret_cast<uintptr_t>(events) & 15) return fail(MDN_EINVAL, "events must be 16-byte aligned float4 rows");
  cudaStream_t s = (cudaStream_t)stream;
  MatBlock mb{};
  mb.compose = 1;
  mb.nops = nops;
  mb.nmat = nops;
  std::memcpy(mb.UB, UB, sizeof mb.UB);
  std::memcpy(mb.W, g->W, sizeof mb.W);
  std::memcpy(mb.u.c.ops, ops, sizeof(double) * 9 * nops);
  const int64_t nboxes = (nevents + box_events - 1) / box_events;
  int slot = 0;
  if ((st = binmd_plan(g, mb, L, s, &slot, bounds, nboxes)) != MDN_OK) return st;
  mdn::BinParams p = bin_params(g, events, nevents, L);
  p.tables = g->d_btab[slot];
  p.box_list = g->d_blist[slot] + 1;
  p.box_count = reinterpret_cast<const unsigned*>(g->d_blist[slot]);
  int lg = 0;
  while ((32 << lg) < box_events) ++lg;
  p.box_log2 = lg;
  MDN_CUDA(mdn::launch_binmd(p, mb, g->num_sms, s), "binmd kernel");
  g->path[1] = mdn::last_binmd_path();
  MDN_CUDA(cudaEventRecord(g->ev_tab_free[slot], s), "event record");
  return ok();
}

mdn_status mdnorm_histograms(mdn_grid* g, void** norm_dev, void** binmd_dev, int64_t* nbins_total) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (norm_dev) *norm_dev = g->d_hist;
  if (binmd_dev) *binmd_dev = g->d_hist + g->g.nbins;
  if (nbins_total) *nbins_total = g->g.nbins;
  return ok();
}

mdn_status mdnorm_error_histogram(mdn_grid* g, void** err2_dev) {
  if (!g || !err2_dev) return fail(MDN_EINVAL, "NULL argument");
  *err2_dev = g->d_hist + 2 * g->g.nbins;
  return ok();
}

mdn_status mdnorm_set_pixel_krange(mdn_grid* g, int64_t npix, const double* kmin, const double* kmax) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (!kmin && !kmax) {
    DeviceGuard dg(g->device);
    cudaDeviceSynchronize();
    cudaFree(g->d_pkr);
    g->d_pkr = nullptr;
    return ok();
  }
  if (!g->d_pix) return fail(MDN_ESTATE, "mdnorm_set_instrument has not been called");
  if (!kmin || !kmax) return fail(MDN_EINVAL, "give both kmin and kmax (or neither)");
  if (npix != g->npix) return fail(MDN_EINVAL, "npix %lld != instrument's %lld", (long long)npix, (long long)g->npix);
  DeviceGuard dg(g->device);
  std::vector<double> lo, hi;
  MDN_CUDA(to_host(kmin, npix, lo), "read kmin");
  MDN_CUDA(to_host(kmax, npix, hi), "read kmax");
  std::vector<double2> r((size_t)npix);
  for (int64_t i = 0; i < npix; ++i) {
    if (std::isnan(lo[i]) || std::isnan(hi[i])) return fail(MDN_EINVAL, "NaN momentum limit at pixel %lld", (long long)i);
    r[i] = make_double2(lo[i], hi[i]);
  }
  double2* d = nullptr;
  cudaError_t e = cudaMalloc(&d, sizeof(double2) * npix);
  if (e == cudaSuccess) e = cudaMemcpy(d, r.data(), sizeof(double2) * npix, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    cudaFree(d);
    return cuda_fail(e, "set_pixel_krange");
  }
  cudaDeviceSynchronize();
  cudaFree(g->d_pkr);
  g->d_pkr = d;
  return ok();
}

mdn_status mdnorm_cross_section_err(mdn_grid* g, double* xs, double* xs_err, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (!xs || !xs_err) return fail(MDN_EINVAL, "xs or xs_err is NULL");
  const bool dx = is_device_ptr(xs), de = is_device_ptr(xs_err);
  if (dx != de) return fail(MDN_EINVAL, "xs and xs_err must both be host or both device arrays");
  DeviceGuard dg(g->device);
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t n = g->g.nbins;
  const double* h = g->d_hist;
  if (dx) {
    MDN_CUDA(mdn::launch_cross_section_err(h, h + n, h + 2 * n, xs, xs_err, n, g->num_sms, s), "xs kernel");
    return ok();
  }
  double* d2 = nullptr;
  MDN_CUDA(cudaMallocAsync(&d2, sizeof(double) * 2 * n, s), "xs scratch");
  cudaError_t e = mdn::launch_cross_section_err(h, h + n, h + 2 * n, d2, d2 + n, n, g->num_sms, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(xs, d2, sizeof(double) * n, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(xs_err, d2 + n, sizeof(double) * n, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d2, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "xs_err");
  return ok();
}

mdn_status mdn_divide(int device, const double* norm, const double* binmd, double* xs, int64_t n,
                      void* stream) {
  if (n < 0) return fail(MDN_EINVAL, "n < 0");
  if (n == 0) return ok();
  if (!norm || !binmd || !xs) return fail(MDN_EINVAL, "NULL argument");
  int ndev = 0;
  MDN_CUDA(cudaGetDeviceCount(&ndev), "cudaGetDeviceCount");
  if (device < 0 || device >= ndev) return fail(MDN_EINVAL, "device %d outside [0, %d)", device, ndev);
  DeviceGuard dg(device);
  if (!is_device_ptr(norm) || !is_device_ptr(binmd) || !is_device_ptr(xs))
    return fail(MDN_EINVAL, "mdn_divide needs device arrays");
  int nsm = 148;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device);
  MDN_CUDA(mdn::launch_cross_section(norm, binmd, xs, n, nsm, (cudaStream_t)stream), "xs kernel");
  return ok();
}

mdn_status mdnorm_cross_section(mdn_grid* g, double* xs, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (!xs) return fail(MDN_EINVAL, "xs is NULL");
  DeviceGuard dg(g->device);
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t n = g->g.nbins;
  if (is_device_ptr(xs)) {
    MDN_CUDA(mdn::launch_cross_section(g->d_hist, g->d_hist + n, xs, n, g->num_sms, s), "xs kernel");
    return ok();
  }
  if (!g->d_xs) MDN_CUDA(cudaMalloc(&g->d_xs, sizeof(double) * n), "xs scratch");
  MDN_CUDA(mdn::launch_cross_section(g->d_hist, g->d_hist + n, g->d_xs, n, g->num_sms, s), "xs kernel");
  MDN_CUDA(cudaMemcpyAsync(xs, g->d_xs, sizeof(double) * n, cudaMemcpyDeviceToHost, s), "D2H xs");
  MDN_CUDA(cudaStreamSynchronize(s), "sync");
  return ok();
}

mdn_status mdnorm_reset(mdn_grid* g, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  DeviceGuard dg(g->device);
  MDN_CUDA(cudaMemsetAsync(g->d_hist, 0, sizeof(double) * 3 * g->g.nbins, (cudaStream_t)stream), "memset");
  if (g->d_stats) MDN_CUDA(cudaMemsetAsync(g->d_stats, 0, sizeof(unsigned long long) * 6, (cudaStream_t)stream), "memset");
  if (!g->ev_epoch) MDN_CUDA(cudaEventCreateWithFlags(&g->ev_epoch, cudaEventDisableTiming), "event");
  MDN_CUDA(cudaEventRecord(g->ev_epoch, (cudaStream_t)stream), "event record");
  return ok();
}

mdn_status mdnorm_set_privatization(mdn_grid* g, int32_t mode) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (mode < -1 || mode > 1) return fail(MDN_EINVAL, "privatization mode must be -1, 0 or 1");
  g->priv = mode;
  return ok();
}

mdn_status mdnorm_accumulation_paths(mdn_grid* g, int32_t out[2]) {
  if (!g || !out) return fail(MDN_EINVAL, "NULL argument");
  out[0] = g->path[0];
  out[1] = g->path[1];
  return ok();
}

mdn_status mdnorm_stats(mdn_grid* g, int enable, int64_t out[6]) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (enable < -1 || enable > 1) return fail(MDN_EINVAL, "enable must be -1, 0 or 1");
  DeviceGuard dg(g->device);
  if (!g->d_stats) {
    MDN_CUDA(cudaMalloc(&g->d_stats, sizeof(unsigned long long) * 6), "stats alloc");
    MDN_CUDA(cudaMemset(g->d_stats, 0, sizeof(unsigned long long) * 6), "stats memset");
  }
  if (enable >= 0) g->stats_on = enable == 1;
  if (out) {
    unsigned long long h[6];
    MDN_CUDA(cudaDeviceSynchronize(), "sync");
    MDN_CUDA(cudaMemcpy(h, g->d_stats, sizeof h, cudaMemcpyDeviceToHost), "stats D2H");
    for (int i = 0; i < 6; ++i) out[i] = (int64_t)h[i];
  }
  return ok();
}

// ------------------------------------------------------------------ parity / test entry points

mdn_status mdnorm_accumulate_matrices(mdn_grid* g, int32_t nmat, const double* M, const double* charge,
                                      double k_min, double k_max, int64_t pix_begin, int64_t pix_end,
                                      int64_t pix_stride, void* stream) {
  mdn_status st;
  if ((st = check_ready(g)) != MDN_OK) return st;
  if (nmat < 1 || nmat > MDN_MAX_MATS || !M || !charge) return fail(MDN_EINVAL, "nmat %d outside [1, %d]", nmat, MDN_MAX_MATS);
  if (!finite_all(M, 9 * (int64_t)nmat) || !finite_all(charge, nmat)) return fail(MDN_EINVAL, "non-finite matrices");
  for (int m = 0; m < nmat; ++m)
    if (charge[m] < 0) return fail(MDN_EINVAL, "charge[%d] < 0", m);
  if ((st = check_krange(k_min, k_max)) != MDN_OK) return st;
  int64_t nshard = 0;
  if ((st = shard(g, pix_begin, pix_end, pix_stride, &nshard)) != MDN_OK) return st;
  DeviceGuard dg(g->device);
  MatBlock mb{};
  mb.compose = 0;
  mb.nmat = nmat;
  std::memcpy(mb.u.M, M, sizeof(double) * 9 * nmat);
  std::memcpy(mb.charge, charge, sizeof(double) * nmat);
  if ((st = run_mdnorm(g, mdn_params(g, k_min, k_max, pix_begin, pix_stride, nshard), mb, (cudaStream_t)stream)) !=
      MDN_OK)
    return st;
  return ok();
}

mdn_status binmd_accumulate_matrices(mdn_grid* g, int32_t nmat, const double* N, int64_t nevents, const float* events,
                                     int64_t stride_floats, int32_t col_w, int32_t col_q, void* stream) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (nmat < 1 || nmat > MDN_MAX_MATS || !N) return fail(MDN_EINVAL, "nmat %d outside [1, %d]", nmat, MDN_MAX_MATS);
  if (!finite_all(N, 9 * (int64_t)nmat)) return fail(MDN_EINVAL, "non-finite matrices");
  mdn_status st;
  if ((st = check_events(nevents, events, EvLayout{stride_floats, col_w, -1, col_q})) != MDN_OK) return st;
  DeviceGuard dg(g->device);
  MatBlock mb{};
  mb.compose = 0;
  mb.nmat = nmat;
  std::memcpy(mb.u.M, N, sizeof(double) * 9 * nmat);
  return binmd_run(g, mb, nevents, events, EvLayout{stride_floats, col_w, -1, col_q}, (cudaStream_t)stream);
}

mdn_status mdnorm_debug_trajectories(mdn_grid* g, int32_t nmat, const double* M, const double* charge,
                                     double k_min, double k_max, int64_t ntraj, const int64_t* traj_ids,
                                     int32_t* n_cross, int32_t* n_seg, int64_t* seg_bins, double* seg_vals,
                                     int64_t max_segs) {
  mdn_status st;
  if ((st = check_ready(g)) != MDN_OK) return st;
  if (nmat < 1 || nmat > MDN_MAX_MATS || !M || !charge) return fail(MDN_EINVAL, "nmat %d outside [1, %d]", nmat, MDN_MAX_MATS);
  if ((st = check_krange(k_min, k_max)) != MDN_OK) return st;
  if (ntraj < 0 || max_segs < 0 || (ntraj > 0 && (!traj_ids || !n_cross || !n_seg)) ||
      (max_segs > 0 && ntraj > 0 && (!seg_bins || !seg_vals)))
    return fail(MDN_EINVAL, "bad debug arguments");
  for (int64_t t = 0; t < ntraj; ++t)
    if (traj_ids[t] < 0 || traj_ids[t] >= (int64_t)nmat * g->npix) return fail(MDN_EINVAL, "traj id %lld out of range", (long long)traj_ids[t]);
  if (ntraj == 0) return ok();
  DeviceGuard dg(g->device);
  MatBlock mb{};
  mb.compose = 0;
  mb.nmat = nmat;
  std::memcpy(mb.u.M, M, sizeof(double) * 9 * nmat);
  std::memcpy(mb.charge, charge, sizeof(double) * nmat);
  const int64_t ms = std::max<int64_t>(max_segs, 1);
  int64_t* d_ids = nullptr;
  int32_t* d_nc = nullptr;
  int32_t* d_ns = nullptr;
  int64_t* d_bins = nullptr;
  double* d_vals = nullptr;
  cudaError_t e = cudaMalloc(&d_ids, sizeof(int64_t) * ntraj);
  if (e == cudaSuccess) e = cudaMalloc(&d_nc, sizeof(int32_t) * ntraj);
  if (e == cudaSuccess) e = cudaMalloc(&d_ns, sizeof(int32_t) * ntraj);
  if (e == cudaSuccess) e = cudaMalloc(&d_bins, sizeof(int64_t) * ntraj * ms);
  if (e == cudaSuccess) e = cudaMalloc(&d_vals, sizeof(double) * ntraj * ms);
  if (e == cudaSuccess) e = cudaMemcpy(d_ids, traj_ids, sizeof(int64_t) * ntraj, cudaMemcpyHostToDevice);
  if (e == cudaSuccess)
    e = mdn::launch_debug_traj(mdn_params(g, k_min, k_max, 0, 1, 0), mb, ntraj, d_ids, g->npix, d_nc, d_ns, d_bins,
                               d_vals, max_segs, nullptr);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(n_cross, d_nc, sizeof(int32_t) * ntraj, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemcpy(n_seg, d_ns, sizeof(int32_t) * ntraj, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && max_segs > 0) e = cudaMemcpy(seg_bins, d_bins, sizeof(int64_t) * ntraj * max_segs, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && max_segs > 0) e = cudaMemcpy(seg_vals, d_vals, sizeof(double) * ntraj * max_segs, cudaMemcpyDeviceToHost);
  cudaFree(d_ids);
  cudaFree(d_nc);
  cudaFree(d_ns);
  cudaFree(d_bins);
  cudaFree(d_vals);
  if (e != cudaSuccess) return cuda_fail(e, "debug trajectories");
  return ok();
}

mdn_status binmd_debug_bins(mdn_grid* g, int32_t nmat, const double* N, int64_t nevents, const float* events,
                            int64_t stride_floats, int32_t col_w, int32_t col_q, int64_t* bins) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (nmat < 1 || nmat > MDN_MAX_MATS || !N || !bins) return fail(MDN_EINVAL, "bad debug arguments");
  mdn_status st;
  if ((st = check_events(nevents, events, EvLayout{stride_floats, col_w, -1, col_q})) != MDN_OK) return st;
  if (nevents == 0) return ok();
  DeviceGuard dg(g->device);
  MatBlock mb{};
  mb.compose = 0;
  mb.nmat = nmat;
  std::memcpy(mb.u.M, N, sizeof(double) * 9 * nmat);
  float* d_ev = nullptr;
  int64_t* d_bins = nullptr;
  const bool dev = is_device_ptr(events);
  cudaError_t e = cudaSuccess;
  if (!dev) {
    e = cudaMalloc(&d_ev, sizeof(float) * nevents * stride_floats);
    if (e == cudaSuccess) e = cudaMemcpy(d_ev, events, sizeof(float) * nevents * stride_floats, cudaMemcpyHostToDevice);
  }
  if (e == cudaSuccess) e = cudaMalloc(&d_bins, sizeof(int64_t) * nevents * nmat);
  if (e == cudaSuccess)
    e = mdn::launch_debug_bins(bin_params(g, dev ? events : d_ev, nevents, EvLayout{stride_floats, col_w, -1, col_q}), mb, d_bins,
                               nullptr);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(bins, d_bins, sizeof(int64_t) * nevents * nmat, cudaMemcpyDeviceToHost);
  cudaFree(d_ev);
  cudaFree(d_bins);
  if (e != cudaSuccess) return cuda_fail(e, "debug bins");
  return ok();
}

mdn_status mdnorm_debug_set_max_slab(mdn_grid* g, int64_t max_traj) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  if (max_traj < 0 || max_traj > (int64_t)kMaxSlab)
    return fail(MDN_EINVAL, "max_traj %lld outside [0, %u]", (long long)max_traj, kMaxSlab);
  g->slab_limit = max_traj == 0 ? kMaxSlab : (uint32_t)max_traj;
  return ok();
}

mdn_status mdnorm_debug_last_launch(mdn_grid* g, int64_t out[4]) {
  if (!g || !out) return fail(MDN_EINVAL, "NULL argument");
  DeviceGuard dg(g->device);
  mdn::DevCounters c{};
  if (g->d_ctr) {
    MDN_CUDA(cudaDeviceSynchronize(), "sync");
    MDN_CUDA(cudaMemcpy(&c, g->d_ctr, sizeof c, cudaMemcpyDeviceToHost), "counters D2H");
  }
  out[0] = g->last_nslab;
  out[1] = c.last_nhit;
  out[2] = mdn::walk_big_claim_threshold(g->g.n[2] > 1, g->num_sms);
  out[3] = g->slab_limit;
  return ok();
}

mdn_status mdnorm_debug_flux_guess(mdn_grid* g, int32_t table, double out[2]) {
  if (!g || !out) return fail(MDN_EINVAL, "NULL argument");
  if (table < 0 || table >= g->nftables) return fail(MDN_EINVAL, "table %d outside [0, %d)", table, g->nftables);
  std::vector<mdn::FluxView> hv(1);
  DeviceGuard dg(g->device);
  MDN_CUDA(cudaMemcpy(hv.data(), g->d_fviews + table, sizeof(mdn::FluxView), cudaMemcpyDeviceToHost), "view D2H");
  out[0] = (double)hv[0].gmode;
  out[1] = g->fguess_hit[(size_t)table];
  return ok();
}

mdn_status mdnorm_debug_compose(mdn_grid* g, const double UB[9], int32_t nruns, const double* R, int32_t nops,
                                const double* ops, double* M, double* N) {
  if (!g) return fail(MDN_EINVAL, "grid is NULL");
  mdn_status st;
  if ((st = check_matrix(UB, "UB")) != MDN_OK) return st;
  if ((st = check_ops(nops, ops)) != MDN_OK) return st;
  if (nruns < 1 || nruns > mdn::kRunsPerLaunch || !R || !M || !N) return fail(MDN_EINVAL, "bad debug arguments");
  DeviceGuard dg(g->device);
  MatBlock a{}, b{};
  a.compose = b.compose = 1;
  a.nops = b.nops = nops;
  a.nruns = nruns;
  a.nmat = nruns * nops;
  b.nmat = nops;
  std::memcpy(a.UB, UB, sizeof a.UB);
  std::memcpy(b.UB, UB, sizeof b.UB);
  std::memcpy(a.W, g->W, sizeof a.W);
  std::memcpy(b.W, g->W, sizeof b.W);
  std::memcpy(a.u.c.ops, ops, sizeof(double) * 9 * nops);
  std::memcpy(b.u.c.ops, ops, sizeof(double) * 9 * nops);
  std::memcpy(a.u.c.R, R, sizeof(double) * 9 * nruns);
  double *dM = nullptr, *dN = nullptr;
  int32_t* dok = nullptr;
  int32_t hok = 1;
  cudaError_t e = cudaMalloc(&dM, sizeof(double) * 9 * a.nmat);
  if (e == cudaSuccess) e = cudaMalloc(&dN, sizeof(double) * 9 * nops);
  if (e == cudaSuccess) e = cudaMalloc(&dok, sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMemcpy(dok, &hok, sizeof hok, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = mdn::launch_debug_compose(a, b, dM, dN, dok, nullptr);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(M, dM, sizeof(double) * 9 * a.nmat, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemcpy(N, dN, sizeof(double) * 9 * nops, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemcpy(&hok, dok, sizeof hok, cudaMemcpyDeviceToHost);
  cudaFree(dM);
  cudaFree(dN);
  cudaFree(dok);
  if (e != cudaSuccess) return cuda_fail(e, "debug compose");
  if (!hok) return fail(MDN_EINVAL, "a composed matrix is singular");
  return ok();
}

}  // extern "C"
