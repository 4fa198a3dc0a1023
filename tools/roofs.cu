// roofs.cu -- G5 microbenchmarks: the "atomic roof" and the fp64 ALU
// rate that bound the MDNorm walk (M7: one fp64 reduction per segment) and BinMD (B3), measured on
// this B200 at whatever clock the driver runs it (no clock changes).  Not part of the product: a
// standalone executable that prints one JSON object; bench.py / DESIGN.md quote its numbers.
//
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o tools/roofs tools/roofs.cu \
//        -L/usr/local/cuda/lib64/stubs -lnvidia-ml
//   tools/roofs > profiles/rNN_roofs.json
// Every case records the SM clock (NVML, sampled every 0.5 ms while it runs: median and
// minimum) and the OR of the clock-event (throttle) reasons seen, so a roof carries its clock.
//
// Cases (all reductions compile to RED.E.ADD: the return value is unused):
//   red_f64_random  S    fp64 red.global.add to uniformly random bins of an S-byte histogram
//   red_f64_walk    S    fp64 red.global.add along random 3-D DDA walks (+1 / +n0 / +n0 n1 steps,
//                        the access pattern of a trajectory's consecutive segments)
//   red_f32_random  S    the same with fp32
//   red_shared_f64       fp64 atomicAdd to shared memory (privatised accumulation)
//   red_shared_f32       fp32 atomicAdd to shared memory (MDN_ACC_F32 partials)
//   red_dsmem_f64        fp64 atomicAdd to random bins of a histogram distributed over the shared
//                        memory of an 8-CTA cluster (red.shared::cluster via map_shared_rank)
//   fp64_alu             independent DADD/DMUL chains (FP64-pipe rate, no FMA)
// Histogram sizes: CORELLI 600x600 (2.88 MB), TOPAZ 200^3 (64 MB), stress 500^3 (1 GB).
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <algorithm>
#include <atomic>
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <nvml.h>
#include <thread>
#include <vector>
namespace cg = cooperative_groups;

#define CK(x)                                                                         \
  do {                                                                                \
    cudaError_t e_ = (x);                                                             \
    if (e_ != cudaSuccess) {                                                          \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_));      \
      exit(1);                                                                        \
    }                                                                                 \
  } while (0)

__device__ __forceinline__ uint32_t xs32(uint32_t& s) {
  s ^= s << 13;
  s ^= s >> 17;
  s ^= s << 5;
  return s;
}
__device__ __forceinline__ uint32_t below(uint32_t x, uint32_t n) {
  return (uint32_t)(((uint64_t)x * n) >> 32);
}

template <typename T>
__global__ void red_random(T* h, uint32_t nbins, int iters) {
  uint32_t s = 0x9e3779b9u ^ (blockIdx.x * blockDim.x + threadIdx.x) * 0x85ebca6bu;
  xs32(s);
  for (int i = 0; i < iters; ++i) atomicAdd(h + below(xs32(s), nbins), (T)1);
}

// one thread = a sequence of walks of `len` steps; each step moves one bin along a random axis
__global__ void red_walk(double* h, uint32_t n0, uint32_t n1, uint32_t n2, int iters, int len) {
  uint32_t s = 0x1234567u ^ (blockIdx.x * blockDim.x + threadIdx.x) * 0x27d4eb2du;
  xs32(s);
  const uint32_t nb = n0 * n1 * n2;
  for (int w = 0; w < iters / len; ++w) {
    uint32_t b = below(xs32(s), nb);
    for (int i = 0; i < len; ++i) {
      atomicAdd(h + b, 1.0);
      const uint32_t r = xs32(s) % 3u;
      const uint32_t st = r == 0 ? 1u : (r == 1 ? n0 : n0 * n1);
      b += st;
      if (b >= nb) b -= nb;
    }
  }
}

__global__ void red_shared(double* out, int iters, uint32_t nbins) {
  extern __shared__ double sh[];
  for (uint32_t i = threadIdx.x; i < nbins; i += blockDim.x) sh[i] = 0.0;
  __syncthreads();
  uint32_t s = 0x51ed27u ^ (blockIdx.x * blockDim.x + threadIdx.x) * 0x85ebca6bu;
  xs32(s);
  for (int i = 0; i < iters; ++i) atomicAdd(sh + below(xs32(s), nbins), 1.0);
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = sh[0];
}

template <typename T>
__global__ void red_shared_t(double* out, int iters, uint32_t nbins) {
  extern __shared__ double shd[];
  T* sh = reinterpret_cast<T*>(shd);
  for (uint32_t i = threadIdx.x; i < nbins; i += blockDim.x) sh[i] = T(0);
  __syncthreads();
  uint32_t s = 0x51ed27u ^ (blockIdx.x * blockDim.x + threadIdx.x) * 0x85ebca6bu;
  xs32(s);
  for (int i = 0; i < iters; ++i) atomicAdd(sh + below(xs32(s), nbins), T(1));
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = (double)sh[0];
}

// nbins per CTA; every update goes to a random CTA of the cluster (7/8 of them remote)
__global__ void red_dsmem(double* out, int iters, uint32_t nbins) {
  extern __shared__ double sh[];
  cg::cluster_group cl = cg::this_cluster();
  for (uint32_t i = threadIdx.x; i < nbins; i += blockDim.x) sh[i] = 0.0;
  cl.sync();
  const uint32_t nr = cl.num_blocks();
  uint32_t s = 0x2545f491u ^ (blockIdx.x * blockDim.x + threadIdx.x) * 0x9e3779b9u;
  xs32(s);
  for (int i = 0; i < iters; ++i) {
    const uint32_t r = xs32(s);
    double* dst = cl.map_shared_rank(sh, below(r, nr));
    atomicAdd(dst + below(xs32(s), nbins), 1.0);
  }
  cl.sync();
  if (threadIdx.x == 0) out[blockIdx.x] = sh[0];
}

__global__ void fp64_alu(double* out, int iters) {
  double a[8];
  const double x = 1.0 + 1e-9 * threadIdx.x, y = 1.0 - 1e-9 * blockIdx.x;
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = x + j;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) a[j] = __dadd_rn(__dmul_rn(a[j], y), x);  // 2 ops, no FMA
  }
  double t = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) t += a[j];
  if (t == 1234.5) out[0] = t;
}

// NVML sampler of the SM clock and the clock-event reasons while a case runs.
struct ClockLog {
  nvmlDevice_t dev{};
  bool ok = false;
  std::vector<unsigned> mhz;
  unsigned long long reasons = 0;
  ClockLog() { ok = nvmlInit_v2() == NVML_SUCCESS && nvmlDeviceGetHandleByIndex_v2(0, &dev) == NVML_SUCCESS; }
  template <class F>
  void run(F f) {
    mhz.clear();
    reasons = 0;
    std::atomic<bool> stop{false};
    std::thread th([&] {
      while (!stop.load() && ok) {
        unsigned c = 0;
        unsigned long long r = 0;
        if (nvmlDeviceGetClockInfo(dev, NVML_CLOCK_SM, &c) == NVML_SUCCESS) mhz.push_back(c);
        if (nvmlDeviceGetCurrentClocksEventReasons(dev, &r) == NVML_SUCCESS) reasons |= r;
        std::this_thread::sleep_for(std::chrono::microseconds(500));
      }
    });
    f();
    stop = true;
    th.join();
  }
  // JSON fragment: "clock": {"sm_mhz_median": M, "sm_mhz_min": m, "samples": n, "reasons": "0x.."}
  void print(const char* key = "clock") {
    std::vector<unsigned> v = mhz;
    std::sort(v.begin(), v.end());
    // idle (0x1) is expected between the timed repetitions
    printf("\"%s\": {\"sm_mhz_median\": %u, \"sm_mhz_min\": %u, \"samples\": %zu, \"reasons\": \"0x%llx\"}",
           key, v.empty() ? 0 : v[v.size() / 2], v.empty() ? 0 : v[0], v.size(), reasons & ~1ull);
  }
};

struct Timer {
  cudaEvent_t a, b;
  ClockLog* log = nullptr;
  Timer() {
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
  }
  // best of `reps` timings, each `inner` back-to-back launches (long enough for clock samples)
  template <class F>
  float best(F f, int reps = 5, int inner = 20) {
    f();
    CK(cudaDeviceSynchronize());
    float best = 1e30f;
    auto body = [&] {
      for (int r = 0; r < reps; ++r) {
        CK(cudaEventRecord(a));
        for (int i = 0; i < inner; ++i) f();
        CK(cudaEventRecord(b));
        CK(cudaEventSynchronize(b));
        float ms;
        CK(cudaEventElapsedTime(&ms, a, b));
        if (ms / inner < best) best = ms / inner;
      }
    };
    if (log) log->run(body);
    else body();
    return best;
  }
};

int main() {
  int dev = 0, nsm = 0, clk = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev));
  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, dev));
  Timer t;
  ClockLog clog;
  t.log = &clog;
  const int threads = 512, blocks = nsm * 4;
  const double nthr = (double)threads * blocks;
  printf("{\n \"gpu\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, \"clock_khz_attr\": %d,\n", prop.name, nsm,
         prop.l2CacheSize, clk);
  const size_t big = (size_t)1 << 30;
  void* h = nullptr;
  CK(cudaMalloc(&h, big));
  CK(cudaMemset(h, 0, big));
  double* out = nullptr;
  CK(cudaMalloc(&out, 1 << 20));
  struct Case {
    const char* name;
    uint32_t n0, n1, n2;
  } grids[] = {{"corelli_600x600", 600, 600, 1}, {"topaz_200^3", 200, 200, 200}, {"stress_500^3", 500, 500, 500}};
  const int iters = 256;
  printf(" \"atomics_per_s\": {\n");
  for (int gi = 0; gi < 3; ++gi) {
    const Case& c = grids[gi];
    const uint32_t nb = c.n0 * c.n1 * c.n2;
    double* hd = static_cast<double*>(h);
    float* hf = static_cast<float*>(h);
    const float ms_r = t.best([&] { red_random<double><<<blocks, threads>>>(hd, nb, iters); });
    ClockLog cr = clog;
    const float ms_w = t.best([&] { red_walk<<<blocks, threads>>>(hd, c.n0, c.n1, c.n2, iters, 64); });
    const float ms_f = t.best([&] { red_random<float><<<blocks, threads>>>(hf, nb, iters); });
    CK(cudaGetLastError());
    const double n = nthr * iters;
    printf("  \"%s\": {\"bins\": %u, \"f64_bytes\": %zu, \"red_f64_random\": %.4g, \"red_f64_walk\": %.4g, "
           "\"red_f32_random\": %.4g, ",
           c.name, nb, (size_t)nb * 8, n / (ms_r * 1e-3), (nthr * (iters / 64 * 64)) / (ms_w * 1e-3),
           n / (ms_f * 1e-3));
    cr.print();
    printf("}%s\n", gi < 2 ? "," : "");
  }
  printf(" },\n");
  {
    const int sb = 4096;  // 32 KB fp64 sub-histogram per CTA
    CK(cudaFuncSetAttribute(red_shared, cudaFuncAttributeMaxDynamicSharedMemorySize, sb * 8));
    const int it = 4096;
    const float ms = t.best([&] { red_shared<<<blocks, threads, sb * 8>>>(out, it, sb); });
    CK(cudaGetLastError());
    printf(" \"red_shared_f64_per_s\": %.4g, ", nthr * it / (ms * 1e-3));
    clog.print("red_shared_f64_clock");
    printf(",\n");
    CK(cudaFuncSetAttribute(red_shared_t<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, sb * 8));
    const float msf = t.best([&] { red_shared_t<float><<<blocks, threads, sb * 8>>>(out, it, sb); });
    CK(cudaGetLastError());
    printf(" \"red_shared_f32_per_s\": %.4g,\n", nthr * it / (msf * 1e-3));
    // cluster of 8 CTAs, 8 x 4096 fp64 bins distributed over their shared memory
    CK(cudaFuncSetAttribute(red_dsmem, cudaFuncAttributeMaxDynamicSharedMemorySize, sb * 8));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(nsm / 8 * 8 * 2);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = sb * 8;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 8;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    const float msd = t.best([&] { CK(cudaLaunchKernelEx(&cfg, red_dsmem, out, it, (uint32_t)sb)); });
    CK(cudaGetLastError());
    printf(" \"red_dsmem_f64_per_s\": %.4g,\n", (double)cfg.gridDim.x * threads * it / (msd * 1e-3));
  }
  {
    const int it = 4096;
    const float ms = t.best([&] { fp64_alu<<<blocks, threads>>>(out, it); });
    CK(cudaGetLastError());
    const double ops = nthr * it * 8 * 2;
    printf(" \"fp64_alu_ops_per_s\": %.4g,\n \"fp64_lanes_per_sm_at_attr_clock\": %.3g,\n ", ops / (ms * 1e-3),
           ops / (ms * 1e-3) / nsm / (clk * 1e3));
    clog.print("fp64_alu_clock");
    printf("\n}\n");
  }
  CK(cudaFree(h));
  CK(cudaFree(out));
  return 0;
}
