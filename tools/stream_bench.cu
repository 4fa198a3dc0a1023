// Streaming-read microbenchmark (tools only): what event-stream rate can a BinMD-like kernel reach
// on this B200?  Reads n float4 (16 B) with several grid shapes / in-flight depths and a trivial
// per-element test (so the loads are not dead), CUDA-event timed, L2 flushed between runs.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/stream_bench tools/stream_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int D, int MINB>
__global__ void __launch_bounds__(256, MINB) rd(const float4* __restrict__ e, long long n, int* out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  long long base = ((long long)(threadIdx.x >> 5) * gridDim.x + blockIdx.x) * 32 + (threadIdx.x & 31);
  float4 v[D];
#pragma unroll
  for (int u = 0; u < D; ++u) v[u] = base + u * stride < n ? __ldcs(e + base + u * stride) : make_float4(0, 0, 0, 0);
  int cnt = 0;
  for (;;) {
#pragma unroll
    for (int u = 0; u < D; ++u) {
      if (base >= n) goto done;
      cnt += fabsf(v[u].y * 0.3f + v[u].z * 0.2f - v[u].w) < 0.01f;
      const long long nx = base + D * stride;
      v[u] = nx < n ? __ldcs(e + nx) : make_float4(0, 0, 0, 0);
      base += stride;
    }
  }
done:
  if (cnt == 123456789) out[0] = cnt;
}

template <int D, int MINB>
void run(const float4* e, long long n, int* out, char* flush, int sms) {
  int per = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, rd<D, MINB>, 256, 0);
  int grid = sms * per;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e9, tot = 0;
  for (int it = 0; it < 13; ++it) {
    cudaMemsetAsync(flush, it, 256 << 20);
    cudaEventRecord(a);
    rd<D, MINB><<<grid, 256>>>(e, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (it >= 3) {
      tot += ms;
      if (ms < best) best = ms;
    }
  }
  printf("D=%d minb=%d grid=%d  mean %.2f us  best %.2f us  %.0f GB/s\n", D, MINB, grid, tot / 10 * 1e3, best * 1e3,
         16.0 * n / (tot / 10) / 1e6);
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (long long n : {10000000LL, 100000000LL}) {
    float4* e;
    int* out;
    char* flush;
    cudaMalloc(&e, 16 * n);
    cudaMemset(e, 0, 16 * n);
    cudaMalloc(&out, 4);
    cudaMalloc(&flush, 256 << 20);
    printf("n = %lld float4 (%.0f MB)\n", n, 16.0 * n / 1e6);
    run<1, 4>(e, n, out, flush, sms);
    run<2, 4>(e, n, out, flush, sms);
    run<3, 4>(e, n, out, flush, sms);
    run<4, 4>(e, n, out, flush, sms);
    run<6, 4>(e, n, out, flush, sms);
    run<3, 8>(e, n, out, flush, sms);
    run<4, 8>(e, n, out, flush, sms);
    run<2, 8>(e, n, out, flush, sms);
    run<8, 2>(e, n, out, flush, sms);
    cudaFree(e);
    cudaFree(out);
    cudaFree(flush);
  }
  return 0;
}
