// Microbenchmark: random gather of 637k 400-byte rows out of a 2.45M-row
// table (the products workload) -- does the table's row STRIDE change the
// DRAM efficiency?  stride 100 (400 B, rows straddle 64 B lines), 112 (448 B,
// 64-B aligned rows, today's layout), 128 (512 B: a row never crosses a 512-B
// boundary).  Also reads-only.  Flat float4 index space, 4 loads in flight.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a stride_bench.cu -o stride_bench
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <numeric>
#include <vector>
#include <cuda_runtime.h>

template <bool WRITE>
__global__ void __launch_bounds__(256) k_flat(const int *rd, int n, const float4 *f, int dim4, int stride4,
                                              float4 *out) {
  const uint32_t total = (uint32_t)n * dim4, nth = gridDim.x * blockDim.x;
  float acc = 0.f;
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += nth * 4) {
    float4 v[4];
    int g[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t e = e0 + u * nth;
      g[u] = e < total ? __ldg(rd + e / dim4) : 0;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t e = e0 + u * nth;
      if (e < total) v[u] = __ldg(f + (size_t)g[u] * stride4 + (e - (e / dim4) * dim4));
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t e = e0 + u * nth;
      if (e < total) {
        if (WRITE) out[e] = v[u];
        else acc += v[u].x;
      }
    }
  }
  if (!WRITE && acc == 12345.f) out[0] = make_float4(acc, 0, 0, 0);
}

__global__ void k_flush(float4 *b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = make_float4(1, 1, 1, 1);
}

int main() {
  const int N = 2449029, n = 636863, dim = 100, dim4 = dim / 4;
  std::vector<int> all(N), rnd(n);
  std::iota(all.begin(), all.end(), 0);
  uint64_t x = 88172645463325252ull;
  for (int i = 0; i < n; ++i) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    int j = i + (int)(x % (uint64_t)(N - i));
    std::swap(all[i], all[j]);
    rnd[i] = all[i];
  }
  int *d_rnd;
  cudaMalloc(&d_rnd, sizeof(int) * n);
  cudaMemcpy(d_rnd, rnd.data(), sizeof(int) * n, cudaMemcpyHostToDevice);
  float4 *f, *out, *fl;
  const size_t fbytes = (size_t)N * 128 * 4;
  cudaMalloc(&f, fbytes + 4096);
  cudaMemset(f, 0, fbytes + 4096);
  cudaMalloc(&out, (size_t)n * dim * 4);
  const size_t flushn = (size_t)256 << 20;  // 4 GB / 16
  cudaMalloc(&fl, flushn * 16);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int strides[] = {100, 104, 112, 128};
  for (int rep = 0; rep < 2; ++rep)
    for (int w = 1; w >= 0; --w)
      for (int s : strides) {
        float best = 1e9f;
        for (int it = 0; it < 5; ++it) {
          k_flush<<<sms * 4, 256>>>(fl, flushn / 16);  // 256 MB: evict L2
          cudaEventRecord(a);
          if (w) k_flat<true><<<sms * 8, 256>>>(d_rnd, n, f, dim4, s / 4, out);
          else k_flat<false><<<sms * 8, 256>>>(d_rnd, n, f, dim4, s / 4, out);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          best = std::min(best, ms);
        }
        const double bytes = (double)n * dim * 4 * (w ? 2 : 1);
        printf("stride %3d floats (%4d B) %s: %7.1f us  %6.0f GB/s\n", s, s * 4, w ? "read+write" : "read only ",
               best * 1e3, bytes / (best * 1e-3) / 1e9);
      }
  return 0;
}
