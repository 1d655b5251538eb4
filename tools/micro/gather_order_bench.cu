// Microbenchmark: does the ORDER of a 637k-row gather (400-byte rows of a
// 2.45M x 448-byte table, the products workload) change its DRAM efficiency?
//   out[wr[r]] = f[rd[r]]  for r in [0, n)
// (1) random reads, sequential writes (what the loader does today)
// (2) sorted reads, sequential writes (upper bound of read locality)
// (3) sorted reads, random writes  (a gather that walks the relabel map)
// (4) reads only / writes only, random / sequential
// (5) plain copy of the same byte count
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a gather_order_bench.cu -o gather_order_bench
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <numeric>
#include <vector>
#include <cuda_runtime.h>

template <bool READ, bool WRITE>
__global__ void __launch_bounds__(256) k_move(const int *rd, const int *wr, int n, const float4 *f, int dim4,
                                              int stride4, float4 *out, float4 *sink) {
  const uint32_t total = (uint32_t)n * dim4, nth = gridDim.x * blockDim.x;
  float4 acc = make_float4(0, 0, 0, 0);
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += nth * 4) {
    float4 v[4];
    uint32_t e[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      e[u] = e0 + u * nth;
      v[u] = make_float4(1, 2, 3, 4);
      if (READ && e[u] < total) {
        uint32_t r = e[u] / dim4, c = e[u] - r * dim4;
        v[u] = __ldg(f + (size_t)__ldg(rd + r) * stride4 + c);
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (e[u] < total) {
        if (WRITE) {
          uint32_t r = e[u] / dim4, c = e[u] - r * dim4;
          out[(size_t)__ldg(wr + r) * dim4 + c] = v[u];
        } else {
          acc.x += v[u].x;
        }
      }
  }
  if (!WRITE && acc.x == 12345.f) sink[0] = acc;
}

// flat float4 index space, U loads in flight per thread
template <int U>
__global__ void __launch_bounds__(256) k_flat(const int *rd, int n, const float4 *f, int dim4, int stride4, float4 *out) {
  const uint32_t total = (uint32_t)n * dim4, nth = gridDim.x * blockDim.x;
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += nth * U) {
    float4 v[U];
    int g[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t e = e0 + u * nth;
      g[u] = e < total ? __ldg(rd + e / dim4) : 0;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t e = e0 + u * nth;
      if (e < total) v[u] = __ldg(f + (size_t)g[u] * stride4 + (e - (e / dim4) * dim4));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t e = e0 + u * nth;
      if (e < total) out[e] = v[u];
    }
  }
}

// warp per group of R rows: lane c < dim4 moves column c of each row; the
// R ids come from one coalesced load; R row loads in flight per lane
template <int R>
__global__ void __launch_bounds__(256) k_warp(const int *rd, int n, const float4 *f, int dim4, int stride4, float4 *out) {
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  for (int r0 = gw * R; r0 < n; r0 += nw * R) {
    const int myid = (lane < R && r0 + lane < n) ? __ldg(rd + r0 + lane) : 0;
    for (int c = lane; c < dim4; c += 32) {
      float4 v[R];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        const int g = __shfl_sync(0xffffffffu, myid, j);
        if (r0 + j < n) v[j] = __ldg(f + (size_t)g * stride4 + c);
      }
#pragma unroll
      for (int j = 0; j < R; ++j)
        if (r0 + j < n) out[(size_t)(r0 + j) * dim4 + c] = v[j];
    }
  }
}

__global__ void k_copy(const float4 *a, float4 *b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

int main() {
  const int N = 2449029, n = 636863, dim = 100, stride = 112;
  std::vector<int> rnd(n), srt(n), seq(n), perm(n);
  // distinct random ids (the sampled node set is a set)
  std::vector<int> all(N);
  std::iota(all.begin(), all.end(), 0);
  uint64_t x = 88172645463325252ull;
  for (int i = 0; i < n; ++i) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    int j = i + (int)(x % (uint64_t)(N - i));
    std::swap(all[i], all[j]);
    rnd[i] = all[i];
  }
  srt = rnd;
  std::sort(srt.begin(), srt.end());
  std::iota(seq.begin(), seq.end(), 0);
  perm = seq;
  for (int i = n - 1; i > 0; --i) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    std::swap(perm[i], perm[(int)(x % (uint64_t)(i + 1))]);
  }
  int *d_rnd, *d_srt, *d_seq, *d_perm;
  for (auto p : {&d_rnd, &d_srt, &d_seq, &d_perm}) cudaMalloc(p, n * 4);
  cudaMemcpy(d_rnd, rnd.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(d_srt, srt.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(d_seq, seq.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(d_perm, perm.data(), n * 4, cudaMemcpyHostToDevice);
  float *f, *out, *sink;
  cudaMalloc(&f, (size_t)N * stride * 4);
  cudaMemset(f, 1, (size_t)N * stride * 4);
  cudaMalloc(&out, (size_t)n * dim * 4);
  cudaMalloc(&sink, 64);
  char *flush;
  cudaMalloc(&flush, 512 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const double row_bytes = (double)n * dim * 4;
  auto time = [&](auto launch, const char *name, double bytes) {
    float best = 1e9, ms;
    for (int rep = 0; rep < 5; ++rep) {
      cudaMemset(flush, rep, 512 << 20);
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
      best = std::min(best, ms);
    }
    printf("%-48s %8.1f us  %6.0f GB/s  %s\n", name, best * 1e3, bytes / best / 1e6, cudaGetErrorString(cudaGetLastError()));
  };
  for (int blocksPerSM : {4, 8}) {
    const int g = 148 * blocksPerSM;
    printf("-- grid %d x 256\n", g);
    time([&] { k_move<true, true><<<g, 256>>>(d_rnd, d_seq, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(1) random read -> sequential write", 2 * row_bytes);
    time([&] { k_move<true, true><<<g, 256>>>(d_srt, d_seq, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(2) sorted read -> sequential write", 2 * row_bytes);
    time([&] { k_move<true, true><<<g, 256>>>(d_srt, d_perm, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(3) sorted read -> random write", 2 * row_bytes);
    time([&] { k_move<true, false><<<g, 256>>>(d_rnd, d_seq, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(4a) random read only", row_bytes);
    time([&] { k_move<true, false><<<g, 256>>>(d_srt, d_seq, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(4b) sorted read only", row_bytes);
    time([&] { k_move<false, true><<<g, 256>>>(d_rnd, d_seq, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(4c) sequential write only", row_bytes);
    time([&] { k_move<false, true><<<g, 256>>>(d_rnd, d_perm, n, (const float4 *)f, 25, 28, (float4 *)out, (float4 *)sink); },
         "(4d) random write only", row_bytes);
  }
  for (int bps : {8, 16}) {
    const int g = 148 * bps;
    printf("-- grid %d x 256, random read -> sequential write\n", g);
    time([&] { k_flat<4><<<g, 256>>>(d_rnd, n, (const float4 *)f, 25, 28, (float4 *)out); }, "flat U=4", 2 * row_bytes);
    time([&] { k_flat<8><<<g, 256>>>(d_rnd, n, (const float4 *)f, 25, 28, (float4 *)out); }, "flat U=8", 2 * row_bytes);
    time([&] { k_warp<4><<<g, 256>>>(d_rnd, n, (const float4 *)f, 25, 28, (float4 *)out); }, "warp R=4", 2 * row_bytes);
    time([&] { k_warp<8><<<g, 256>>>(d_rnd, n, (const float4 *)f, 25, 28, (float4 *)out); }, "warp R=8", 2 * row_bytes);
    time([&] { k_warp<16><<<g, 256>>>(d_rnd, n, (const float4 *)f, 25, 28, (float4 *)out); }, "warp R=16", 2 * row_bytes);
  }
  time([&] { k_copy<<<148 * 8, 256>>>((const float4 *)f, (float4 *)out, (size_t)n * 25); }, "(5) copy of the same bytes",
       2 * row_bytes);
  return 0;
}
