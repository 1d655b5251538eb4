// Microbenchmark: random reads from a 512 MB array (the products adjacency
// size), by request size.  Question: is the random-read ceiling per request
// (so reading a whole short adjacency row costs what one 4-byte pick costs)
// or per byte?
//   S = 4 / 8 / 16 B: one thread per request, U independent requests in flight
//   S = 32..512 B:    S/16 lanes of a warp read one request with 16-B vectors
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a random_read_bench.cu -o random_read_bench
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x85EBCA6Bu; x ^= x >> 13; x *= 0xC2B2AE35u; x ^= x >> 16;
  return x;
}

// thread-per-request, S bytes (4, 8 or 16)
template <int S, int U>
__global__ void __launch_bounds__(256) k_thread(const char *a, uint64_t nbytes, int reqs_per_thread, uint32_t *sink) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t acc = 0;
  const uint64_t nslots = nbytes / S;
  for (int it = 0; it < reqs_per_thread; it += U) {
    uint32_t v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t slot = ((uint64_t)hash32(tid * 977u + (it + u) * 7919u) * 2654435761ull) % nslots;
      const char *p = a + slot * S;
      if (S == 4) v[u] = __ldg((const uint32_t *)p);
      else if (S == 8) { uint2 x = __ldg((const uint2 *)p); v[u] = x.x ^ x.y; }
      else { uint4 x = __ldg((const uint4 *)p); v[u] = x.x ^ x.w; }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  if (acc == 0x12345678u) sink[0] = acc;
}

// warp-cooperative: each request = S bytes read by S/16 lanes (16 B each); a
// warp handles 32/(S/16) requests per instruction, U instructions in flight
template <int S, int U>
__global__ void __launch_bounds__(256) k_warp(const char *a, uint64_t nbytes, int reqs_per_thread, uint32_t *sink) {
  constexpr int LPR = S / 16;               // lanes per request
  constexpr int RPW = 32 / LPR;             // requests per warp instruction
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const uint32_t grp = tid / LPR;           // request group id
  uint32_t acc = 0;
  const uint64_t nslots = nbytes / S;
  // reqs_per_thread requests per *request group*, so total requests = threads / LPR * reqs
  for (int it = 0; it < reqs_per_thread; it += U) {
    uint32_t v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t slot = ((uint64_t)hash32(grp * 977u + (it + u) * 7919u) * 2654435761ull) % nslots;
      const uint4 x = __ldg((const uint4 *)(a + slot * S) + (lane % LPR));
      v[u] = x.x ^ x.w;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  (void)RPW;
  if (acc == 0x12345678u) sink[0] = acc;
}

int main() {
  const uint64_t nbytes = 512ull << 20;
  char *a;
  uint32_t *sink;
  cudaMalloc(&a, nbytes);
  cudaMemset(a, 1, nbytes);
  cudaMalloc(&sink, 64);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int grid = 148 * 8, block = 256, reqs = 64;
  auto run = [&](auto kern, const char *name, double requests, double bytes_per_req) {
    float best = 1e9, ms;
    for (int rep = 0; rep < 4; ++rep) {
      cudaEventRecord(e0);
      kern<<<grid, block>>>(a, nbytes, reqs, sink);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    printf("%-34s %8.1f us  %6.1f G req/s  %6.0f GB/s  %s\n", name, best * 1e3, requests / best / 1e6,
           requests * bytes_per_req / best / 1e6, cudaGetErrorString(cudaGetLastError()));
  };
  const double threads = (double)grid * block;
  run(k_thread<4, 4>, "4 B, thread, U=4", threads * reqs, 4);
  run(k_thread<4, 8>, "4 B, thread, U=8", threads * reqs, 4);
  run(k_thread<8, 8>, "8 B, thread, U=8", threads * reqs, 8);
  run(k_thread<16, 8>, "16 B, thread, U=8", threads * reqs, 16);
  run(k_warp<32, 8>, "32 B, 2 lanes, U=8", threads / 2 * reqs, 32);
  run(k_warp<64, 8>, "64 B, 4 lanes, U=8", threads / 4 * reqs, 64);
  run(k_warp<128, 8>, "128 B, 8 lanes, U=8", threads / 8 * reqs, 128);
  run(k_warp<256, 8>, "256 B, 16 lanes, U=8", threads / 16 * reqs, 256);
  run(k_warp<512, 8>, "512 B, 32 lanes, U=8", threads / 32 * reqs, 512);
  return 0;
}
