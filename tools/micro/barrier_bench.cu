// Microbenchmarks for design decisions of the persistent CSP kernel:
//  (1) grid barrier variants at the persistent grid shape,
//  (2) random 4-byte DRAM reads under cudaLimitMaxL2FetchGranularity 32/64/128,
//  (3) random 400-byte row gathers under the same limits.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_ppopp_caiz0zszck23_b200/csrc/dsp_kernels.cuh"
using namespace dsp;

__device__ __forceinline__ void barrier_v2(WsHeader *hdr, int sleep) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t gen = ld_acquire_gpu_u32(&hdr->bar_gen);
    if (atom_add_acqrel_gpu(&hdr->bar_count, 1u) == gridDim.x - 1) {
      hdr->bar_count = 0u;
      st_release_gpu_u32(&hdr->bar_gen, gen + 1);
    } else {
      while (ld_acquire_gpu_u32(&hdr->bar_gen) == gen)
        if (sleep) __nanosleep(sleep);
    }
  }
  __syncthreads();
}

__device__ __forceinline__ void red_add_release_gpu(uint32_t *p, uint32_t v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// monotonic arrival counter: no return-value round trip, one poll loop
__device__ __forceinline__ void barrier_v3(WsHeader *hdr, uint32_t &epoch) {
  __syncthreads();
  epoch += gridDim.x;
  if (threadIdx.x == 0) {
    red_add_release_gpu(&hdr->bar_count, 1u);
    while (ld_acquire_gpu_u32(&hdr->bar_count) < epoch) {
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(NT, 4) k_bar(WsHeader *hdr, int n, int variant) {
  uint32_t epoch = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) hdr->t[0] = globaltimer_ns();
  for (int i = 0; i < n; ++i) {
    if (variant == 0) grid_barrier(hdr);
    else if (variant == 3) barrier_v3(hdr, epoch);
    else barrier_v2(hdr, variant == 1 ? 0 : 32);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) hdr->t[23] = globaltimer_ns();
}

__device__ __forceinline__ uint32_t mix(uint32_t x) { return hash32(x * 0x9E3779B9u + 7u); }

__global__ void k_rand4(const int *a, size_t n, int iters, int *out) {
  int acc = 0;
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < iters; ++i) acc += __ldg(a + (mix(tid * 131u + i) % n));
  out[tid] = acc;
}

__global__ void k_rows(const float4 *f, int nrows, int row4, int stride4, int rows_per_thread_block, float4 *o) {
  // each warp gathers random rows; lanes stride the row
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  for (int r = 0; r < rows_per_thread_block; ++r) {
    const uint32_t g = mix(warp * 977u + r) % nrows;
    for (int c = lane; c < row4; c += 32) o[(size_t)(warp * rows_per_thread_block + r) * row4 + c] = __ldg(f + (size_t)g * stride4 + c);
  }
}

int main() {
  WsHeader *hdr;
  cudaMalloc(&hdr, sizeof(WsHeader));
  for (int variant = 0; variant < 4; ++variant)
    for (int nb : {148, 592}) {
      int n = 200;
      cudaMemset(hdr, 0, sizeof(WsHeader));
      void *args[] = {&hdr, &n, &variant};
      cudaLaunchCooperativeKernel((void *)k_bar, dim3(nb), dim3(NT), args, 0, 0);
      cudaDeviceSynchronize();
      WsHeader h;
      cudaMemcpy(&h, hdr, sizeof(h), cudaMemcpyDeviceToHost);
      printf("barrier v%d blocks %d: %.2f us\n", variant, nb, (h.t[23] - h.t[0]) / 1e3 / n);
    }
  // short kernels with host sync in between (how the sampler runs)
  for (int variant : {0, 3}) {
    double acc = 0;
    int reps = 20, n = 10, nb = 592;
    for (int r = 0; r < reps; ++r) {
      cudaMemset(hdr, 0, sizeof(WsHeader));
      void *args[] = {&hdr, &n, &variant};
      cudaLaunchCooperativeKernel((void *)k_bar, dim3(nb), dim3(NT), args, 0, 0);
      cudaDeviceSynchronize();
      WsHeader h;
      cudaMemcpy(&h, hdr, sizeof(h), cudaMemcpyDeviceToHost);
      acc += (h.t[23] - h.t[0]) / 1e3 / n;
    }
    printf("short kernels (10 barriers, host sync between) v%d: %.2f us per barrier\n", variant, acc / reps);
  }
  size_t n = (size_t)256 << 20;  // 1 GiB of int
  int *a, *out;
  cudaMalloc(&a, n * 4);
  cudaMemset(a, 1, n * 4);
  cudaMalloc(&out, 64 << 20);
  float4 *fo;
  cudaMalloc(&fo, (size_t)1 << 30);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (size_t gran : {32, 64, 128}) {
    cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, gran);
    size_t got = 0;
    cudaDeviceGetLimit(&got, cudaLimitMaxL2FetchGranularity);
    const int iters = 64;
    k_rand4<<<1184, 256>>>(a, n, iters, out);
    cudaEventRecord(e0);
    k_rand4<<<1184, 256>>>(a, n, iters, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double loads = 1184.0 * 256 * iters;
    printf("L2 fetch granularity %zu (got %zu): random 4B loads %.1f G/s\n", gran, got, loads / ms / 1e6);
    for (int stride4 : {25, 28, 32}) {
      const int row4 = 25, nrows = (int)(((size_t)1 << 30) / (stride4 * 16)) - 1, rpt = 16;
      k_rows<<<1184, 256>>>(reinterpret_cast<float4 *>(a), nrows, row4, stride4, rpt, fo);
      cudaEventRecord(e0);
      k_rows<<<1184, 256>>>(reinterpret_cast<float4 *>(a), nrows, row4, stride4, rpt, fo);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
      const double bytes = 1184.0 * 8 * rpt * row4 * 16 * 2;
      printf("   400 B rows, stride %d B: %.0f GB/s (read+write)\n", stride4 * 16, bytes / ms / 1e6);
    }
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
