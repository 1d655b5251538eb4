// Dependent-chain latency (cycles per op) of warp collectives on one warp,
// and throughput with 32 warps per SM: REDUX.SUM, SHFL, VOTE+POPC, IMAD.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int OP>
__global__ void k_chain(uint32_t *out, long long *cyc, int n) {
  uint32_t x = threadIdx.x * 7 + 1;
  __syncwarp();
  const long long t0 = clock64();
  for (int i = 0; i < n; ++i) {
    if (OP == 0) x = __reduce_add_sync(0xffffffffu, x) + threadIdx.x;
    if (OP == 1) x = __shfl_sync(0xffffffffu, x, (x + 3) & 31) + 1;
    if (OP == 2) x = __popc(__ballot_sync(0xffffffffu, (x & 1) != 0)) + threadIdx.x;
    if (OP == 3) x = x * 0x9E3779B1u + 7u;
    if (OP == 4) x = __shfl_up_sync(0xffffffffu, x, 1) + x;
    if (OP == 5) x = __reduce_max_sync(0xffffffffu, x) + threadIdx.x;
  }
  const long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}

int main() {
  uint32_t *out; long long *cyc, h;
  cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 8);
  const char *names[] = {"REDUX.SUM", "SHFL.IDX", "VOTE+POPC", "IMAD", "SHFL.UP+IADD", "REDUX.MAX"};
  const int n = 4096;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int op = 0; op < 6; ++op) {
    for (int warps : {1, 8, 32}) {
      auto launch = [&]() {
        switch (op) {
          case 0: k_chain<0><<<148, 32 * warps>>>(out, cyc, n); break;
          case 1: k_chain<1><<<148, 32 * warps>>>(out, cyc, n); break;
          case 2: k_chain<2><<<148, 32 * warps>>>(out, cyc, n); break;
          case 3: k_chain<3><<<148, 32 * warps>>>(out, cyc, n); break;
          case 4: k_chain<4><<<148, 32 * warps>>>(out, cyc, n); break;
          case 5: k_chain<5><<<148, 32 * warps>>>(out, cyc, n); break;
        }
      };
      launch();
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
      printf("%-14s warps/SM %2d: %6.1f cycles per dependent op (warp 0), %.2f ns per op per SM at %d warps\n", names[op], warps,
             (double)h / n, ms * 1e6 / n / warps, warps);
    }
  }
  return 0;
}
