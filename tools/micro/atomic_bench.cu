// Throughput of the relabel-table atomics at the layer-2 shape of the
// products workload: ~900k random operations from 151k threads (6 each)
// into a 16 MB (2M x 8 B) table / a 2.45M-entry direct array.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_ppopp_caiz0zszck23_b200/csrc/dsp_device.cuh"
using namespace dsp;

__global__ void k_cas(unsigned long long *t, uint32_t mask, int per, unsigned long long *sink) {
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0, prev[8];
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < per) {
      uint32_t key = hash32(tid * 8 + j) % 2449029u;
      prev[j] = atomicCAS(&t[hash32(key) & mask], ~0ull, ((unsigned long long)key << 32) | j);
    }
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < per) acc += prev[j];
  if (acc == 12345) sink[0] = acc;
}
__global__ void k_redmax(unsigned long long *t, int per) {
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < per) {
      uint32_t key = hash32(tid * 8 + j) % 2449029u;
      atomicMax(&t[key], ((unsigned long long)7 << 32) | (0xffffffffu - (tid + j)));
    }
}
__global__ void k_redmin32(unsigned *t, int per) {
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < per) {
      uint32_t key = hash32(tid * 8 + j) % 2449029u;
      atomicMin(&t[key], tid + j);
    }
}
__global__ void k_ld(const unsigned long long *t, int per, unsigned long long *sink) {
  uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j)
    if (j < per) acc += __ldcg(&t[hash32(tid * 8 + j) % 2449029u]);
  if (acc == 12345) sink[0] = acc;
}

int main() {
  unsigned long long *t, *sink;
  cudaMalloc(&t, 32 << 20);
  cudaMalloc(&sink, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int blocks = 148, threads = 1024, per = 6;
  const double ops = (double)blocks * threads * per;
  float ms;
  for (int rep = 0; rep < 3; ++rep) {
    cudaMemset(t, 0xff, 16 << 20);
    cudaEventRecord(e0);
    k_cas<<<blocks, threads>>>(t, (2u << 20) - 1, per, sink);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("64-bit CAS (with return) into 16 MB hash table: %.1f us, %.0f G ops/s\n", ms * 1e3, ops / ms / 1e6);
    cudaMemset(t, 0, 20 << 20);
    cudaEventRecord(e0);
    k_redmax<<<blocks, threads>>>(t, per);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("64-bit atomicMax (no return use) into 20 MB direct array: %.1f us, %.0f G ops/s\n", ms * 1e3, ops / ms / 1e6);
    cudaEventRecord(e0);
    k_redmin32<<<blocks, threads>>>((unsigned *)t, per);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("32-bit atomicMin (no return use) into 10 MB direct array: %.1f us, %.0f G ops/s\n", ms * 1e3, ops / ms / 1e6);
    cudaEventRecord(e0);
    k_ld<<<blocks, threads>>>(t, per, sink);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("64-bit random ldcg from 20 MB: %.1f us, %.0f G ops/s\n", ms * 1e3, ops / ms / 1e6);
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
