// Microbenchmark: does splitting 400-byte feature rows into a 128-B-aligned
// 384-byte head (3 full L2 lines) and a 16-byte tail kept in a separate dense
// array cut the DRAM bytes of the random-row gather?  A 400-byte row at any
// alignment touches 4 lines (512 B of DRAM reads); the split head touches 3,
// and the 39 MB tail array can stay in L2 (evict_last) while the heads stream
// (evict_first).  Gather = TMA bulk copies into a shared-memory ring (as
// k_gather_tma), one bulk store per 32-row chunk.  Several batches of 637k
// ids (products, uniform or degree-like skewed) per layout; L2 flushed once
// before each layout, not between batches (steady state across steps).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cmath>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t phase) {
  uint32_t ok;
  asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
               : "=r"(ok) : "r"(smem_addr(bar)), "r"(phase) : "memory");
  return ok != 0;
}
__device__ __forceinline__ unsigned long long pol_first() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long pol_last() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long pol_normal() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar, unsigned long long pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               ::"r"(smem_addr(dst)), "l"(src), "r"(bytes), "r"(smem_addr(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes, unsigned long long pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
               "r"(smem_addr(src)), "r"(bytes), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

struct Layout {
  const char *head; int head_bytes; int head_stride;  // head part of row g at head + g * head_stride
  const char *tail; int tail_bytes; int tail_stride;
  int tail_policy;  // 0 evict_first, 1 evict_last, 2 normal
  int head_policy;
};

constexpr int R = 32, S = 2;
__global__ void k_gather(const int *ids, int n, Layout L, char *out, int nchunks) {
  extern __shared__ __align__(128) char smem[];
  const int row_bytes = L.head_bytes + L.tail_bytes;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;
  const int slot_bytes = (R * row_bytes + 127) / 128 * 128;
  char *ring = smem + (size_t)warp * S * slot_bytes;
  __shared__ __align__(8) uint64_t bars[32][S];
  if (lane == 0)
    for (int s = 0; s < S; ++s) mbar_init(&bars[warp][s], 1);
  __syncwarp();
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const unsigned long long pf = pol_first();
  const unsigned long long ph = L.head_policy == 1 ? pol_last() : L.head_policy == 2 ? pol_normal() : pf;
  const unsigned long long pt = L.tail_policy == 1 ? pol_last() : L.tail_policy == 2 ? pol_normal() : pf;
  const int gw = blockIdx.x * W + warp, nw = gridDim.x * W;
  int issued = 0, done = 0;
  const int my_chunks = (nchunks - gw + nw - 1) / nw;
  while (done < my_chunks) {
    while (issued < my_chunks && issued - done < S) {
      const int s = issued % S;
      const int c = gw + issued * nw;
      const int r0 = c * R;
      const int rows = min(R, n - r0);
      if (issued >= S) {
        if (lane == 0) bulk_wait_read<S - 1>();
        __syncwarp();
      }
      if (lane == 0) mbar_expect_tx(&bars[warp][s], rows * row_bytes);
      __syncwarp();
      if (lane < rows) {
        const int g = __ldg(ids + r0 + lane);
        char *dst = ring + (size_t)s * slot_bytes + lane * row_bytes;
        if (L.head_bytes) bulk_g2s(dst, L.head + (size_t)g * L.head_stride, L.head_bytes, &bars[warp][s], ph);
        if (L.tail_bytes) bulk_g2s(dst + L.head_bytes, L.tail + (size_t)g * L.tail_stride, L.tail_bytes, &bars[warp][s], pt);
      }
      ++issued;
    }
    const int s = done % S;
    while (!mbar_try_wait(&bars[warp][s], (done / S) & 1)) {
    }
    const int c = gw + done * nw;
    const int r0 = c * R;
    const int rows = min(R, n - r0);
    if (lane == 0) {
      bulk_s2g(out + (size_t)r0 * row_bytes, ring + (size_t)s * slot_bytes, rows * row_bytes, pf);
      bulk_commit();
    }
    __syncwarp();
    ++done;
  }
  if (lane == 0) bulk_wait_all();
}

int main() {
  const int N = 2449029, n = 636863, dim = 100, B = 8;
  std::vector<int> h((size_t)n * B);
  uint64_t x = 88172645463325252ull;
  auto rnd = [&]() { x ^= x << 13; x ^= x >> 7; x ^= x << 17; return x; };
  char *flush;
  cudaMalloc(&flush, 512 << 20);
  char *big;    // 448-stride table, also reused for 400-stride and the head array
  cudaMalloc(&big, (size_t)N * 448);
  cudaMemset(big, 1, (size_t)N * 448);
  char *tail;
  cudaMalloc(&tail, (size_t)N * 16);
  cudaMemset(tail, 2, (size_t)N * 16);
  char *out;
  cudaMalloc(&out, (size_t)n * dim * 4);
  int *ids;
  cudaMalloc(&ids, (size_t)n * B * 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaFuncSetAttribute(k_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, 6 * S * 12800);
  for (int skew = 0; skew < 2; ++skew) {
    for (size_t i = 0; i < h.size(); ++i) {
      double u = (rnd() >> 11) * (1.0 / 9007199254740992.0);
      // skew 1: P(id) ~ a power law over a random permutation (popular rows reused across batches)
      uint64_t v = skew ? (uint64_t)(N * pow(u, 2.0)) : (uint64_t)(u * N);
      h[i] = (int)((v * 2654435761ull) % N);
    }
    cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    struct Case { const char *name; Layout L; };
    Case cases[] = {
        {"400 B rows, 448 stride (current)", {big, 400, 448, nullptr, 0, 0, 0, 0}},
        {"400 B rows, 400 stride (packed)", {big, 400, 400, nullptr, 0, 0, 0, 0}},
        {"split 384 + 16 tail, tail evict_first", {big, 384, 384, tail, 16, 16, 0, 0}},
        {"split 384 + 16 tail, tail evict_last", {big, 384, 384, tail, 16, 16, 1, 0}},
        {"split 384 + 16 tail, tail normal", {big, 384, 384, tail, 16, 16, 2, 0}},
        {"384 B head only (floor)", {big, 384, 384, nullptr, 0, 0, 0, 0}},
        {"400 B rows, 448 stride, normal policy", {big, 400, 448, nullptr, 0, 0, 0, 2}},
    };
    for (auto &cs : cases) {
      const int row_bytes = cs.L.head_bytes + cs.L.tail_bytes;
      const int nchunks = (n + R - 1) / R;
      const int smem = 6 * S * ((R * row_bytes + 127) / 128 * 128);
      cudaMemset(flush, 3, 512 << 20);
      float tot = 0, best = 1e9;
      for (int b = 0; b < B; ++b) {
        cudaEventRecord(e0);
        k_gather<<<148, 6 * 32, smem>>>(ids + (size_t)b * n, n, cs.L, out, nchunks);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (b >= 2) tot += ms;
        best = fminf(best, ms);
      }
      const float mean = tot / (B - 2);
      printf("%s ids %-40s mean %.1f us  best %.1f us  (%.0f GB/s algorithmic read+write)  %s\n", skew ? "skewed " : "uniform",
             cs.name, mean * 1e3, best * 1e3, 2.0 * n * row_bytes / (mean * 1e6), cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
