// Microbenchmark: row gather (637k random 400-byte rows of a 2.45M x 448-byte
// table -> contiguous output) with (a) 16-byte register loads from every
// thread, (b) cp.async.bulk (TMA bulk copies) issued by a few warps per SM
// into a shared-memory ring, with one bulk store per chunk of consecutive
// output rows.  Question: can a couple of warps per SM sustain the gather, so
// that the rest of the SM can run the sampling phases concurrently?
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t phase) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok) : "r"(smem_addr(bar)), "r"(phase) : "memory");
  return ok != 0;
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_addr(dst)), "l"(src), "r"(bytes), "r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_addr(src)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__device__ __forceinline__ float4 ld_stream_f4(const float4 *p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
// variants: bit0 = streaming load, bit1 = streaming store, bit2 = ldcg ids
template <int V>
__global__ void __launch_bounds__(256) k_regv(const int *ids, int n, const float4 *f, int dim4, int stride4, float4 *out) {
  const uint32_t total = n * dim4, nth = gridDim.x * blockDim.x;
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += nth * 4) {
    float4 v[4];
    uint32_t e[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      e[u] = e0 + u * nth;
      if (e[u] < total) {
        uint32_t r = e[u] / dim4, c = e[u] - r * dim4;
        const int g = (V & 4) ? __ldcg(ids + r) : __ldg(ids + r);
        const float4 *p = f + (size_t)g * stride4 + c;
        v[u] = (V & 1) ? ld_stream_f4(p) : __ldg(p);
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (e[u] < total) {
        if (V & 2) __stcs(out + e[u], v[u]);
        else out[e[u]] = v[u];
      }
  }
}

// (a) register gather, flat float4 index space, UNROLL 4
__global__ void __launch_bounds__(256) k_reg(const int *ids, int n, const float4 *f, int dim4, int stride4, float4 *out) {
  const uint32_t total = n * dim4, nth = gridDim.x * blockDim.x;
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += nth * 4) {
    float4 v[4];
    uint32_t e[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      e[u] = e0 + u * nth;
      if (e[u] < total) {
        uint32_t r = e[u] / dim4, c = e[u] - r * dim4;
        v[u] = __ldg(f + (size_t)__ldg(ids + r) * stride4 + c);
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (e[u] < total) out[e[u]] = v[u];
  }
}

// (b) TMA bulk gather: W warps per block; each warp owns S ring slots of R rows.
// Lane l < R of the warp issues the bulk load of row l of the chunk.
template <int R, int S>
__global__ void k_tma(const int *ids, int n, const char *f, int row_bytes, int stride_bytes, char *out, int nchunks) {
  extern __shared__ __align__(128) char smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = blockDim.x >> 5;
  const int slot_bytes = R * row_bytes;
  char *ring = smem + (size_t)warp * S * slot_bytes;
  __shared__ __align__(8) uint64_t bars[32][S];
  if (lane == 0)
    for (int s = 0; s < S; ++s) mbar_init(&bars[warp][s], 1);
  __syncwarp();
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int gw = blockIdx.x * W + warp, nw = gridDim.x * W;
  // chunk c of this warp: global chunk gw + it * nw
  int issued = 0, done = 0;
  const int my_chunks = (nchunks - gw + nw - 1) / nw;
  while (done < my_chunks) {
    // issue as many as the ring allows
    while (issued < my_chunks && issued - done < S) {
      const int s = issued % S;
      const int c = gw + issued * nw;
      const int r0 = c * R;
      const int rows = min(R, n - r0);
      // the slot's previous store must have finished reading smem
      if (issued >= S) {
        if (lane == 0) bulk_wait_read<S - 1>();
        __syncwarp();
      }
      if (lane == 0) mbar_expect_tx(&bars[warp][s], rows * row_bytes);
      __syncwarp();
      if (lane < rows) {
        const int g = __ldg(ids + r0 + lane);
        bulk_g2s(ring + (size_t)s * slot_bytes + lane * row_bytes, f + (size_t)g * stride_bytes, row_bytes,
                 &bars[warp][s]);
      }
      ++issued;
    }
    // complete the oldest
    const int s = done % S;
    const uint32_t phase = (done / S) & 1;
    while (!mbar_try_wait(&bars[warp][s], phase)) {
    }
    const int c = gw + done * nw;
    const int r0 = c * R;
    const int rows = min(R, n - r0);
    if (lane == 0) {
      bulk_s2g(out + (size_t)r0 * row_bytes, ring + (size_t)s * slot_bytes, rows * row_bytes);
      bulk_commit();
    }
    __syncwarp();
    ++done;
  }
  if (lane == 0) bulk_wait_all();
}

int main() {
  const int N = 2449029, n = 636863, dim = 100, stride = 112;
  std::vector<int> h(n);
  uint64_t x = 88172645463325252ull;
  for (int i = 0; i < n; ++i) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    h[i] = (int)(x % N);
  }
  int *ids;
  float *f, *out, *ref;
  cudaMalloc(&ids, n * 4);
  cudaMemcpy(ids, h.data(), n * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&f, (size_t)N * stride * 4);
  cudaMemset(f, 1, (size_t)N * stride * 4);
  cudaMalloc(&out, (size_t)n * dim * 4);
  cudaMalloc(&ref, (size_t)n * dim * 4);
  char *flush;
  cudaMalloc(&flush, 256 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const double bytes = 2.0 * n * dim * 4;
  float ms;
  for (int rep = 0; rep < 3; ++rep) {
    cudaMemset(flush, rep, 256 << 20);
    cudaEventRecord(e0);
    k_reg<<<148 * 6, 256>>>(ids, n, (const float4 *)f, dim / 4, stride / 4, (float4 *)ref);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("register gather (all warps): %.1f us, %.0f GB/s\n", ms * 1e3, bytes / ms / 1e6);
  }
  auto runv = [&](auto kern, const char *name, int grid) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaMemset(flush, rep, 256 << 20);
      cudaEventRecord(e0);
      kern<<<grid, 256>>>(ids, n, (const float4 *)f, dim / 4, stride / 4, (float4 *)out);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
    }
    printf("register gather %s grid %d: %.1f us, %.0f GB/s\n", name, grid, ms * 1e3, bytes / ms / 1e6);
  };
  runv(k_regv<0>, "ldg/st", 148 * 6);
  runv(k_regv<1>, "ld.nc.no_allocate/st", 148 * 6);
  runv(k_regv<2>, "ldg/st.cs", 148 * 6);
  runv(k_regv<3>, "no_allocate/st.cs", 148 * 6);
  runv(k_regv<7>, "no_allocate/st.cs/ldcg ids", 148 * 6);
  runv(k_regv<0>, "ldg/st", 148 * 8);
  runv(k_regv<0>, "ldg/st", 148 * 4);
  runv(k_regv<0>, "ldg/st", 148 * 16);
  auto run = [&](auto kern, int R, int S, int W, const char *name) {
    const int smem = W * S * R * dim * 4;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int nchunks = (n + R - 1) / R;
    for (int rep = 0; rep < 2; ++rep) {
      cudaMemset(flush, rep, 256 << 20);
      cudaMemset(out, 0, (size_t)n * dim * 4);
      cudaEventRecord(e0);
      kern<<<148, W * 32, smem>>>(ids, n, (const char *)f, dim * 4, stride * 4, (char *)out, nchunks);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
      printf("TMA gather %s W=%d warps/SM, R=%d rows/chunk, S=%d slots (%d KB smem): %.1f us, %.0f GB/s  %s\n", name, W,
             R, S, smem >> 10, ms * 1e3, bytes / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
    }
    // check
    std::vector<float> a(1000 * dim), b(1000 * dim);
    cudaMemcpy(a.data(), out + (size_t)(n - 1000) * dim, 1000 * dim * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(b.data(), ref + (size_t)(n - 1000) * dim, 1000 * dim * 4, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (size_t i = 0; i < a.size(); ++i) bad += a[i] != b[i];
    printf("   mismatches in the last 1000 rows: %d\n", bad);
  };
  run(k_tma<16, 4>, 16, 4, 4, "");
  run(k_tma<32, 2>, 32, 2, 4, "");
  run(k_tma<32, 3>, 32, 3, 4, "");
  run(k_tma<16, 6>, 16, 6, 4, "");
  run(k_tma<32, 2>, 32, 2, 6, "");
  run(k_tma<32, 4>, 32, 4, 2, "");
  return 0;
}
