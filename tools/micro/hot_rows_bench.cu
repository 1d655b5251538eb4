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


// Hot-row experiment: sampled rows of real products batches (oracle ids,
// .scratch/ids16.bin), rows of the X nodes of largest degree read with
// L2::evict_last, all others evict_first (the library's policy).  Batches run
// back to back (steady state), 4 concurrent streams x 37 blocks as the bench.
constexpr int R = 32, S = 2, W = 4;
__global__ void k_gather(const int *ids, int n, const char *tab, int row_bytes, const int *rank, int X, char *out) {
  extern __shared__ __align__(128) char smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int slot_bytes = (R * row_bytes + 127) / 128 * 128;
  char *ring = smem + (size_t)warp * S * slot_bytes;
  __shared__ __align__(8) uint64_t bars[W][S];
  if (lane == 0)
    for (int s = 0; s < S; ++s) mbar_init(&bars[warp][s], 1);
  __syncwarp();
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const unsigned long long pf = pol_first(), pl = pol_last();
  const int nchunks = (n + R - 1) / R;
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
        const bool hot = X > 0 && __ldg(rank + g) < X;
        char *dst = ring + (size_t)s * slot_bytes + lane * row_bytes;
        bulk_g2s(dst, tab + (size_t)g * row_bytes, row_bytes, &bars[warp][s], hot ? pl : pf);
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

int main(int argc, char **argv) {
  const int N = 2449029, dim = 100, NB = 16, ROWB = dim * 4;
  FILE *f = fopen(".scratch/ids16.bin", "rb");
  std::vector<std::vector<int>> b(NB);
  for (int i = 0; i < NB; ++i) {
    int n; fread(&n, 4, 1, f); b[i].resize(n); fread(b[i].data(), 4, n, f);
  }
  fclose(f);
  std::vector<int> rk(N);
  f = fopen(".scratch/degrank.bin", "rb"); fread(rk.data(), 4, N, f); fclose(f);
  char *tab; cudaMalloc(&tab, (size_t)N * ROWB); cudaMemset(tab, 1, (size_t)N * ROWB);
  int *rank; cudaMalloc(&rank, (size_t)N * 4); cudaMemcpy(rank, rk.data(), (size_t)N * 4, cudaMemcpyHostToDevice);
  int *ids[NB]; char *out[4];
  for (int i = 0; i < NB; ++i) { cudaMalloc(&ids[i], b[i].size() * 4); cudaMemcpy(ids[i], b[i].data(), b[i].size() * 4, cudaMemcpyHostToDevice); }
  for (int s = 0; s < 4; ++s) cudaMalloc(&out[s], (size_t)700000 * ROWB);
  // a 40 MB "relabel map" stand-in touched with evict_last between batches is not modelled
  char *flush; cudaMalloc(&flush, 512 << 20);
  cudaStream_t st[4]; for (int s = 0; s < 4; ++s) cudaStreamCreateWithFlags(&st[s], cudaStreamNonBlocking);
  const int smem = W * S * ((R * ROWB + 127) / 128 * 128);
  cudaFuncSetAttribute(k_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int Xs[] = {0, 50000, 100000, 150000, 200000, 300000, 0};
  for (int rep = 0; rep < 2; ++rep)
  for (int xi = 0; xi < 7; ++xi) {
    const int X = Xs[xi];
    cudaMemset(flush, xi, 512 << 20);
    const int rounds = 8;  // 8 x 16 batches
    double tot_rows = 0;
    for (int warm = 0; warm < 2; ++warm) {
      cudaDeviceSynchronize();
      cudaEventRecord(e0, 0);
      for (int s = 0; s < 4; ++s) cudaStreamWaitEvent(st[s], e0, 0);
      tot_rows = 0;
      for (int r = 0; r < (warm ? rounds : 1); ++r)
        for (int i = 0; i < NB; ++i) {
          const int s = i % 4; const int n = (int)b[i].size(); tot_rows += n;
          k_gather<<<37, 32 * W, smem, st[s]>>>(ids[i], n, tab, ROWB, rank, X, out[s]);
        }
      for (int s = 0; s < 4; ++s) { cudaEvent_t e; cudaEventCreateWithFlags(&e, cudaEventDisableTiming); cudaEventRecord(e, st[s]); cudaStreamWaitEvent(0, e, 0); }
      cudaEventRecord(e1, 0);
      cudaEventSynchronize(e1);
    }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double per = ms * 1e3 / (rounds * NB);
    printf("X=%7d (%5.1f MB hot): %.1f us per batch, %.2f TB/s algorithmic (2 x 400 B per row)\n", X, X * 400.0 / 1e6, per,
           tot_rows * 2 * ROWB / (ms * 1e-3) / 1e12);
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
