// dsp_kernels.cuh -- the CSP layer kernels and the feature gather (sm_100a).
//
// Per layer l:
//   world == 1 : k_sample_local           (sample + hash insert, fused)
//   world  > 1 : k_bucket_scatter         (shuffle: ids -> owners' inboxes over NVLink)
//                k_sample_remote          (sample at the owner, rows -> requesters)
//                k_unpermute_insert       (reshuffle consumer + hash insert)
//   then       : k_scan_assign            (single-pass scan: indptr, first occurrences,
//                                          new local ids, src_ids)
//                k_write_indices          (local src ids per edge)
// and k_gather for the loader.
#pragma once
#include "dsp_device.cuh"

namespace dsp {

// Device-side per-call state at the start of the caller's workspace.  The
// host copies it back once per dsp_sample.
struct WsHeader {
  int32_t err;
  int32_t pad0;
  int32_t F[9];          // frontier size per layer (F[0] = num_seeds)
  int32_t S[8];          // num_src per layer
  int64_t E[8];          // num_edges per layer
  uint32_t done;         // last-block counter (bucket / remote sample)
  uint32_t bucket[8];    // per-owner send counters (bucket scatter)
  uint32_t pad1[3];
};

// ----------------------------------------------------------- local sample
struct LocalSampleArgs {
  const int32_t *frontier;  // layer 0: seeds; else the previous block's src_ids
  int32_t F0;               // layer 0 only
  int32_t layer, k;
  uint2 key;                // rng_seed
  const int64_t *indptr;    // this rank's CSR
  const int32_t *indices;
  int64_t lo, n_local;      // rows [lo, lo + n_local) are local
  unsigned long long *tbl;
  uint32_t mask;
  int32_t *cnt;             // [F]
  int32_t *hpos;            // [F*k] table slot of each sampled edge
  WsHeader *hdr;
};

__device__ __forceinline__ int frontier_size(const WsHeader *hdr, int layer, int F0) {
  return layer == 0 ? F0 : *(volatile const int32_t *)&hdr->F[layer];
}

// World size 1: sample every frontier node and insert dst + sampled srcs into
// the relabel table in the same pass.
template <int G>
__global__ void __launch_bounds__(256) k_sample_local(LocalSampleArgs a) {
  const int F = frontier_size(a.hdr, a.layer, a.F0);
  if (a.layer == 0 && blockIdx.x == 0 && threadIdx.x == 0) a.hdr->F[0] = a.F0;
  constexpr int NPW = 32 / G;  // nodes per warp-iteration
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  const int k = a.k;
  for (int base = warp * NPW; base < F; base += nwarps * NPW) {
    const int i = base + lane / G;
    const bool active = i < F;
    int32_t v = active ? __ldg(a.frontier + i) : 0;
    const int64_t lv = (int64_t)v - a.lo;
    const bool ok = active && v >= 0 && lv >= 0 && lv < a.n_local;
    if (active && !ok && (lane & (G - 1)) == 0) latch(&a.hdr->err, E_RANGE);
    int64_t s = 0, d = 0;
    if (ok) {
      s = __ldg(a.indptr + lv);
      d = __ldg(a.indptr + lv + 1) - s;
    }
    bool valid;
    int slot, cnt;
    int32_t u;
    sample_node<G>(ok, v, s, d, k, a.layer, a.key, a.indices, &valid, &slot, &u, &cnt);
    if (ok && (lane & (G - 1)) == 0) {
      a.cnt[i] = cnt;
      uint32_t old;
      table_insert_min(a.tbl, a.mask, (uint32_t)v, (uint32_t)i, &old);
      if (a.layer == 0 && old < (uint32_t)F && old != (uint32_t)i) latch(&a.hdr->err, E_DUP);
    } else if (active && !ok && (lane & (G - 1)) == 0) {
      a.cnt[i] = 0;
    }
    if (valid) {
      const int64_t q = (int64_t)i * k + slot;
      uint32_t old;
      a.hpos[q] = (int32_t)table_insert_min(a.tbl, a.mask, (uint32_t)u, (uint32_t)(F + q), &old);
    }
  }
}

// ------------------------------------------------------------ scan/assign
// Decoupled look-back scan over edge slots q in [0, F*k) of two counts:
// valid (edge exists) and first (first occurrence of a new src node).
// Tile status word: [63:62] flag (3 = not ready, 1 = aggregate, 2 = inclusive)
// [61:31] first count, [30:0] valid count.  The status array and the tile
// ticket are reset to all ones by the per-layer table memset.
constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;
constexpr unsigned long long ST_VAL_MASK = (1ull << 62) - 1;
constexpr unsigned long long ST_AGG = 1ull << 62;
constexpr unsigned long long ST_INC = 2ull << 62;

struct ScanArgs {
  int32_t layer, k;
  const int32_t *frontier;
  const int32_t *cnt;
  const int32_t *hpos;
  unsigned long long *tbl;
  unsigned long long *status;  // [0] = ticket, [1 + tile] = tile status
  int32_t *indptr_out;         // [F+1]
  int32_t *src_ids_out;        // [F + new]
  WsHeader *hdr;
};

__device__ __forceinline__ unsigned long long pack2(uint32_t valid, uint32_t first) {
  return ((unsigned long long)first << 31) | valid;
}

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
  return *(volatile const unsigned long long *)p;
}

__global__ void __launch_bounds__(SCAN_THREADS) k_scan_assign(ScanArgs a) {
  __shared__ unsigned long long s_warp[SCAN_THREADS / 32];
  __shared__ unsigned long long s_prefix;
  __shared__ uint32_t s_tile;
  const int F = *(volatile const int32_t *)&a.hdr->F[a.layer];
  const int k = a.k;
  const int64_t total = (int64_t)F * k;
  const int64_t ntiles = total > 0 ? (total + SCAN_TILE - 1) / SCAN_TILE : 1;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  unsigned long long *ticket = a.status;
  unsigned long long *st = a.status + 1;

  while (true) {
    if (tid == 0) s_tile = (uint32_t)(atomicAdd(ticket, 1ull) + 1ull);  // starts at ~0
    __syncthreads();
    const int64_t tile = s_tile;
    __syncthreads();
    if (tile >= ntiles) break;
    const int64_t q0 = tile * SCAN_TILE + (int64_t)tid * SCAN_ITEMS;

    // pass 1: per-item flags
    uint32_t vbits = 0, fbits = 0;
    uint32_t keys[SCAN_ITEMS];
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; ++j) {
      const int64_t q = q0 + j;
      keys[j] = 0;
      if (q < total) {
        const int i = (int)(q / k);
        const int t = (int)(q - (int64_t)i * k);
        if (t < __ldg(a.cnt + i)) {
          vbits |= 1u << j;
          const unsigned long long w = ld_volatile_u64(a.tbl + __ldg(a.hpos + q));
          keys[j] = (uint32_t)(w >> 32);
          if ((uint32_t)w == (uint32_t)(F + q)) fbits |= 1u << j;
        }
      }
    }
    const unsigned long long mine = pack2(__popc(vbits), __popc(fbits));

    // block exclusive scan of `mine`
    unsigned long long incl = mine;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const unsigned long long y = __shfl_up_sync(FULL_MASK, incl, off);
      if (lane >= off) incl += y;
    }
    if (lane == 31) s_warp[wid] = incl;
    __syncthreads();
    if (wid == 0) {
      unsigned long long w = lane < SCAN_THREADS / 32 ? s_warp[lane] : 0ull;
#pragma unroll
      for (int off = 1; off < SCAN_THREADS / 32; off <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL_MASK, w, off);
        if (lane >= off) w += y;
      }
      if (lane < SCAN_THREADS / 32) s_warp[lane] = w;  // inclusive warp totals
    }
    __syncthreads();
    const unsigned long long warp_excl = wid ? s_warp[wid - 1] : 0ull;
    const unsigned long long thread_excl = warp_excl + incl - mine;
    const unsigned long long agg = s_warp[SCAN_THREADS / 32 - 1];

    // decoupled look-back (warp 0)
    if (wid == 0) {
      unsigned long long prefix = 0;
      if (tile == 0) {
        if (lane == 0) *(volatile unsigned long long *)&st[0] = ST_INC | agg;
      } else {
        if (lane == 0) *(volatile unsigned long long *)&st[tile] = ST_AGG | agg;
        int64_t idx = tile - 1;
        while (true) {
          const int64_t p = idx - lane;
          unsigned long long s = ST_INC;  // virtual inclusive zero before tile 0
          if (p >= 0) {
            do {
              s = ld_volatile_u64(&st[p]);
            } while ((s >> 62) == 3ull);
          }
          const unsigned incm = __ballot_sync(FULL_MASK, (s >> 62) == 2ull);
          const int stop = incm ? (__ffs(incm) - 1) : 31;
          unsigned long long v = (lane <= stop) ? (s & ST_VAL_MASK) : 0ull;
#pragma unroll
          for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(FULL_MASK, v, off);
          prefix += v;
          if (incm) break;
          idx -= 32;
        }
        if (lane == 0) *(volatile unsigned long long *)&st[tile] = ST_INC | (prefix + agg);
      }
      if (lane == 0) s_prefix = prefix;
    }
    __syncthreads();
    const unsigned long long base = s_prefix + thread_excl;
    uint32_t pv = (uint32_t)(base & 0x7fffffffull);
    uint32_t pf = (uint32_t)((base >> 31) & 0x7fffffffull);

    // pass 2: outputs
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; ++j) {
      const int64_t q = q0 + j;
      if (q < total) {
        const int i = (int)(q / k);
        const int t = (int)(q - (int64_t)i * k);
        if (t == 0) {
          a.indptr_out[i] = (int32_t)pv;
          a.src_ids_out[i] = __ldg(a.frontier + i);
        }
        if (fbits & (1u << j)) {
          const uint32_t nid = (uint32_t)F + pf;
          a.tbl[__ldg(a.hpos + q)] = ((unsigned long long)keys[j] << 32) | nid;
          a.src_ids_out[nid] = (int32_t)keys[j];
        }
        pv += (vbits >> j) & 1u;
        pf += (fbits >> j) & 1u;
      }
    }
    if (tile == ntiles - 1 && tid == 0) {
      const unsigned long long tot = s_prefix + agg;
      const int32_t E = (int32_t)(tot & 0x7fffffffull);
      const int32_t nnew = (int32_t)((tot >> 31) & 0x7fffffffull);
      a.indptr_out[F] = E;
      a.hdr->E[a.layer] = E;
      a.hdr->S[a.layer] = F + nnew;
      a.hdr->F[a.layer + 1] = F + nnew;
    }
  }
}

// ---------------------------------------------------------- write indices
struct IndicesArgs {
  int32_t layer, k;
  const int32_t *cnt;
  const int32_t *hpos;
  const unsigned long long *tbl;
  const int32_t *indptr;  // block indptr
  int32_t *indices_out;
  WsHeader *hdr;
};

__global__ void __launch_bounds__(256) k_write_indices(IndicesArgs a) {
  const int F = *(volatile const int32_t *)&a.hdr->F[a.layer];
  const int k = a.k;
  const int64_t total = (int64_t)F * k;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < total;
       q += (int64_t)gridDim.x * blockDim.x) {
    const int i = (int)(q / k);
    const int t = (int)(q - (int64_t)i * k);
    if (t < __ldg(a.cnt + i)) {
      const unsigned long long w = a.tbl[__ldg(a.hpos + q)];
      a.indices_out[__ldg(a.indptr + i) + t] = (int32_t)(uint32_t)w;
    }
  }
}

// ----------------------------------------------------------------- gather
struct GatherArgs {
  const int32_t *ids;
  int64_t n;
  int32_t dim4;             // dim / 4
  float4 *out;
  const float4 *base[8];    // feature shard of each rank (local or peer-mapped)
  Bounds bd;
  int *err;
};

// One float4 per thread-iteration over the flat [n][dim4] output; UNROLL
// independent 16-byte loads in flight per thread before any store.
template <int UNROLL>
__global__ void __launch_bounds__(256) k_gather(GatherArgs a) {
  const int64_t total = a.n * a.dim4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t start = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  for (int64_t e0 = start; e0 < total; e0 += stride * UNROLL) {
    float4 v[UNROLL];
    int64_t e[UNROLL];
    bool ok[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      e[u] = e0 + (int64_t)u * stride;
      ok[u] = false;
      if (e[u] < total) {
        const int64_t r = e[u] / a.dim4;
        const int64_t c = e[u] - r * a.dim4;
        const int32_t g = __ldg(a.ids + r);
        if (g >= 0 && g < a.bd.b[a.bd.world]) {
          const int o = owner_of(a.bd, g);
          v[u] = __ldg(a.base[o] + (g - a.bd.b[o]) * a.dim4 + c);
          ok[u] = true;
        } else {
          latch(a.err, E_RANGE);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u)
      if (ok[u]) a.out[e[u]] = v[u];
  }
}

// ===================================================== world > 1 (CSP)
// Peer-visible exchange region of each rank (library-owned, CUDA-IPC mapped
// by every peer).  p = parity of the layer call, s = sender / owner rank.
struct XchLayout {
  int64_t cap;              // slots per (parity, peer)
  int32_t kmax;
  size_t off_inbox_flag;    // u64 [2][8]
  size_t off_ret_flag;      // u64 [2][8]
  size_t off_inbox_hdr;     // uint4 [2][8]  {count, k | layer << 8, seed lo, seed hi}
  size_t off_inbox;         // i32 [2][8][cap]
  size_t off_ret_cnt;       // i32 [2][8][cap]
  size_t off_ret_rows;      // i32 [2][8][cap * kmax]
  size_t bytes;
};

struct XchPeers {
  char *base[8];            // exchange region of each rank (local pointer for self)
};

__device__ __forceinline__ unsigned long long *xch_inbox_flag(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_inbox_flag) + p * 8 + s;
}
__device__ __forceinline__ unsigned long long *xch_ret_flag(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_ret_flag) + p * 8 + s;
}
__device__ __forceinline__ uint4 *xch_inbox_hdr(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<uint4 *>(b + L.off_inbox_hdr) + p * 8 + s;
}
__device__ __forceinline__ int32_t *xch_inbox(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<int32_t *>(b + L.off_inbox) + ((int64_t)p * 8 + s) * L.cap;
}
__device__ __forceinline__ int32_t *xch_ret_cnt(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<int32_t *>(b + L.off_ret_cnt) + ((int64_t)p * 8 + s) * L.cap;
}
__device__ __forceinline__ int32_t *xch_ret_rows(char *b, const XchLayout &L, int p, int s) {
  return reinterpret_cast<int32_t *>(b + L.off_ret_rows) + ((int64_t)p * 8 + s) * L.cap * L.kmax;
}

constexpr unsigned long long WAIT_TIMEOUT_NS = 20ull * 1000 * 1000 * 1000;  // 20 s

// Waits until flags[s] >= seq for every s < world.  On timeout latches
// E_STATE and returns false (a peer never arrived; never hang the GPU).
__device__ __forceinline__ bool wait_flags(unsigned long long *flags0, int world,
                                           unsigned long long seq, int *err) {
  __shared__ int s_ok;
  if (threadIdx.x == 0) {
    const unsigned long long t0 = globaltimer_ns();
    int ok = 1;
    for (int s = 0; s < world && ok; ++s) {
      while (ld_acquire_sys(flags0 + s) < seq) {
        if (globaltimer_ns() - t0 > WAIT_TIMEOUT_NS) {
          latch(err, E_STATE);
          ok = 0;
          break;
        }
        __nanosleep(64);
      }
    }
    s_ok = ok;
  }
  __syncthreads();
  return s_ok != 0;
}

// Last-block-done: every block fences its (peer) stores and counts itself;
// returns true in exactly one thread of the last block to finish.
__device__ __forceinline__ bool last_block_done(uint32_t *done) {
  __shared__ int s_last;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t t = atomicAdd(done, 1u);
    s_last = (t == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (s_last && threadIdx.x == 0) {
    __threadfence_system();
    *(volatile uint32_t *)done = 0u;  // reset for the next use
    return true;
  }
  return false;
}

struct BucketArgs {
  const int32_t *frontier;
  int32_t F0, layer, k;
  uint32_t seed_lo, seed_hi;
  int32_t rank, parity;
  unsigned long long seq;
  Bounds bd;
  XchLayout L;
  XchPeers peers;
  int32_t *perm;            // [F] slot of frontier i in its owner's inbox
  WsHeader *hdr;
};

// Shuffle: group the frontier by owner (range check) and
// write each id straight into the owner's inbox over NVLink; the slot order
// inside a bucket is irrelevant (results come back to the same slot).  The
// last block publishes the per-owner counts + header, then the flag
// (count notification before use).
__global__ void __launch_bounds__(256) k_bucket_scatter(BucketArgs a) {
  __shared__ uint32_t s_cnt[8], s_base[8];
  const int F = frontier_size(a.hdr, a.layer, a.F0);
  if (a.layer == 0 && blockIdx.x == 0 && threadIdx.x == 0 && F <= a.L.cap) a.hdr->F[0] = a.F0;
  if (F > a.L.cap && blockIdx.x == 0 && threadIdx.x == 0) {
    latch(&a.hdr->err, E_CAP);
    a.hdr->F[a.layer] = 0;  // later kernels of this layer see an empty frontier
  }
  const int limit = F > a.L.cap ? 0 : F;
  const int chunk = blockDim.x;
  for (int b0 = blockIdx.x * chunk; b0 < ((limit + chunk - 1) / chunk) * chunk;
       b0 += gridDim.x * chunk) {
    if (threadIdx.x < 8) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    const int i = b0 + threadIdx.x;
    int o = -1;
    uint32_t local = 0;
    int32_t v = 0;
    if (i < limit) {
      v = __ldg(a.frontier + i);
      if (v < 0 || v >= a.bd.b[a.bd.world]) {
        latch(&a.hdr->err, E_RANGE);
      } else {
        o = owner_of(a.bd, v);
        local = atomicAdd(&s_cnt[o], 1u);
      }
    }
    __syncthreads();
    if (threadIdx.x < a.bd.world) s_base[threadIdx.x] = atomicAdd(&a.hdr->bucket[threadIdx.x], s_cnt[threadIdx.x]);
    __syncthreads();
    if (o >= 0) {
      const uint32_t j = s_base[o] + local;
      xch_inbox(a.peers.base[o], a.L, a.parity, a.rank)[j] = v;
      a.perm[i] = (int32_t)j;
    }
    __syncthreads();
  }
  if (last_block_done(&a.hdr->done)) {
    for (int o = 0; o < a.bd.world; ++o) {
      const uint32_t c = *(volatile uint32_t *)&a.hdr->bucket[o];
      a.hdr->bucket[o] = 0u;
      *xch_inbox_hdr(a.peers.base[o], a.L, a.parity, a.rank) =
          make_uint4(c, (uint32_t)a.k | ((uint32_t)a.layer << 8), a.seed_lo, a.seed_hi);
    }
    __threadfence_system();
    for (int o = 0; o < a.bd.world; ++o)
      st_release_sys(xch_inbox_flag(a.peers.base[o], a.L, a.parity, a.rank), a.seq);
  }
}

struct RemoteSampleArgs {
  int32_t layer, k;
  uint2 key;
  int32_t rank, parity;
  unsigned long long seq;
  const int64_t *indptr;
  const int32_t *indices;
  int64_t lo, n_local;
  Bounds bd;
  XchLayout L;
  XchPeers peers;
  WsHeader *hdr;
};

// Sample stage at the owner: one kernel over every task received in
// this layer, results written straight into each requester's
// return slots over NVLink, then the return flags.
template <int G>
__global__ void __launch_bounds__(256) k_sample_remote(RemoteSampleArgs a) {
  __shared__ uint32_t s_off[9];
  char *self = a.peers.base[a.rank];
  const int world = a.bd.world;
  if (wait_flags(xch_inbox_flag(self, a.L, a.parity, 0), world, a.seq, &a.hdr->err)) {
    if (threadIdx.x == 0) {
      uint32_t acc = 0;
      for (int s = 0; s < world; ++s) {
        const uint4 h = __ldcv(xch_inbox_hdr(self, a.L, a.parity, s));
        if (h.y != ((uint32_t)a.k | ((uint32_t)a.layer << 8)) || h.z != a.key.x || h.w != a.key.y)
          latch(&a.hdr->err, E_STATE);
        s_off[s] = acc;
        acc += (h.x <= (uint32_t)a.L.cap) ? h.x : 0u;
      }
      s_off[world] = acc;
    }
    __syncthreads();
    const int T = (int)s_off[world];
    constexpr int NPW = 32 / G;
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * blockDim.x) >> 5;
    const int k = a.k;
    for (int base = warp * NPW; base < T; base += nwarps * NPW) {
      const int q = base + lane / G;
      const bool active = q < T;
      int s = 0;
      if (active) {
        while (s + 1 < world && (uint32_t)q >= s_off[s + 1]) ++s;
      }
      const int j = q - (int)s_off[s];
      int32_t v = active ? *(volatile int32_t *)(xch_inbox(self, a.L, a.parity, s) + j) : 0;
      const int64_t lv = (int64_t)v - a.lo;
      const bool ok = active && lv >= 0 && lv < a.n_local;
      if (active && !ok && (lane & (G - 1)) == 0) latch(&a.hdr->err, E_STATE);
      int64_t rs = 0, d = 0;
      if (ok) {
        rs = __ldg(a.indptr + lv);
        d = __ldg(a.indptr + lv + 1) - rs;
      }
      bool valid;
      int slot, cnt;
      int32_t u;
      sample_node<G>(ok, v, rs, d, k, a.layer, a.key, a.indices, &valid, &slot, &u, &cnt);
      char *req = a.peers.base[s];
      if (active && (lane & (G - 1)) == 0) xch_ret_cnt(req, a.L, a.parity, a.rank)[j] = cnt;
      if (valid) xch_ret_rows(req, a.L, a.parity, a.rank)[(int64_t)j * a.L.kmax + slot] = u;
    }
  }
  if (last_block_done(&a.hdr->done)) {
    for (int s = 0; s < world; ++s)
      st_release_sys(xch_ret_flag(a.peers.base[s], a.L, a.parity, a.rank), a.seq);
  }
}

struct UnpermuteArgs {
  const int32_t *frontier;
  int32_t layer, k;
  int32_t rank, parity;
  unsigned long long seq;
  Bounds bd;
  XchLayout L;
  char *self;
  const int32_t *perm;
  unsigned long long *tbl;
  uint32_t mask;
  int32_t *cnt;
  int32_t *hpos;
  WsHeader *hdr;
};

// Reshuffle consumer ("transferred back to the GPU requesting"):
// frontier node i reads its row from the owner's return slot perm[i], and
// the dst + sampled srcs go into the relabel table (as k_sample_local does).
template <int G>
__global__ void __launch_bounds__(256) k_unpermute_insert(UnpermuteArgs a) {
  const int world = a.bd.world;
  if (!wait_flags(xch_ret_flag(a.self, a.L, a.parity, 0), world, a.seq, &a.hdr->err)) return;
  const int F = *(volatile const int32_t *)&a.hdr->F[a.layer];
  const int lim = F > a.L.cap ? 0 : F;
  constexpr int NPW = 32 / G;
  const int lane = threadIdx.x & 31;
  const int t = lane & (G - 1);
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nwarps = (gridDim.x * blockDim.x) >> 5;
  const int k = a.k;
  for (int base = warp * NPW; base < lim; base += nwarps * NPW) {
    const int i = base + lane / G;
    if (i >= lim) continue;
    const int32_t v = __ldg(a.frontier + i);
    if (v < 0 || v >= a.bd.b[world]) {  // latched by the bucket kernel
      if (t == 0) a.cnt[i] = 0;
      continue;
    }
    const int o = owner_of(a.bd, v);
    const int j = __ldg(a.perm + i);
    const int c = *(volatile int32_t *)(xch_ret_cnt(a.self, a.L, a.parity, o) + j);
    if (t == 0) {
      a.cnt[i] = c;
      uint32_t old;
      table_insert_min(a.tbl, a.mask, (uint32_t)v, (uint32_t)i, &old);
      if (a.layer == 0 && old < (uint32_t)F && old != (uint32_t)i) latch(&a.hdr->err, E_DUP);
    }
    if (t < c) {
      const int32_t u =
          *(volatile int32_t *)(xch_ret_rows(a.self, a.L, a.parity, o) + (int64_t)j * a.L.kmax + t);
      const int64_t q = (int64_t)i * k + t;
      uint32_t old;
      a.hpos[q] = (int32_t)table_insert_min(a.tbl, a.mask, (uint32_t)u, (uint32_t)(F + q), &old);
    }
  }
}

}  // namespace dsp
