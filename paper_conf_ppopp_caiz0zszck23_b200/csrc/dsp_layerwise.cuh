// dsp_layerwise.cuh -- layer-wise CSP (Sec. 4.2, Eq. 2;
// Table 7 "layer-wise sampling without replacement"; R28-R30).
//
// Per layer l with layer size n, phases of ONE cooperative launch per rank
// and call (k_lw_persistent at world 1, k_lw_multi at world > 1), separated by
// grid barriers:
//   alloc   (block 0)  W_u = deg u read from the OWNER's indptr over peer
//                      memory (8 B per frontier node instead of its adjacency
//                      list), exclusive scan P, n Philox draws
//                      r = mulhi64(word, T) mapped to the frontier interval
//                      containing r (Eq. 2, with replacement), counts c_u,
//                      slot offsets, then the sampling tasks (u, c_u) pushed to
//                      the owners' inboxes (shuffle).
//   sample  (grid)     owner side: one warp per task, c_u <= 32 by the warp
//                      Floyd of the node-wise path, whole rows when
//                      deg <= c_u; rows written straight into the requester's
//                      return slots.
//   big     (grid)     tasks with 32 < c_u < deg: one block per task, draws in
//                      parallel, Floyd's resolution by one thread against a
//                      shared-memory hash set, bitonic sort; then the return
//                      flags.
//   collect (grid)     requester: dst marks + first-occurrence marks of the
//                      returned rows (epoch-tagged map).
//   finish  (block 0)  scan over the <= n edge slots, relabel, indptr /
//                      indices / src_ids, sizes.
// At world 1 the "peer" is the ctx itself (its exchange slots sit in the
// workspace).  The phase bodies take PERS = true (inside the persistent
// kernel: the flag waits of a phase that follows a grid barrier are skipped).
#pragma once
#include "dsp_kernels.cuh"

namespace dsp {

constexpr int LWT = 1024;            // threads of the single-block kernels
constexpr int LW_MAX_SIZE = 8192;    // DSP_MAX_LAYER_SIZE

struct LwLayout {
  int64_t cap;               // frontier capacity = requests per (parity, requester)
  int32_t ncap;              // edge-slot capacity = max layer size
  size_t off_inbox_flag;     // u64 [2][8]
  size_t off_ret_flag;       // u64 [2][8]
  size_t off_inbox_hdr;      // uint4 [2][8] {count, n | layer << 16, seed lo, seed hi}
  size_t off_inbox;          // int4 [2][8][cap] {i, v, c, slot offset}
  size_t off_ret_cnt;        // i32 [2][cap]  sampled count of requester frontier node i
  size_t off_ret_rows;       // i32 [2][ncap] sampled neighbours by requester edge slot
  size_t bytes;
};

__device__ __forceinline__ unsigned long long *lw_inbox_flag(char *b, const LwLayout &L, int p, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_inbox_flag) + p * 8 + s;
}
__device__ __forceinline__ unsigned long long *lw_ret_flag(char *b, const LwLayout &L, int p, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_ret_flag) + p * 8 + s;
}
__device__ __forceinline__ uint4 *lw_inbox_hdr(char *b, const LwLayout &L, int p, int s) {
  return reinterpret_cast<uint4 *>(b + L.off_inbox_hdr) + p * 8 + s;
}
__device__ __forceinline__ int4 *lw_inbox(char *b, const LwLayout &L, int p, int s) {
  return reinterpret_cast<int4 *>(b + L.off_inbox) + ((int64_t)p * 8 + s) * L.cap;
}
__device__ __forceinline__ int32_t *lw_ret_cnt(char *b, const LwLayout &L, int p) {
  return reinterpret_cast<int32_t *>(b + L.off_ret_cnt) + (int64_t)p * L.cap;
}
__device__ __forceinline__ int32_t *lw_ret_rows(char *b, const LwLayout &L, int p) {
  return reinterpret_cast<int32_t *>(b + L.off_ret_rows) + (int64_t)p * L.ncap;
}

// Per-call workspace arrays of the layer-wise path (after persist|hdr|first).
struct LwBufs {
  unsigned long long *P;   // [cap + 1] W, then its exclusive prefix (P[F] = T)
  int32_t *c;              // [cap] draws per frontier node
  int32_t *off;            // [cap + 1] edge-slot offset of frontier node i (exclusive scan of c)
  int32_t *slot_node;      // [ncap] frontier node of edge slot q
  int32_t *excl;           // [ncap + 1] valid slots before q
  int32_t *newid;          // [ncap] first-occurrence slots before q
  int2 *big;               // [8 * ncap / 32 + 8] owner-side (requester, inbox index) with 32 < c < deg
  int32_t big_cap;
};

struct LwArgs {
  const int32_t *seeds;    // g0 = seeds[0] identifies the graph sample (R29)
  const int32_t *frontier;
  int32_t F0, layer, n, rank, parity;
  uint2 key;
  unsigned long long seq;
  Bounds bd;
  const int64_t *peer_indptr[8];
  const int64_t *indptr;   // own shard
  const int32_t *indices;
  int64_t lo, n_local;
  LwLayout L;
  XchPeers peers;
  LwBufs w;
  unsigned long long *first;
  const WsPersist *persist;
  Outputs out;             // block l arrays in out.*[0]
  WsHeader *hdr;
  int *err;
  int32_t sys;             // peers on other devices: system-scope fences (else GPU scope)
};

// Last-block-done with a fence of the given scope (see last_block_done).
__device__ __forceinline__ bool lw_last_block_done(uint32_t *done, int sys) {
  __shared__ int s_last;
  if (sys) __threadfence_system(); else __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t t = atomicAdd(done, 1u);
    s_last = (t == gridDim.x - 1) ? 1 : 0;
  }
  __syncthreads();
  if (s_last && threadIdx.x == 0) {
    if (sys) __threadfence_system(); else __threadfence();
    *(volatile uint32_t *)done = 0u;
    return true;
  }
  return false;
}

__device__ __forceinline__ uint32_t lw_tag(int n, int layer) { return (uint32_t)n | ((uint32_t)layer << 16); }

// Block-wide exclusive scan of one value per thread (LWT threads); returns the
// exclusive prefix and writes the block total to *total.
template <typename T>
__device__ __forceinline__ T block_excl_scan(T x, T *s_warp, T *total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  T incl = x;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T y = __shfl_up_sync(FULL_MASK, incl, off);
    if (lane >= off) incl += y;
  }
  if (lane == 31) s_warp[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    T v = s_warp[lane];  // LWT / 32 == 32 warps
    T vi = v;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const T y = __shfl_up_sync(FULL_MASK, vi, off);
      if (lane >= off) vi += y;
    }
    s_warp[lane] = vi - v;  // exclusive warp offsets
    if (lane == 31) s_warp[32] = vi;
  }
  __syncthreads();
  const T r = s_warp[wid] + incl - x;
  *total = s_warp[32];
  __syncthreads();
  return r;
}

constexpr int LW_IPT = 4;                 // frontier nodes per thread per pass of k_lw_alloc
constexpr int LW_SMEM_F = 8192;           // frontier sizes whose prefix + counts fit in shared memory
constexpr size_t LW_ALLOC_SMEM = (size_t)LW_SMEM_F * (sizeof(unsigned long long) + sizeof(int32_t));

// Dynamic shared memory: LW_ALLOC_SMEM (prefix u64 + counts i32 of up to
// LW_SMEM_F frontier nodes); larger frontiers use the workspace copies.
// PERS: inside the world-1 persistent kernel (k_lw_persistent): no flags, the
// phases are ordered by its grid barriers.
#ifdef DSP_DEBUG_STAMPS
#define LWSTAMP(a, idx) \
  do { if (threadIdx.x == 0) (a).hdr->dbg[16 + 4 * ((a).layer & 3) + (idx)] = globaltimer_ns(); } while (0)
#else
#define LWSTAMP(a, idx) do { } while (0)
#endif
template <bool PERS>
__device__ __forceinline__ void lw_alloc_body(const LwArgs &a, unsigned long long *lw_alloc_smem) {
  __shared__ unsigned long long s_u64[33];
  __shared__ int32_t s_i32[33];
  __shared__ uint32_t s_cnt[8];
  const int tid = threadIdx.x;
  int F = a.layer == 0 ? a.F0 : ld_volatile_i32(&a.hdr->F[a.layer]);
  if (F > a.L.cap) {  // bounded by the plan; never expected
    if (tid == 0) latch(a.err, E_CAP);
    F = 0;
  }
  if (tid == 0 && a.layer == 0) a.hdr->F[0] = F;
  const bool in_smem = F + 1 <= LW_SMEM_F;
  unsigned long long *P = in_smem ? lw_alloc_smem : a.w.P;
  int32_t *cnt = in_smem ? reinterpret_cast<int32_t *>(lw_alloc_smem + LW_SMEM_F) : a.w.c;
  const int32_t g0 = a.F0 > 0 ? __ldg(a.seeds) : 0;
  LWSTAMP(a, 0);
  // W_u from the owner's indptr (peer memory): LW_IPT independent loads per
  // thread in flight, then the block-wide exclusive scan
  unsigned long long carry = 0;
  for (int b0 = 0; b0 < F; b0 += LWT * LW_IPT) {
    unsigned long long W[LW_IPT];
    unsigned long long sum = 0;
#pragma unroll
    for (int j = 0; j < LW_IPT; ++j) {
      const int i = b0 + tid * LW_IPT + j;
      W[j] = 0;
      if (i < F) {
        const int32_t v = ldw_i32(a.frontier + i);  // may be written earlier in the same kernel (PERS)
        if (v < 0 || v >= a.bd.b[a.bd.world]) {
          latch(a.err, E_RANGE);
        } else {
          const int o = owner_of(a.bd, v);
          const int64_t lv = (int64_t)v - a.bd.b[o];
          const int64_t *ip = a.peer_indptr[o];
          W[j] = (unsigned long long)(ip[lv + 1] - ip[lv]);
        }
        cnt[i] = 0;
      }
      sum += W[j];
    }
    unsigned long long tot;
    unsigned long long ex = carry + block_excl_scan<unsigned long long>(sum, s_u64, &tot);
#pragma unroll
    for (int j = 0; j < LW_IPT; ++j) {
      const int i = b0 + tid * LW_IPT + j;
      if (i < F) P[i] = ex;
      ex += W[j];
    }
    carry += tot;
  }
  if (tid == 0) P[F] = carry;
  const unsigned long long T = carry;
  __syncthreads();
  LWSTAMP(a, 1);
  // Eq. 2: n draws with replacement, frontier node i with probability W_i / T
  if (T > 0)
    for (int j = tid; j < a.n; j += LWT) {
      const uint4 x = philox4x32_10(make_uint4((uint32_t)j, (uint32_t)g0, (uint32_t)a.layer, 0x4453504Cu), a.key);
      const unsigned long long word = ((unsigned long long)x.y << 32) | x.x;
      const unsigned long long r = __umul64hi(word, T);
      int lo = 0, hi = F - 1;  // largest i with P[i] <= r
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (P[mid] <= r) lo = mid; else hi = mid - 1;
      }
      atomicAdd(cnt + lo, 1);
    }
  __syncthreads();
  LWSTAMP(a, 2);
  // slot offsets, slot -> node, and the tasks pushed to the owners
  if (tid < 8) s_cnt[tid] = 0;
  int32_t ocarry = 0;
  for (int b0 = 0; b0 < F; b0 += LWT) {
    const int i = b0 + tid;
    const int32_t ci = i < F ? cnt[i] : 0;
    int o_req = -1;
    int4 req = make_int4(0, 0, 0, 0);
    int32_t tot;
    const int32_t ex = block_excl_scan<int32_t>(ci, s_i32, &tot);
    if (i < F) {
      const int32_t off = ocarry + ex;
      a.w.off[i] = off;
      if (ci > 0) {
        for (int t = 0; t < ci; ++t) a.w.slot_node[off + t] = i;
        const int32_t v = ldw_i32(a.frontier + i);  // may be written earlier in the same kernel (PERS)
        o_req = owner_of(a.bd, v);
        req = make_int4(i, v, ci, off);
      }
    }
    {  // warp-aggregated slot in the owner's inbox
      const unsigned peers = __match_any_sync(FULL_MASK, o_req);
      const int leader = __ffs(peers) - 1;
      const int lane = threadIdx.x & 31;
      uint32_t base = 0;
      if (o_req >= 0 && lane == leader) base = atomicAdd(&s_cnt[o_req], (uint32_t)__popc(peers));
      base = __shfl_sync(FULL_MASK, base, leader);
      if (o_req >= 0)
        lw_inbox(a.peers.base[o_req], a.L, a.parity, a.rank)[base + __popc(peers & ((1u << lane) - 1u))] = req;
    }
    ocarry += tot;
  }
  if (tid == 0) a.w.off[F] = ocarry;
  __syncthreads();
  LWSTAMP(a, 3);
  if (tid == 0) {
    for (int o = 0; o < a.bd.world; ++o)
      *lw_inbox_hdr(a.peers.base[o], a.L, a.parity, a.rank) = make_uint4(s_cnt[o], lw_tag(a.n, a.layer), a.key.x, a.key.y);
    if (!PERS) {
      if (a.sys) __threadfence_system();
      for (int o = 0; o < a.bd.world; ++o)
        st_release_flag(lw_inbox_flag(a.peers.base[o], a.L, a.parity, a.rank), a.seq, a.sys);
    }
  }
}

// Owner side: every task received in this layer, one warp each.
template <bool PERS>
__device__ __forceinline__ void lw_sample_remote_body(const LwArgs &a) {
  __shared__ uint32_t s_off[9];
  char *self = a.peers.base[a.rank];
  const int world = a.bd.world;
  if (PERS || wait_flags(lw_inbox_flag(self, a.L, a.parity, 0), world, a.seq, a.err)) {
    if (threadIdx.x == 0) {
      uint32_t acc = 0;
      for (int s = 0; s < world; ++s) {
        const uint4 h = __ldcv(lw_inbox_hdr(self, a.L, a.parity, s));
        if (h.y != lw_tag(a.n, a.layer) || h.z != a.key.x || h.w != a.key.y) latch(a.err, E_STATE);
        s_off[s] = acc;
        acc += (h.x <= (uint32_t)a.L.cap) ? h.x : 0u;
      }
      s_off[world] = acc;
    }
    __syncthreads();
    const int T = (int)s_off[world];
    const int lane = threadIdx.x & 31;
    const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int nwarps = (gridDim.x * blockDim.x) >> 5;
    for (int q = warp; q < T; q += nwarps) {
      int s = 0;
      while (s + 1 < world && (uint32_t)q >= s_off[s + 1]) ++s;
      const int j = q - (int)s_off[s];
      const int4 req = __ldcv(lw_inbox(self, a.L, a.parity, s) + j);  // {i, v, c, off}
      const int64_t lv = (int64_t)req.y - a.lo;
      const bool ok = lv >= 0 && lv < a.n_local && req.z > 0 && req.w >= 0 && req.w + req.z <= a.L.ncap;
      if (!ok) {
        if (lane == 0) latch(a.err, E_STATE);
        continue;
      }
      const int64_t rs = __ldg(a.indptr + lv);
      const int64_t d = __ldg(a.indptr + lv + 1) - rs;
      char *req_base = a.peers.base[s];
      int32_t *rows = lw_ret_rows(req_base, a.L, a.parity) + req.w;
      const int k = req.z;
      if (d <= k) {  // the whole row (no draw)
        for (int t = lane; t < d; t += 32) rows[t] = __ldg(a.indices + rs + t);
        if (lane == 0) lw_ret_cnt(req_base, a.L, a.parity)[req.x] = (int32_t)d;
      } else if (k <= 32) {
        bool valid;
        int slot, cnt;
        int32_t u;
        sample_node<32>(true, req.y, rs, d, k, a.layer, a.key, a.indices, &valid, &slot, &u, &cnt);
        if (valid) rows[slot] = u;
        if (lane == 0) lw_ret_cnt(req_base, a.L, a.parity)[req.x] = cnt;
      } else if (lane == 0) {  // 32 < c < deg: a block of k_lw_sample_big
        const uint32_t b = atomicAdd(&a.hdr->lw_big, 1u);
        if (b < (uint32_t)a.w.big_cap) a.w.big[b] = make_int2(s, j);
        else latch(a.err, E_CAP);
      }
    }
  }
  if (!PERS && a.sys) __threadfence_system();  // this kernel's peer stores, before k_lw_sample_big's flags
}

// Tasks with 32 < c < deg: Floyd over c draws with a shared-memory hash set.
// Dynamic shared memory: kp (pow2 >= c) positions + 2 kp hash slots.
template <bool PERS>
__device__ __forceinline__ void lw_sample_big_body(const LwArgs &a, int kp_max, int32_t *lw_smem) {
  int32_t *sel = lw_smem;                 // [kp_max]
  int32_t *hkeys = lw_smem + kp_max;      // [2 * kp_max]
  char *self = a.peers.base[a.rank];
  const uint32_t nbig = min(ld_volatile_i32(reinterpret_cast<const int32_t *>(&a.hdr->lw_big)), a.w.big_cap);
  for (uint32_t b = blockIdx.x; b < nbig; b += gridDim.x) {
    const int2 sj = a.w.big[b];
    const int4 req = __ldcv(lw_inbox(self, a.L, a.parity, sj.x) + sj.y);
    const int64_t lv = (int64_t)req.y - a.lo;
    const int64_t rs = __ldg(a.indptr + lv);
    const uint32_t d = (uint32_t)(__ldg(a.indptr + lv + 1) - rs);
    const int k = req.z;
    int kp = 1;
    while (kp < k) kp <<= 1;
    const uint32_t hmask = 2u * (uint32_t)kp - 1u;
    for (int t = threadIdx.x; t < kp; t += LWT)
      sel[t] = t < k ? (int32_t)draw_range(a.key, (uint32_t)t, req.y, a.layer, d - (uint32_t)k + (uint32_t)t + 1u)
                     : 0x7fffffff;
    for (int h = threadIdx.x; h < 2 * kp; h += LWT) hkeys[h] = -1;
    __syncthreads();
    if (threadIdx.x == 0) {  // Floyd's resolution, step by step (R7)
      for (int t = 0; t < k; ++t) {
        int32_t x = sel[t];
        uint32_t h = hash32((uint32_t)x) & hmask;
        while (hkeys[h] != -1 && hkeys[h] != x) h = (h + 1) & hmask;
        if (hkeys[h] == x) {  // taken: j = d - k + t, never chosen before
          x = (int32_t)(d - (uint32_t)k + (uint32_t)t);
          h = hash32((uint32_t)x) & hmask;
          while (hkeys[h] != -1) h = (h + 1) & hmask;
        }
        hkeys[h] = x;
        sel[t] = x;
      }
    }
    __syncthreads();
    for (int size = 2; size <= kp; size <<= 1)  // bitonic sort, ascending
      for (int stride = size >> 1; stride > 0; stride >>= 1) {
        for (int t = threadIdx.x; t < kp; t += LWT) {
          const int p = t ^ stride;
          if (p > t) {
            const bool up = (t & size) == 0;
            const int32_t x = sel[t], y = sel[p];
            if ((x > y) == up) {
              sel[t] = y;
              sel[p] = x;
            }
          }
        }
        __syncthreads();
      }
    char *req_base = a.peers.base[sj.x];
    int32_t *rows = lw_ret_rows(req_base, a.L, a.parity) + req.w;
    for (int t = threadIdx.x; t < k; t += LWT) rows[t] = __ldg(a.indices + rs + sel[t]);
    if (threadIdx.x == 0) lw_ret_cnt(req_base, a.L, a.parity)[req.x] = k;
    __syncthreads();
  }
  if (!PERS && lw_last_block_done(&a.hdr->done, a.sys)) {
    a.hdr->lw_big = 0u;
    for (int s = 0; s < a.bd.world; ++s)
      st_release_flag(lw_ret_flag(a.peers.base[s], a.L, a.parity, a.rank), a.seq, a.sys);
  }
}

// Requester: dst copy + marks, first-occurrence marks of the returned rows.
template <bool PERS>
__device__ __forceinline__ void lw_collect_body(const LwArgs &a) {
  char *self = a.peers.base[a.rank];
  if (!PERS && !wait_flags(lw_ret_flag(self, a.L, a.parity, 0), a.bd.world, a.seq, a.err)) return;
  const uint32_t epoch = a.persist->epoch + 1u + (uint32_t)a.layer;
  const int F = ld_volatile_i32(&a.hdr->F[a.layer]);
  const int Q = a.w.off[F];
  const int32_t *ret_cnt = lw_ret_cnt(self, a.L, a.parity);
  const int32_t *ret_rows = lw_ret_rows(self, a.L, a.parity);
  const int tid = blockIdx.x * blockDim.x + threadIdx.x, nth = gridDim.x * blockDim.x;
  for (int i = tid; i < F; i += nth) {
    const int32_t v = ldw_i32(a.frontier + i);  // written by the previous layer (same kernel when PERS)
    a.out.src_ids[0][i] = v;
    if (v >= 0 && v < a.bd.b[a.bd.world]) mark_dst(a.first, v, i, F, a.layer, epoch, a.err);
  }
  for (int q = tid; q < Q; q += nth) {
    const int i = a.w.slot_node[q];
    if (q - a.w.off[i] < __ldcv(ret_cnt + i)) mark(a.first, __ldcv(ret_rows + q), epoch, (uint32_t)F + (uint32_t)q);
  }
}

// Requester: block l from the marks (one block; Q <= n <= 8192 slots).
__device__ __forceinline__ void lw_finish_body(const LwArgs &a) {
  __shared__ unsigned long long s_u64[33];
  char *self = a.peers.base[a.rank];
  const uint32_t epoch = a.persist->epoch + 1u + (uint32_t)a.layer;
  const int F = ld_volatile_i32(&a.hdr->F[a.layer]);
  const int Q = a.w.off[F];
  const int32_t *ret_cnt = lw_ret_cnt(self, a.L, a.parity);
  const int32_t *ret_rows = lw_ret_rows(self, a.L, a.parity);
  const int tid = threadIdx.x;
  unsigned long long carry = 0;  // (valid, first) counts packed
  for (int b0 = 0; b0 < Q; b0 += LWT) {
    const int q = b0 + tid;
    uint32_t valid = 0, fst = 0;
    if (q < Q) {
      const int i = a.w.slot_node[q];
      if (q - a.w.off[i] < __ldcv(ret_cnt + i)) {
        valid = 1;
        fst = a.first[__ldcv(ret_rows + q)] == mark_word(epoch, (uint32_t)F + (uint32_t)q) ? 1u : 0u;
      }
    }
    unsigned long long tot;
    const unsigned long long ex = carry + block_excl_scan<unsigned long long>(pack2(valid, fst), s_u64, &tot);
    if (q < Q) {
      a.w.excl[q] = (int32_t)(ex & 0x7fffffffull);
      a.w.newid[q] = (int32_t)(ex >> 31);
    }
    carry += tot;
  }
  const int32_t E = (int32_t)(carry & 0x7fffffffull), nnew = (int32_t)(carry >> 31);
  if (tid == 0) a.w.excl[Q] = E;
  __syncthreads();
  for (int q = tid; q < Q; q += LWT) {
    const int i = a.w.slot_node[q];
    if (q - a.w.off[i] >= __ldcv(ret_cnt + i)) continue;
    const int32_t u = __ldcv(ret_rows + q);
    const uint32_t x = mark_x(a.first[u]);
    const int32_t loc = x < (uint32_t)F ? (int32_t)x : F + a.w.newid[x - (uint32_t)F];
    a.out.indices[0][a.w.excl[q]] = loc;
    if (x == (uint32_t)F + (uint32_t)q) a.out.src_ids[0][F + a.w.newid[q]] = u;
  }
  for (int i = tid; i <= F; i += LWT) a.out.indptr[0][i] = a.w.excl[a.w.off[i]];
  if (tid == 0) {
    a.hdr->E[a.layer] = E;
    a.hdr->S[a.layer] = F + nnew;
    a.hdr->F[a.layer + 1] = F + nnew;
    a.hdr->sizes[3 * a.layer + 0] = F;
    a.hdr->sizes[3 * a.layer + 1] = F + nnew;
    a.hdr->sizes[3 * a.layer + 2] = E;
  }
}

// World 1: every layer of the call in ONE cooperative launch (the per-layer
// kernels above are launch- and drain-bound at Table 7's sizes: ~1000 nodes
// per layer).  Phases per layer, separated by grid barriers: allocation
// (block 0), owner-side sampling (one warp per task), tasks with c > 32,
// marks, block construction (block 0).
struct LwPersistArgs {
  LwArgs l[DSP_MAX_LAYERS];
  int32_t L;
  int32_t kp_max;
  WsHeader *hdr;
  WsPersist *persist;       // epoch advanced by the last block
  int32_t gather;           // gather this call's last block (fused call)
  GatherArgs g;
  int32_t prev;             // pipelined: gather the previous call's rows (blocks >= 1, during allocation 0)
  GatherArgs gp;
  int32_t *pend_n;          // pipelined: where this call's row count goes
};

__global__ void __launch_bounds__(LWT, 1) k_lw_persistent(const __grid_constant__ LwPersistArgs p) {
  extern __shared__ unsigned long long lw_dyn[];
  uint32_t bar = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) p.hdr->t[0] = globaltimer_ns();
  for (int l = 0; l < p.L; ++l) {
    const LwArgs &a = p.l[l];
    if (blockIdx.x == 0)
      lw_alloc_body<true>(a, lw_dyn);
    else if (l == 0 && p.prev)  // the other blocks gather the previous pipelined call's rows meanwhile
      phase_gather<GATHER_UNROLL>(p.gp, ld_volatile_i32(p.gp.n_dev), (blockIdx.x - 1) * (int64_t)LWT + threadIdx.x,
                                  (gridDim.x - 1) * (int64_t)LWT);
    grid_barrier<LWT>(p.hdr, bar);
    lw_sample_remote_body<true>(a);
    grid_barrier<LWT>(p.hdr, bar);
    lw_sample_big_body<true>(a, p.kp_max, reinterpret_cast<int32_t *>(lw_dyn));
    grid_barrier<LWT>(p.hdr, bar);
    if (blockIdx.x == 0 && threadIdx.x == 0) p.hdr->lw_big = 0u;
    lw_collect_body<true>(a);
    grid_barrier<LWT>(p.hdr, bar);
    if (blockIdx.x == 0) lw_finish_body(a);
    grid_barrier<LWT>(p.hdr, bar);
  }
  const int32_t S = ld_volatile_i32(&p.hdr->S[p.L - 1]);
  if (p.prev && gridDim.x == 1)  // no spare block during allocation 0
    phase_gather<GATHER_UNROLL>(p.gp, ld_volatile_i32(p.gp.n_dev), threadIdx.x, LWT);
  if (p.gather) phase_gather<GATHER_UNROLL>(p.g, S, blockIdx.x * (int64_t)LWT + threadIdx.x, gridDim.x * (int64_t)LWT);
  if (p.pend_n && blockIdx.x == 0 && threadIdx.x == 0) *p.pend_n = S;
  __syncthreads();
  if (threadIdx.x == 0) {  // the last block advances the workspace epoch (k_epoch_advance of the staged path)
    __threadfence();
    if (atomicAdd(&p.hdr->done, 1u) == gridDim.x - 1) {
      p.persist->epoch += (uint32_t)p.L;
      p.hdr->done = 0u;
    }
  }
}

// World > 1: every layer of the call in ONE cooperative launch per rank; the
// phases keep the flag protocol of the per-stage kernels (the requests and the
// sampled rows cross GPUs through the peer-mapped exchange region), with grid
// barriers where a stage used to end at a kernel boundary.  Every rank's kernel
// is resident on its own GPU (virtual ranks: 1/P of the SMs each), so waiting
// on a peer's flag inside the kernel is safe; waits are bounded (wait_flags).
__global__ void __launch_bounds__(LWT, 1) k_lw_multi(const __grid_constant__ LwPersistArgs p) {
  extern __shared__ unsigned long long lw_dyn[];
  uint32_t bar = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) p.hdr->t[0] = globaltimer_ns();
  for (int l = 0; l < p.L; ++l) {
    const LwArgs &a = p.l[l];
    if (blockIdx.x == 0)  // Eq. 2 allocation, tasks pushed to the owners + inbox flags
      lw_alloc_body<false>(a, lw_dyn);
    else if (l == 0 && p.prev)  // meanwhile the other blocks gather the previous pipelined call's rows
      phase_gather<GATHER_UNROLL>(p.gp, ld_volatile_i32(p.gp.n_dev), (blockIdx.x - 1) * (int64_t)LWT + threadIdx.x,
                                  (gridDim.x - 1) * (int64_t)LWT);
    lw_sample_remote_body<false>(a);  // waits for every rank's tasks
    grid_barrier<LWT>(p.hdr, bar);    // every task with c > 32 queued
    lw_sample_big_body<false>(a, p.kp_max, reinterpret_cast<int32_t *>(lw_dyn));  // then the return flags
    lw_collect_body<false>(a);        // waits for every owner's rows
    grid_barrier<LWT>(p.hdr, bar);
    if (blockIdx.x == 0) lw_finish_body(a);
    grid_barrier<LWT>(p.hdr, bar);
  }
  const int32_t S = ld_volatile_i32(&p.hdr->S[p.L - 1]);
  if (p.prev && gridDim.x == 1) phase_gather<GATHER_UNROLL>(p.gp, ld_volatile_i32(p.gp.n_dev), threadIdx.x, LWT);
  if (p.gather) phase_gather<GATHER_UNROLL>(p.g, S, blockIdx.x * (int64_t)LWT + threadIdx.x, gridDim.x * (int64_t)LWT);
  if (p.pend_n && blockIdx.x == 0 && threadIdx.x == 0) *p.pend_n = S;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&p.hdr->done, 1u) == gridDim.x - 1) {
      p.persist->epoch += (uint32_t)p.L;
      p.hdr->done = 0u;
    }
  }
}

}  // namespace dsp
