// dsp_kernels.cuh -- CSP layer phases and the feature gather (sm_100a).
//
// Phases of one layer l:
//   sample  : world == 1: sample every frontier node, record the sampled
//             neighbour of each edge slot and mark dst / src in the relabel
//             map (fused).  world > 1: bucket scatter -> sample at the owner ->
//             unpermute + mark (exchange through NVLink peer memory)
//   scan    : prefix over edge slots: block indptr, first occurrences, new
//             local ids, src_ids
//   indices : local src id of every edge
// and the gather of the last block's src_ids.
//
// Relabel map: first[p][u] for every global id u, a
// 64-bit word (epoch << 32) | ~x where x is the smallest "order key" marked
// for u in this layer: the dst index i (< F) or F + q for edge slot q.  One
// fire-and-forget atomicMax per mark (no return value, no probing); a newer
// epoch beats every stale word, so the map is never cleared.  Edge slots are
// ordered exactly as the output edges (dst index, then row position), so
// "x == F + q" identifies the first occurrence of a new src node.
//
// world == 1 runs the whole call in ONE persistent cooperative kernel
// (k_csp_persistent, one 1024-thread block per SM) with grid barriers between
// phases; world > 1 runs it in one persistent kernel per rank as well
// (k_csp_multi, dsp_multi.cuh), the exchanges done inside it through peer
// memory.
//
// Data a phase reads after another phase of the same kernel wrote it is read
// with plain (weak) loads after the grid barrier's release/acquire, never
// through the non-coherent path.
#pragma once
#include "dsp_device.cuh"

namespace dsp {

// Inlining of the phase bodies into the persistent kernels.  DSP_PHASE_NOINLINE
// (experiment build) compiles each phase as its own function, so the code a
// phase runs stays contiguous (instruction-cache footprint of the huge kernels).
#ifdef DSP_PHASE_NOINLINE
#define DSP_PHASE __noinline__
#else
#define DSP_PHASE __forceinline__
#endif

constexpr int NT = 256;    // threads per block of the per-phase kernels
constexpr int PNT = 1024;  // threads per block of the persistent kernel (1 block per SM)
constexpr int MAX_PERSIST_BLOCKS = 1024;

// Persistent part of the workspace (offset 0).  Zero-filled before first use.
struct WsPersist {
  uint32_t epoch;      // last relabel epoch used with this workspace
  int32_t pend_n[2];   // row counts of pipelined calls (alternating), read by the next call / flush
  uint32_t hclear;     // epoch at the last zeroing of the relabel hash table (tags unique within 255)
  uint32_t hmask, hoff; // its layout then (slots - 1, offset in 256-B units)
  uint32_t dwin;       // compact direct map: 1 + the epoch window it was last zeroed for (0 = never)
  uint32_t pad[57];
};

// Compact direct map (4 B per node and parity, the node-wise default when the
// graph is small enough for a direct map): word = tag(8) | ~x(24), tag = the
// epoch's position in its window of 255 epochs, so tags grow monotonically
// within a window and the fire-and-forget max keeps working.  A call never
// straddles two windows (its first epoch is moved to the next window's start
// instead) and zeroes the map when it enters a window other than the one of
// the last zeroing (every ~255 / L calls).  x < 2^24 (checked by the host plan).
constexpr uint32_t DWIN = 255u;
// first epoch - 1 of a call of L layers starting after epoch e0 (same window for all L epochs)
__host__ __device__ __forceinline__ uint32_t dwin_start(uint32_t e0, uint32_t L) {
  return (e0 % DWIN) + L > DWIN ? (e0 / DWIN + 1u) * DWIN : e0;
}
__device__ __forceinline__ uint32_t dtag(uint32_t epoch) { return epoch - DWIN * ((epoch - 1u) / DWIN); }
__device__ __forceinline__ uint32_t dword(uint32_t epoch, uint32_t x) { return (dtag(epoch) << 24) | (0xffffffu - x); }
__device__ __forceinline__ bool dclear_due(const WsPersist *ps, uint32_t e0s) {
  return *(volatile const uint32_t *)&ps->dwin != e0s / DWIN + 1u;
}

// A call using epochs (e0, e0 + L] must first zero the hash table when a tag
// could repeat (every word alive was written after the last zeroing) or when
// the table sits elsewhere than at the last zeroing (a plan of another size).
__device__ __forceinline__ uint32_t hash_off(const WsPersist *ps, const unsigned long long *first) {
  return (uint32_t)((reinterpret_cast<const char *>(first) - reinterpret_cast<const char *>(ps)) >> 8);
}
__device__ __forceinline__ bool hash_clear_due(const WsPersist *ps, uint32_t e0, uint32_t L, uint32_t mask,
                                               const unsigned long long *first) {
  if (!mask) return false;
  const volatile WsPersist *v = ps;
  return e0 + L >= v->hclear + 255u || v->hmask != mask || v->hoff != hash_off(ps, first);
}
__device__ __forceinline__ void hash_cleared(WsPersist *ps, uint32_t e0, uint32_t mask,
                                             const unsigned long long *first) {
  ps->hclear = e0;
  ps->hmask = mask;
  ps->hoff = hash_off(ps, first);
}

// Per-call state (memset to 0 by the host before every call).
struct WsHeader {
  int32_t F[9];          // frontier size per layer (F[0] = num_seeds)
  int32_t S[8];          // num_src per layer
  int64_t E[8];          // num_edges per layer
  int64_t sizes[24];     // {num_dst, num_src, num_edges} per layer, for async callers
  uint32_t done;         // last-block counter
  uint32_t bucket[8];    // per-owner send counters (bucket scatter)
  uint32_t bar_count;    // grid barrier arrivals
  uint32_t unused0;
  uint32_t chunks_loader, chunks_helper;  // gather chunks done by loader / sampling warps
  uint32_t lw_big;       // layer-wise tasks with 32 < c < deg (owner side)
  int32_t abort_wait;    // world > 1 persistent call: a wait timed out, later waits end at once
  uint32_t pad[1];
  unsigned long long t[24];   // %globaltimer at kernel start and when block 0 leaves each grid barrier
  unsigned long long ta[24];  // %globaltimer when block 0 arrives at each grid barrier
  unsigned long long dbg[32]; // debug stamps (DSP_DEBUG_STAMPS builds only)
  uint32_t scursor[8];        // biased sampling: next frontier node to claim, per layer
  unsigned long long gcur;    // pipelined gather claims: rows taken from the front (low 32) | from the back (high 32)
};

// One parity (layer % 2) of the workspace.
struct LayerBufs {
  int32_t *cnt;                 // [F] sampled count per frontier node
  int32_t *rows;                // [F*k] sampled neighbour (global id) of edge slot q = i*k + slot
  unsigned long long *first;    // relabel map: [N] direct words, or [mask + 1] hash slots
  uint32_t mask;                // 0: direct map indexed by global id; else hash table of mask + 1 slots
  uint32_t *first32;            // compact direct map [N] (tag | ~x words), or nullptr
  uint32_t n32;                 // its length (N)
};

struct Outputs {
  int32_t *indptr[8];
  int32_t *indices[8];
  int32_t *src_ids[8];
};

__device__ __forceinline__ int ldcg_i32(const int32_t *p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ldcg_u64(const unsigned long long *p) { return __ldcg(p); }
// Weak load of data written earlier in the same kernel by other blocks and
// published by a grid barrier (release / acquire): may be served by L1,
// never through the non-coherent path.
__device__ __forceinline__ int ldw_i32(const int32_t *p) { return *p; }
__device__ __forceinline__ unsigned long long ldw_u64(const unsigned long long *p) { return *p; }
__device__ __forceinline__ int ld_volatile_i32(const int32_t *p) { return *(volatile const int32_t *)p; }
__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
  return *(volatile const unsigned long long *)p;
}

// ------------------------------------------------------------ relabel map
__device__ __forceinline__ unsigned long long mark_word(uint32_t epoch, uint32_t x) {
  return ((unsigned long long)epoch << 32) | (0xffffffffu - x);
}
// x of a word of the current epoch
__device__ __forceinline__ uint32_t mark_x(unsigned long long w) { return 0xffffffffu - (uint32_t)w; }
// Every access to the map carries an L2 evict_last policy: the map (8 B per
// node and parity) is touched at random ~2 times per sampled edge, and
// without the hint the adjacency reads and the gather's stream push it out of
// L2, turning each mark into a DRAM read + write-back.
__device__ __forceinline__ unsigned long long map_policy() { return l2_policy_evict_last(); }
__device__ __forceinline__ void map_red_max(unsigned long long *p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.max.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(map_policy())
               : "memory");
}
__device__ __forceinline__ unsigned long long map_atom_max(unsigned long long *p, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.relaxed.gpu.global.max.L2::cache_hint.u64 %0, [%1], %2, %3;"
               : "=l"(old) : "l"(p), "l"(v), "l"(map_policy()) : "memory");
  return old;
}
// weak load / store (ordered by the grid barriers or kernel boundaries)
__device__ __forceinline__ unsigned long long map_ld(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(map_policy()));
  return v;
}
__device__ __forceinline__ void map_st(unsigned long long *p, unsigned long long v) {
  asm volatile("st.global.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(map_policy()) : "memory");
}
__device__ __forceinline__ void mark(unsigned long long *first, int32_t u, uint32_t epoch, uint32_t x) {
  map_red_max(first + u, mark_word(epoch, x));
}
__device__ __forceinline__ void map32_red_max(uint32_t *p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.max.L2::cache_hint.u32 [%0], %1, %2;" ::"l"(p), "r"(v), "l"(map_policy())
               : "memory");
}
__device__ __forceinline__ uint32_t map32_atom_max(uint32_t *p, uint32_t v) {
  uint32_t old;
  asm volatile("atom.relaxed.gpu.global.max.L2::cache_hint.u32 %0, [%1], %2, %3;"
               : "=r"(old) : "l"(p), "r"(v), "l"(map_policy()) : "memory");
  return old;
}
__device__ __forceinline__ uint32_t map32_ld(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(map_policy()));
  return v;
}
__device__ __forceinline__ void map32_st(uint32_t *p, uint32_t v) {
  asm volatile("st.global.L2::cache_hint.u32 [%0], %1, %2;" ::"l"(p), "r"(v), "l"(map_policy()) : "memory");
}

// ------------------------------------------ relabel hash table (large N)
// For graphs whose direct map (8 B per node and parity) cannot stay in L2,
// the map is an open-addressing table sized to the batch (the north star's
// "GPU hash table"): slot word = tag(8) | key(31) | ~x(25),
// tag = epoch % 255 + 1 (0 = never used).  A key is claimed with a CAS on a
// slot whose tag is not the current one, then lowered with the same
// fire-and-forget max as the direct map (equal high bits: the max keeps the
// smallest x).  Linear probing from hash32(key); the table is zeroed when the
// epoch crosses a multiple of 255, so a tag is never reused while a word
// carrying it is alive.  x < 2^25 (checked by the host plan).
__device__ __forceinline__ uint32_t htag(uint32_t epoch) { return epoch % 255u + 1u; }
__device__ __forceinline__ unsigned long long hword(uint32_t epoch, int32_t u, uint32_t x) {
  return ((unsigned long long)htag(epoch) << 56) | ((unsigned long long)(uint32_t)u << 25) |
         (unsigned long long)(0x1ffffffu - x);
}
// word of (epoch, key, x) in the layout of B
__device__ __forceinline__ unsigned long long mword(const LayerBufs &B, uint32_t epoch, int32_t u, uint32_t x) {
  return B.first32 ? (unsigned long long)dword(epoch, x) : B.mask ? hword(epoch, u, x) : mark_word(epoch, x);
}
// x of a word of the current epoch
__device__ __forceinline__ uint32_t mword_x(const LayerBufs &B, unsigned long long w) {
  return B.first32 ? 0xffffffu - (uint32_t)(w & 0xffffffull)
         : B.mask  ? 0x1ffffffu - (uint32_t)(w & 0x1ffffffull)
                   : mark_x(w);
}
// claims (or finds) the slot of key u; returns its word pointer and the word seen there.
// Out of line (like map_find): the probing loops stay out of the hot inlined code of
// the direct-map layouts (instruction-cache footprint of the persistent kernels).
__device__ __noinline__ unsigned long long *hash_claim(const LayerBufs &B, int32_t u, uint32_t epoch, uint32_t x,
                                                        unsigned long long *seen) {
  const unsigned long long want = hword(epoch, u, x), hi = want >> 25;
  const unsigned long long tag = (unsigned long long)htag(epoch);
  uint32_t h = hash32((uint32_t)u) & B.mask;
  while (true) {
    unsigned long long *p = B.first + h;
    unsigned long long w = map_ld(p);
    if ((w >> 56) != tag) {  // free in this epoch: claim it
      const unsigned long long old = atomicCAS(p, w, want);
      if (old == w) {
        *seen = 0ull;
        return p;
      }
      w = old;
      if ((w >> 56) != tag) continue;  // still another epoch's word: retry this slot
    }
    if ((w >> 25) == hi) {
      *seen = w;
      return p;
    }
    h = (h + 1u) & B.mask;
  }
}
// slot of key u (inserted earlier in this epoch); 64-bit layouts only
__device__ __noinline__ unsigned long long *map_find_hashed(const LayerBufs &B, int32_t u, uint32_t epoch) {
  const unsigned long long hi = ((unsigned long long)htag(epoch) << 31) | (uint32_t)u;
  uint32_t h = hash32((uint32_t)u) & B.mask;
  while ((map_ld(B.first + h) >> 25) != hi) h = (h + 1u) & B.mask;
  return B.first + h;
}
__device__ __forceinline__ unsigned long long *map_find(const LayerBufs &B, int32_t u, uint32_t epoch) {
  if (!B.mask) return B.first + u;
  return map_find_hashed(B, u, epoch);
}
// the word of key u (marked earlier in this epoch), compared with mword()
__device__ __forceinline__ unsigned long long map_get(const LayerBufs &B, int32_t u, uint32_t epoch) {
  if (B.first32) return (unsigned long long)map32_ld(B.first32 + u);
  return map_ld(map_find(B, u, epoch));
}
// overwrite the word of key u (marked earlier in this epoch) with x
__device__ __forceinline__ void map_put(const LayerBufs &B, int32_t u, uint32_t epoch, uint32_t x) {
  if (B.first32) {
    map32_st(B.first32 + u, dword(epoch, x));
    return;
  }
  map_st(map_find(B, u, epoch), mword(B, epoch, u, x));
}
// zero the relabel map in use (hash table or compact direct map; one map
// serves every layer of a node-wise call)
__device__ __forceinline__ void map_zero(const LayerBufs &B, int64_t tid, int64_t nthreads) {
  if (B.first32) {
    for (int64_t i = tid; i < (int64_t)B.n32; i += nthreads) B.first32[i] = 0u;
  } else if (B.mask) {
    for (int64_t i = tid; i <= (int64_t)B.mask; i += nthreads) B.first[i] = 0ull;
  }
}
__device__ __forceinline__ void mark(const LayerBufs &B, int32_t u, uint32_t epoch, uint32_t x) {
  if (B.first32) {
    map32_red_max(B.first32 + u, dword(epoch, x));
    return;
  }
  if (!B.mask) {
    map_red_max(B.first + u, mark_word(epoch, x));
    return;
  }
  unsigned long long seen;
  unsigned long long *p = hash_claim(B, u, epoch, x, &seen);
  if (seen) map_red_max(p, hword(epoch, u, x));
}

// q / k for a fixed small divisor k: one 64-bit multiply-high with
// m = ceil(2^64 / k), exact for q < 2^59 (m = 0 encodes k = 1).
struct FastDiv {
  unsigned long long m;
  uint32_t k;
};
__host__ __device__ __forceinline__ FastDiv make_fastdiv(uint32_t k) {
  FastDiv f;
  f.k = k;
  f.m = k <= 1 ? 0ull : (~0ull / k) + 1ull;
  return f;
}
__device__ __forceinline__ uint32_t fdiv(uint64_t q, const FastDiv &f) {
  return f.m ? (uint32_t)__umul64hi(q, f.m) : (uint32_t)q;
}

#ifdef DSP_DEBUG_STAMPS
// stamp idx once VAL is available (thread 0 of block 0, first iteration)
#define DSTAMP(hdr, idx, VAL, layer)                                                   \
  do {                                                                                 \
    if (blockIdx.x == 0 && threadIdx.x == 0 && dbg_first && (VAL) != 0x7fffffff)       \
      (hdr)->dbg[(layer) * 8 + (idx)] = globaltimer_ns();                              \
  } while (0)
#else
#define DSTAMP(hdr, idx, VAL, layer) \
  do {                               \
  } while (0)
#endif

// Items [0, total) of a phase: each block takes one contiguous chunk of
// ceil(total / nblocks) (small layers spread over every SM instead of
// filling the first blocks), threads stride inside it.
struct Span {
  int64_t end, first, step;
};
// The threads of a persistent block that run the sampling phases ("team"):
// the whole block, or all but the loader warps of a pipelined launch.
template <int TEAM>
__device__ __forceinline__ void team_sync() {
  if (TEAM == PNT)
    __syncthreads();
  else
    asm volatile("bar.sync 1, %0;" ::"n"(TEAM) : "memory");
}
template <int TEAM = PNT>
__device__ __forceinline__ Span block_span(int64_t total) {
  const int64_t chunk = (total + gridDim.x - 1) / gridDim.x;
  const int64_t b = min(total, (int64_t)blockIdx.x * chunk);
  const int64_t e = min(total, b + chunk);
  return Span{e, b + threadIdx.x, (int64_t)TEAM};
}
__device__ __forceinline__ Span grid_span(int64_t total) {
  return Span{total, (int64_t)blockIdx.x * blockDim.x + threadIdx.x, (int64_t)gridDim.x * blockDim.x};
}

// ------------------------------------------------------------ grid barrier
__device__ __forceinline__ void red_add_release_gpu(uint32_t *p, uint32_t v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_gpu_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Grid barrier for the persistent kernel (all blocks co-resident through the
// cooperative launch).  hdr->bar_count is a monotonic arrival counter zeroed
// by the host before the launch; each block tracks the target in a register.
// bar.sync orders the block's writes before thread 0's release reduction (no
// return value, so no extra round trip); pollers acquire.  1.25 us at 148
// blocks, vs 2.5 us for an atomicAdd + generation barrier over 592 blocks
// (tools/micro/barrier_bench.cu).
// SYS: thread 0 also issues a system-scope fence after the block barrier, so
// every store of the block (peer memory included) is ordered before its
// arrival (cumulativity through bar.sync), and a flag released at system scope
// after the barrier publishes them to other GPUs.
template <int TEAM = PNT, bool SYS = false>
__device__ __forceinline__ void grid_barrier(WsHeader *hdr, uint32_t &target) {
  team_sync<TEAM>();
  target += gridDim.x;
  if (threadIdx.x == 0) {
    if (SYS) __threadfence_system();
    const uint32_t g = target / gridDim.x;
    if (blockIdx.x == 0 && g < 23u) hdr->ta[g] = globaltimer_ns();
    red_add_release_gpu(&hdr->bar_count, 1u);
    while (ld_acquire_gpu_u32(&hdr->bar_count) < target) {
    }
    if (blockIdx.x == 0 && g < 23u) hdr->t[g] = globaltimer_ns();
  }
  team_sync<TEAM>();
}

// ---------------------------------------------------------------- sampling
// Marks of one frontier node (dst, index i) and its sampled edges.  At
// layer 0 the dst mark returns the previous word: another dst of the same
// epoch there means a duplicate seed.
__device__ __forceinline__ void mark_dst(unsigned long long *first, int32_t v, int i, int F, int layer,
                                         uint32_t epoch, int *err) {
  if (layer == 0) {
    const unsigned long long old = map_atom_max(first + v, mark_word(epoch, (uint32_t)i));
    if ((uint32_t)(old >> 32) == epoch && mark_x(old) < (uint32_t)F) latch(err, E_DUP);
  } else {
    mark(first, v, epoch, (uint32_t)i);
  }
}
__device__ __forceinline__ void mark_dst(const LayerBufs &B, int32_t v, int i, int F, int layer, uint32_t epoch,
                                         int *err) {
  if (B.first32) {
    const uint32_t w = dword(epoch, (uint32_t)i);
    if (layer == 0) {
      const uint32_t old = map32_atom_max(B.first32 + v, w);
      if ((old >> 24) == (w >> 24) && 0xffffffu - (old & 0xffffffu) < (uint32_t)F) latch(err, E_DUP);
    } else {
      map32_red_max(B.first32 + v, w);
    }
    return;
  }
  if (!B.mask) {
    mark_dst(B.first, v, i, F, layer, epoch, err);
    return;
  }
  unsigned long long seen;
  unsigned long long *p = hash_claim(B, v, epoch, (uint32_t)i, &seen);
  if (!seen) return;
  if (layer == 0) {  // atomic: of two equal seeds the later sees the earlier's dst index
    const unsigned long long old = map_atom_max(p, hword(epoch, v, (uint32_t)i));
    if (mword_x(B, old) < (uint32_t)F) latch(err, E_DUP);
  } else {
    map_red_max(p, hword(epoch, v, (uint32_t)i));
  }
}

// Lane-group sampling (G lanes per node, G = next pow2 >= k): the draws run
// on separate lanes, Floyd's resolution and the ranking via shuffles
// (sample_node).  Used for k > 16.
template <int G, int TEAM = PNT>
__device__ DSP_PHASE void phase_sample_lanes(const int32_t *frontier, int F, int layer, int k, uint2 key,
                                                   const int64_t *__restrict__ indptr,
                                                   const int32_t *__restrict__ indices, int64_t lo,
                                                   int64_t n_local, const LayerBufs &B, uint32_t epoch,
                                                   int32_t *src_out, int *err, WsHeader *hdr) {
  constexpr int NPW = 32 / G;  // nodes per warp-iteration
  const int lane = threadIdx.x & 31;
  const bool leader = (lane & (G - 1)) == 0;
  const Span sp = block_span<TEAM>(F);
  const int64_t b0 = sp.first - threadIdx.x;  // first node of this block's chunk
  const int wib = threadIdx.x >> 5, wpb = TEAM >> 5;
  bool dbg_first = true;
  (void)hdr;
  for (int64_t base = b0 + (int64_t)wib * NPW; base < sp.end; base += (int64_t)wpb * NPW) {
    const int i = (int)(base + lane / G);
    const bool active = i < sp.end;
    DSTAMP(hdr, 0, 0, layer);
    const int32_t v = active ? ldw_i32(frontier + i) : 0;
    DSTAMP(hdr, 1, v, layer);
    const int64_t lv = (int64_t)v - lo;
    const bool ok = active && v >= 0 && lv >= 0 && lv < n_local;
    int64_t s = 0, d = 0;
    if (ok) {
      row_extent(indptr, lv, &s, &d);
    }
    DSTAMP(hdr, 2, (int)d, layer);
    bool valid;
    int slot, cnt;
    int32_t u;
    sample_node<G>(ok, v, s, d, k, layer, key, indices, &valid, &slot, &u, &cnt);
    DSTAMP(hdr, 3, u, layer);
    if (active && leader) {
      B.cnt[i] = cnt;
      if (src_out) src_out[i] = v;  // dst copy (R17)
      if (ok)
        mark_dst(B, v, i, F, layer, epoch, err);
      else
        latch(err, E_RANGE);
    }
    if (valid) {
      const uint32_t q = (uint32_t)i * (uint32_t)k + (uint32_t)slot;
      B.rows[q] = u;
      mark(B, u, epoch, (uint32_t)F + q);
    }
    DSTAMP(hdr, 5, 0, layer);
    dbg_first = false;
  }
}

// Thread-per-node sampling for k <= KB: the draws, Floyd's resolution and the
// ranking run in one thread's registers; the k adjacency loads and the k + 1
// marks are issued back to back (memory-level parallelism k per thread, every
// frontier node in flight at once).
template <int KB, int TEAM = PNT>
__device__ DSP_PHASE void phase_sample_tpn(const int32_t *frontier, int F, int layer, int k, uint2 key,
                                                 const int64_t *__restrict__ indptr,
                                                 const int32_t *__restrict__ indices, int64_t lo,
                                                 int64_t n_local, const LayerBufs &B, uint32_t epoch,
                                                 int32_t *src_out, int *err, WsHeader *hdr) {
  const Span sp = block_span<TEAM>(F);
  bool dbg_first = true;
  (void)hdr;
  for (int64_t ii = sp.first; ii < sp.end; ii += sp.step) {
    const int i = (int)ii;
    DSTAMP(hdr, 0, 0, layer);
    const int32_t v = ldw_i32(frontier + i);
    DSTAMP(hdr, 1, v, layer);
    if (src_out) src_out[i] = v;  // dst copy (R17)
    const int64_t lv = (int64_t)v - lo;
    if (v < 0 || lv < 0 || lv >= n_local) {
      latch(err, E_RANGE);
      B.cnt[i] = 0;
      continue;
    }
    int64_t rs, d;
    row_extent(indptr, lv, &rs, &d);
    DSTAMP(hdr, 2, (int)d, layer);
    const bool full = d <= k;
    const int cnt = full ? (int)d : k;
    uint32_t pos[KB];
#pragma unroll
    for (int t = 0; t < KB; ++t) pos[t] = (uint32_t)t;
    if (!full) {
#pragma unroll
      for (int t = 0; t < KB; ++t)
        if (t < k) pos[t] = draw_range(key, (uint32_t)t, v, layer, (uint32_t)(d - k + t + 1));
      // Floyd: step t keeps r_t unless an earlier step chose it, then takes j_t
#pragma unroll
      for (int t = 1; t < KB; ++t) {
        if (t < k) {
          bool hit = false;
#pragma unroll
          for (int q = 0; q < t; ++q) hit |= (pos[q] == pos[t]);
          if (hit) pos[t] = (uint32_t)(d - k + t);
        }
      }
    }
    int32_t u[KB];
    unsigned long long slots = 0;  // 4 bits per position: its rank (slot in ascending row order)
#pragma unroll
    for (int t = 0; t < KB; ++t) {
      uint32_t r = 0;
#pragma unroll
      for (int q = 0; q < KB; ++q) r += (q < cnt && pos[q] < pos[t]) ? 1u : 0u;
      slots |= (unsigned long long)r << (4 * t);
      u[t] = (t < cnt) ? adj_ld(indices + rs + pos[t]) : 0;
    }
    DSTAMP(hdr, 3, u[0] + u[KB - 1], layer);
    B.cnt[i] = cnt;
    mark_dst(B, v, i, F, layer, epoch, err);
    const uint32_t q0 = (uint32_t)i * (uint32_t)k;
#pragma unroll
    for (int t = 0; t < KB; ++t) {
      if (t < cnt) {
        const uint32_t q = q0 + (uint32_t)((slots >> (4 * t)) & 15u);
        B.rows[q] = u[t];
        mark(B, u[t], epoch, (uint32_t)F + q);
      }
    }
    DSTAMP(hdr, 5, 0, layer);
    dbg_first = false;
  }
}

// Biased sampling, world 1: warps claim runs of consecutive frontier
// nodes from a per-layer cursor (row lengths of the frontier span three
// orders of magnitude, so a static share leaves warps idle at the grid
// barrier); a claim is about half a warp's even share, at most 32
// nodes.  The ids and row extents of a claim are loaded at once (one per
// lane), then biased_claim samples them: lane groups for rows of <= 256
// positions, the warp-wide sampler for longer ones.
struct BiasedOutW1 {
  const LayerBufs &B;
  int g0, k, F, layer;
  uint32_t epoch;
  int32_t *src_out;
  int *err;
  struct Ctx {
    int i;
  };
  __device__ __forceinline__ Ctx ctx(int jn) const { return Ctx{g0 + jn}; }
  __device__ __forceinline__ void node(const Ctx &c, int32_t v, bool ok, int cnt) const {
    B.cnt[c.i] = cnt;
    if (src_out) src_out[c.i] = v;
    if (ok)
      mark_dst(B, v, c.i, F, layer, epoch, err);
    else
      latch(err, E_RANGE);
  }
  __device__ __forceinline__ void edge(const Ctx &c, int slot, int32_t u) const {
    const uint32_t q = (uint32_t)c.i * (uint32_t)k + (uint32_t)slot;
    B.rows[q] = u;
    mark(B, u, epoch, (uint32_t)F + q);
  }
};

template <int TEAM = PNT>
__device__ DSP_PHASE void phase_sample_biased(const int32_t *frontier, int F, int layer, int k, uint2 key,
                                                    const int64_t *__restrict__ indptr,
                                                    const int32_t *__restrict__ indices,
                                                    const uint32_t *__restrict__ weights, int64_t lo,
                                                    int64_t n_local, const LayerBufs &B, uint32_t epoch,
                                                    int32_t *src_out, int *err, uint32_t *cursor) {
  const int lane = threadIdx.x & 31;
  const int nwarps = (int)gridDim.x * (TEAM >> 5);
  const int csz = max(1, min(32, F / (2 * nwarps)));
#ifdef DSP_BPROF
  unsigned long long *bprof = layer == DSP_BPROF ? reinterpret_cast<unsigned long long *>(cursor - layer) - 32 : nullptr;
  const long long p0 = clock64();
#else
  unsigned long long *bprof = nullptr;
#endif
  while (true) {
    BPROF_T(q0);
    int g0 = 0;
    if (lane == 0) g0 = (int)atomicAdd(cursor, (uint32_t)csz);
    g0 = __shfl_sync(FULL_MASK, g0, 0);
    if (g0 >= F) break;
    const int32_t vl = lane < min(csz, F - g0) ? ldw_i32(frontier + g0 + lane) : -1;
    const int nn = min(csz, F - g0);
    const int64_t lvl = (int64_t)vl - lo;
    const bool okl = lane < nn && vl >= 0 && lvl >= 0 && lvl < n_local;
    int64_t sl = 0, dl = 0;
    if (okl) row_extent(indptr, lvl, &sl, &dl);
    const BiasedOutW1 out{B, g0, k, F, layer, epoch, src_out, err};
    BPROF_T(q1);
    BPROF_ADD(0, q1 - q0);
    BPROF_ADD(9, 1);
    biased_claim(nn, vl, okl, sl, dl, k, layer, key, weights, indices, out, bprof);
  }
#ifdef DSP_BPROF
  BPROF_ADD(10, clock64() - p0);
#endif
}

// ------------------------------------------- scan, two-phase (persistent)
// Inside the persistent kernel every block is resident, so the scan over
// edge slots is a static partition: pass 1 computes each item's flags, the
// per-(stripe, warp) counts and the block aggregate (published to `agg`);
// after a grid barrier pass 2 adds the aggregates of the preceding blocks and
// writes the outputs.  Items are striped (item j of thread t is slot
// tile + j*TEAM + t) so every load is a coalesced warp access; the in-block
// prefix comes from warp ballots plus a table kept in shared memory across
// the barrier, the flags in registers.
constexpr int SCAN2_IPT = 8;     // stripes per group (registers of one pass over them)
constexpr int SCAN2_GROUPS = 4;  // groups per block and round of k_csp_multi: up to 32 stripes of TEAM slots


__device__ __forceinline__ unsigned long long pack2(uint32_t valid, uint32_t first) {
  return ((unsigned long long)first << 31) | valid;
}

template <int TEAM, int GROUPS = 1>
struct Scan2Smem {
  unsigned long long tab[GROUPS * SCAN2_IPT * (TEAM / 32)];  // exclusive prefix of (stripe, warp)
  unsigned long long red[2 * (TEAM / 32) + 2];
};

struct Scan2Regs {
  uint32_t vbits, fbits;  // bit s: slot q0 + s * TEAM holds an edge / is a first occurrence
  int32_t r[SCAN2_IPT];   // GROUPS == 1: the slot's rows[] value after pass 1 (pass 2 reads no memory for it)
};

// A block's chunk [tile0, tile_end) of one round is processed as up to
// GROUPS groups of SCAN2_IPT stripes (stripe s = slots tile0 + s * TEAM +
// [0, TEAM)), so a layer of up to GROUPS * 8 * TEAM slots per block needs one
// round (two grid barriers) instead of one round per 8 stripes.  The world-1
// kernel keeps GROUPS = 1 (the bench step is bound by the gather there, and
// its sampling warps finishing earlier only add DRAM contention: 0.1356 vs
// 0.1345 ms/step over 5 alternating runs); k_csp_multi, whose ranks run on
// fractions of the SMs, uses 4 (virtual P = 2 / 4 with 4 channels: 73.3 /
// 76.4 vs 77.5 / 80.0 us per rank-batch).
template <int TEAM, int GROUPS = 1>
__device__ __forceinline__ void scan2_pass1(int F, int k, const LayerBufs &B, uint32_t epoch, int64_t tile0,
                                            int64_t tile_end, Scan2Regs &R, unsigned long long *agg_slot,
                                            Scan2Smem<TEAM, GROUPS> &sm) {
  constexpr int W = TEAM / 32;
  const uint32_t total = (uint32_t)tile_end;  // < 2^31 by the host's plan check
  const FastDiv fd = make_fastdiv((uint32_t)k);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int groups = (int)min((int64_t)GROUPS,
                              max((int64_t)1, (tile_end - tile0 + (int64_t)TEAM * SCAN2_IPT - 1) / ((int64_t)TEAM * SCAN2_IPT)));
  R.vbits = R.fbits = 0;
#pragma unroll 1
  for (int g = 0; g < groups; ++g) {
    const uint32_t q0 = (uint32_t)tile0 + (uint32_t)(g * SCAN2_IPT * TEAM) + threadIdx.x;
    // all loads first: counts + sampled ids, then the map words of the valid slots
    int32_t c[SCAN2_IPT], u[SCAN2_IPT];
#pragma unroll
    for (int j = 0; j < SCAN2_IPT; ++j) {
      const uint32_t q = q0 + j * TEAM;
      c[j] = -1;
      u[j] = 0;
      if (q < total) {
        const uint32_t i = fdiv(q, fd);
        c[j] = ldw_i32(B.cnt + i) - (int32_t)(q - i * (uint32_t)k);  // > 0 iff slot q holds an edge
        u[j] = ldw_i32(B.rows + q);  // garbage unless valid; dereferenced only then
      }
    }
    unsigned long long w[SCAN2_IPT];
#pragma unroll
    for (int j = 0; j < SCAN2_IPT; ++j) w[j] = c[j] > 0 ? map_get(B, u[j], epoch) : 0ull;
#pragma unroll
    for (int j = 0; j < SCAN2_IPT; ++j) {
      const bool valid = c[j] > 0;
      const bool first = valid && w[j] == mword(B, epoch, u[j], (uint32_t)F + q0 + j * TEAM);
      // a valid slot that is not u's first occurrence keeps x (u's smallest order
      // key: its dst index, or F + the slot of its first occurrence) as -1 - x
      const int32_t rv = valid && !first ? -1 - (int32_t)mword_x(B, w[j]) : u[j];
      if (valid && !first) B.rows[q0 + j * TEAM] = rv;
      if (GROUPS == 1) R.r[j] = rv;
      R.vbits |= (valid ? 1u : 0u) << (g * SCAN2_IPT + j);
      R.fbits |= (first ? 1u : 0u) << (g * SCAN2_IPT + j);
      const uint32_t bv = __ballot_sync(FULL_MASK, valid), bf = __ballot_sync(FULL_MASK, first);
      if (lane == 0) sm.tab[(g * SCAN2_IPT + j) * W + wid] = pack2(__popc(bv), __popc(bf));
    }
  }
  team_sync<TEAM>();
  if (wid == 0) {  // exclusive scan of the (stripe, warp) counts, stripe-major, group by group
    constexpr int PER = (SCAN2_IPT * W + 31) / 32;  // entries per lane (the last lanes' tail may be empty)
    unsigned long long carry = 0;
#pragma unroll 1
    for (int g = 0; g < groups; ++g) {
      unsigned long long *tab = sm.tab + g * SCAN2_IPT * W;
      unsigned long long v[PER], run = 0;
#pragma unroll
      for (int e = 0; e < PER; ++e) {
        v[e] = lane * PER + e < SCAN2_IPT * W ? tab[lane * PER + e] : 0ull;
        run += v[e];
      }
      unsigned long long incl = run;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL_MASK, incl, off);
        if (lane >= off) incl += y;
      }
      unsigned long long p = carry + incl - run;
#pragma unroll
      for (int e = 0; e < PER; ++e) {
        if (lane * PER + e < SCAN2_IPT * W) tab[lane * PER + e] = p;
        p += v[e];
      }
      carry += __shfl_sync(FULL_MASK, incl, 31);
    }
    if (lane == 0) __stcg(agg_slot, carry);
  }
  team_sync<TEAM>();
}

// prefix of block `blk` and the round total from the published aggregates
template <int TEAM, int GROUPS = 1>
__device__ __forceinline__ void scan2_prefix(const unsigned long long *agg, int nblk, int blk, Scan2Smem<TEAM, GROUPS> &sm,
                                             unsigned long long *prefix, unsigned long long *round_total) {
  unsigned long long p = 0, t = 0;
  for (int b = threadIdx.x; b < nblk; b += TEAM) {
    const unsigned long long x = __ldcg(agg + b);
    t += x;
    if (b < blk) p += x;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    p += __shfl_xor_sync(FULL_MASK, p, off);
    t += __shfl_xor_sync(FULL_MASK, t, off);
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) {
    sm.red[wid] = p;
    sm.red[TEAM / 32 + wid] = t;
  }
  team_sync<TEAM>();
  if (threadIdx.x == 0) {
    unsigned long long pp = 0, tt = 0;
    for (int w = 0; w < TEAM / 32; ++w) {
      pp += sm.red[w];
      tt += sm.red[TEAM / 32 + w];
    }
    sm.red[2 * (TEAM / 32)] = pp;
    sm.red[2 * (TEAM / 32) + 1] = tt;
  }
  team_sync<TEAM>();
  *prefix = sm.red[2 * (TEAM / 32)];
  *round_total = sm.red[2 * (TEAM / 32) + 1];
  team_sync<TEAM>();
}

// Block indptr at t == 0 slots, and the local src id of every edge whose
// answer is known here: a first occurrence gets nid = F + rank (src_out[nid] =
// u, and rows[q] := nid for the duplicates), a dst hit its dst index x.  The
// remaining edges (duplicates of a first occurrence elsewhere) are resolved by
// phase_indices_dups after the next grid barrier.  The relabel map is not
// touched: a duplicate finds its nid through rows[x - F], a coalesced-slot
// array, instead of a second random map access per edge.  The dst copy of
// src_out is written by the sample phase.
template <int TEAM, int GROUPS = 1>
__device__ __forceinline__ void scan2_pass2(int F, int k, const LayerBufs &B, int64_t tile0, int64_t tile_end,
                                            const Scan2Regs &R, unsigned long long base,
                                            const Scan2Smem<TEAM, GROUPS> &sm, int32_t *indptr_out,
                                            int32_t *indices_out, int32_t *src_out) {
  constexpr int W = TEAM / 32;
  const uint32_t total = (uint32_t)tile_end;
  const FastDiv fd = make_fastdiv((uint32_t)k);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const int groups = (int)min((int64_t)GROUPS,
                              max((int64_t)1, (tile_end - tile0 + (int64_t)TEAM * SCAN2_IPT - 1) / ((int64_t)TEAM * SCAN2_IPT)));
#pragma unroll 1
  for (int g = 0; g < groups; ++g) {
    const uint32_t q0 = (uint32_t)tile0 + (uint32_t)(g * SCAN2_IPT * TEAM) + threadIdx.x;
    const uint32_t vb = R.vbits >> (g * SCAN2_IPT), fb = R.fbits >> (g * SCAN2_IPT);
    int32_t r[SCAN2_IPT];
#pragma unroll
    for (int j = 0; j < SCAN2_IPT; ++j)
      r[j] = GROUPS == 1 ? R.r[j] : ((vb >> j) & 1u) ? ldw_i32(B.rows + q0 + j * TEAM) : 0;
#pragma unroll
    for (int j = 0; j < SCAN2_IPT; ++j) {
      const uint32_t bv = __ballot_sync(FULL_MASK, (vb >> j) & 1u);
      const uint32_t bf = __ballot_sync(FULL_MASK, (fb >> j) & 1u);
      const uint32_t q = q0 + j * TEAM;
      if (q < total) {
        const unsigned long long b = base + sm.tab[(g * SCAN2_IPT + j) * W + wid];
        const uint32_t e = (uint32_t)(b & 0x7fffffffull) + __popc(bv & lt);  // edge index of slot q (if valid)
        const uint32_t i = fdiv(q, fd);
        if (q == i * (uint32_t)k) indptr_out[i] = (int32_t)e;
        if ((fb >> j) & 1u) {
          const uint32_t nid = (uint32_t)F + (uint32_t)((b >> 31) & 0x7fffffffull) + __popc(bf & lt);
          src_out[nid] = r[j];
          B.rows[q] = (int32_t)nid;
          indices_out[e] = (int32_t)nid;
        } else if ((vb >> j) & 1u) {
          const uint32_t x = (uint32_t)(-1 - r[j]);
          if (x < (uint32_t)F) indices_out[e] = (int32_t)x;  // dst hit
        }
      }
    }
  }
}

// Duplicates of layer l (after pass 2 and a grid barrier): a valid slot q
// holding -1 - x with x >= F takes the nid stored at its first occurrence's
// slot x - F.
__device__ DSP_PHASE void phase_indices_dups(int F, int k, const LayerBufs &B, const int32_t *indptr,
                                                   int32_t *indices_out, const Span &sp) {
  constexpr int U = 4;  // items per thread in flight
  const FastDiv fd = make_fastdiv((uint32_t)k);
  const uint32_t end = (uint32_t)sp.end, step = (uint32_t)sp.step;
  for (uint32_t q0 = (uint32_t)sp.first; q0 < end; q0 += step * U) {
    int32_t x[U], ip[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint32_t q = q0 + j * step;
      x[j] = -1;
      if (q < end) {
        const uint32_t i = fdiv(q, fd);
        const int32_t t = (int32_t)(q - i * (uint32_t)k);
        if (ldw_i32(B.cnt + i) > t) {
          const int32_t r = ldw_i32(B.rows + q);
          if (r < 0 && -1 - r >= F) {
            x[j] = -1 - r - F;
            ip[j] = ldw_i32(indptr + i) + t;
          }
        }
      }
    }
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (x[j] >= 0) indices_out[ip[j]] = ldw_i32(B.rows + x[j]);
  }
}

// ----------------------------------------------------------------- gather
// Feature rows are stored split at the last 128-byte boundary (DESIGN.md
// "Data layout"): the head (dim*4 rounded down to a multiple of 128 bytes) in
// a packed head array whose rows are 128-byte aligned whole L2 lines, the tail
// (< 128 bytes, a multiple of 16) in a packed tail array.  A 400-byte row read
// whole touches four 128-byte lines (512 B of DRAM) at any alignment; split it
// touches three, and the tail array (16 B per node) stays L2-resident under an
// evict_last policy while the heads stream with evict_first.  Each region of
// slots (a rank's HBM shard, a rank's cold rows in host memory) holds its
// head array at `head`, its tail array at `tail`.
struct GatherArgs {
  const int32_t *ids;
  int64_t n;                // rows (ignored when n_dev is set)
  const int32_t *n_dev;     // device row count (fused call), or nullptr
  int32_t dim4;             // dim / 4  (output row length in float4)
  int32_t head4;            // head length in float4 (multiple of 8); tail = dim4 - head4 (< 8)
  float4 *out;
  const float4 *base[8];    // feature shard (hot rows) of each rank: head array (local or peer-mapped)
  const float4 *tail[8];    //   ... and its tail array
  // cold-feature tier: feature position list of each rank
  // (>= 0 hot slot, < 0 cold slot -p-1) and its cold rows in host memory (UVA)
  int32_t tiered;
  const int32_t *fpos[8];
  const float4 *cold[8];
  const float4 *cold_tail[8];
  Bounds bd;
  int *err;
};

struct RowRef {
  const float4 *head, *tail;  // the row's head (head4 float4) and tail (dim4 - head4 float4)
};

// The feature row of global id g (owner o): the shard slot, or with the cold
// tier the hot slot in HBM / the cold slot in host memory read over UVA by the
// requesting GPU ("loaded from CPU memory by the requesting GPU").
__device__ __forceinline__ RowRef feature_row(const GatherArgs &a, int o, int32_t g) {
  const uint32_t lv = (uint32_t)(g - (int32_t)a.bd.b[o]);
  const uint32_t h4 = (uint32_t)a.head4, t4 = (uint32_t)(a.dim4 - a.head4);
  const int32_t *fp = a.fpos[o];  // null: rank o keeps all its rows in HBM (in id order)
  if (!a.tiered || !fp) return RowRef{a.base[o] + (size_t)lv * h4, a.tail[o] + (size_t)lv * t4};
  const int32_t p = __ldg(fp + lv);
  if (p >= 0) return RowRef{a.base[o] + (size_t)(uint32_t)p * h4, a.tail[o] + (size_t)(uint32_t)p * t4};
  const uint32_t q = (uint32_t)(-p - 1);
  return RowRef{a.cold[o] + (size_t)q * h4, a.cold_tail[o] + (size_t)q * t4};
}
// float4 column c of a row
__device__ __forceinline__ const float4 *row_col(const RowRef &r, uint32_t c, uint32_t head4) {
  return c < head4 ? r.head + c : r.tail + (c - head4);
}

__device__ __forceinline__ float4 ld_stream_f4(const float4 *p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}

// Flat [n][dim4] float4 index space; UNROLL independent 16-byte loads in
// flight per thread before any store (Little's law over HBM / NVLink).
// 32-bit index math (the host guarantees n * dim4 < 2^31).
template <int UNROLL>
__device__ DSP_PHASE void phase_gather(const GatherArgs &a, int64_t n, int64_t tid64, int64_t nthreads64) {
  const uint32_t total = (uint32_t)(n * a.dim4);
  const uint32_t tid = (uint32_t)tid64, nthreads = (uint32_t)nthreads64;
  const uint32_t dim4 = (uint32_t)a.dim4;
  const int32_t N = (int32_t)a.bd.b[a.bd.world];
  const uint32_t head4 = (uint32_t)a.head4;
  // packed rows (head4 == 0) stream with evict_first; split rows keep their small tail array resident
  const unsigned long long pol = l2_policy_evict_first(), pol_t = head4 ? l2_policy_tail() : pol;
  for (uint32_t e0 = tid; e0 < total; e0 += nthreads * UNROLL) {
    int32_t g[UNROLL];
    uint32_t c[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const uint32_t e = e0 + (uint32_t)u * nthreads;
      g[u] = -1;
      c[u] = 0;
      if (e < total) {
        const uint32_t r = e / dim4;
        c[u] = e - r * dim4;
        g[u] = ldw_i32(a.ids + r);
      }
    }
    float4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      if (g[u] >= 0 && g[u] < N) {
        const int o = owner_of(a.bd, g[u]);
        v[u] = ld_f4_hint(row_col(feature_row(a, o, g[u]), c[u], head4), c[u] < head4 ? pol : pol_t);
      }
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const uint32_t e = e0 + (uint32_t)u * nthreads;
      if (e < total) {
        if (g[u] >= 0 && g[u] < N)
          st_f4_hint(a.out + e, v[u], pol);
        else
          latch(a.err, E_RANGE);
      }
    }
  }
}

constexpr int GATHER_UNROLL = 4;

__global__ void __launch_bounds__(NT) k_gather(const __grid_constant__ GatherArgs a) {
  const int64_t n = a.n_dev ? (int64_t)ld_volatile_i32(a.n_dev) : a.n;
  phase_gather<GATHER_UNROLL>(a, n, blockIdx.x * (int64_t)NT + threadIdx.x, (int64_t)gridDim.x * NT);
}

// ============================================ world == 1: persistent kernel
#ifndef DSP_LOADER_WARPS
#define DSP_LOADER_WARPS 5
#endif
// TMA gather warps of a pipelined launch: 5 (27 sampling warps) measured 0.1314 vs
// 0.1322 ms/step with 4 and 0.1335 with 3 (4 streams); at 2 streams 0.1266 vs 0.1334 with 4
// and 0.1323 with 6
constexpr int LOADER_WARPS = DSP_LOADER_WARPS;
#ifndef DSP_LOADER_SLOTS
#define DSP_LOADER_SLOTS 2
#endif
constexpr int LOADER_SLOTS = DSP_LOADER_SLOTS;       // ring slots per loader warp of a pipelined launch
constexpr int GTMA_SLOTS = 2;                        // ring slots per warp of the standalone gather
constexpr int PIPE_TEAM = PNT - 32 * LOADER_WARPS;   // sampling threads of a pipelined launch
#ifndef DSP_BIASED_LOADERS
#define DSP_BIASED_LOADERS 3
#endif
// biased sampling is bound by the sampling, not the gather: 3 loader warps
// (29 sampling warps) measured 0.2136-0.2148 vs 0.2166 ms/step with 4, 0.219 with 2
constexpr int BIASED_LOADER_WARPS = DSP_BIASED_LOADERS;
#ifndef DSP_BIASED_BLOCK
#define DSP_BIASED_BLOCK 1024
#endif
// threads per block of the biased persistent kernels: 1024 (64 registers) measured 0.2126-0.2173
// ms/step vs 0.2196-0.2209 with 896 (72 registers) and 0.228 with 768 (80 registers): warps beat registers
constexpr int BIASED_BLK = DSP_BIASED_BLOCK;
constexpr int BIASED_PIPE_TEAM = BIASED_BLK - 32 * BIASED_LOADER_WARPS;

struct PersistArgs {
  const int32_t *seeds;
  int32_t B;
  int32_t L;
  int32_t k[8];
  uint2 key;
  const int64_t *indptr;
  const int32_t *indices;
  const uint32_t *weights;  // 16.16 edge weights (biased sampling) or nullptr
  int32_t biased;
  int64_t lo, n_local;
  Outputs out;
  LayerBufs buf[2];
  unsigned long long *agg;  // [2][MAX_PERSIST_BLOCKS] scan aggregates
  WsPersist *persist;
  WsHeader *hdr;
  int *err;
  int32_t gather;           // fuse the gather of this call's last block (non-pipelined)
  GatherArgs g;             // this call's gather
  // pipelined: gather owed by the previous call, by the loader warps + idle samplers
  int32_t prev;             // 1 if there is one
  GatherArgs gp;            // ids / n_dev / out of the previous call
  int32_t *pend_n;          // where this call's row count goes (read by the next call / flush)
  int32_t rows_per_chunk;   // R
  int32_t slot_bytes;       // ring slot size (>= R * row bytes)
  int32_t lane_rounds;      // lane groups per node while F * G <= lane_rounds * team threads
};

// BIASED is a template parameter (not a runtime branch) so the uniform
// kernel carries no biased-sampling code (fewer instruction-cache misses).
template <int TEAM, bool BIASED>
__device__ __forceinline__ void persist_sample(const PersistArgs &a, const int32_t *frontier, int F, int l,
                                               uint32_t epoch) {
  const int k = a.k[l];
  const LayerBufs &B = a.buf[l & 1];
  if (BIASED) {
    phase_sample_biased<TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.weights, a.lo, a.n_local, B, epoch,
                              a.out.src_ids[l], a.err, &a.hdr->scursor[l]);
  } else if (k <= 16 && (int64_t)F * (k <= 4 ? 4 : k <= 8 ? 8 : 16) <= (int64_t)a.lane_rounds * gridDim.x * TEAM) {
    // small frontier (the first layers): a lane group per node, so the k
    // Philox draws run in parallel instead of back to back in one thread,
    // whose dependent-instruction latency dominates when few warps are busy
    if (k <= 4)
      phase_sample_lanes<4, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                                  a.out.src_ids[l], a.err, a.hdr);
    else if (k <= 8)
      phase_sample_lanes<8, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                                  a.out.src_ids[l], a.err, a.hdr);
    else
      phase_sample_lanes<16, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                                   a.out.src_ids[l], a.err, a.hdr);
  } else if (k <= 8) {
    phase_sample_tpn<8, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                              a.out.src_ids[l], a.err, a.hdr);
  } else if (k <= 16) {
    phase_sample_tpn<16, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                               a.out.src_ids[l], a.err, a.hdr);
  } else {
    phase_sample_lanes<32, TEAM>(frontier, F, l, k, a.key, a.indptr, a.indices, a.lo, a.n_local, B, epoch,
                                 a.out.src_ids[l], a.err, a.hdr);
  }
}

// Row claims on the previous call's gather (pipelined launches): runs of rows
// from the front (loader warps, and sampling warps once their phases are
// done) or from the back.  hdr->gcur packs the rows taken from the front (low
// 32 bits) and from the back (high 32 bits); every claim is one 64-bit
// atomicAdd, so it sees all earlier claims of both kinds: a front claim from
// (f, b) owns rows [f, min(f + R, n - b)), a back claim owns
// [max(f, n - b - U), n - b), and no row is owned twice or left over.
// (Back claims by sampling warps waiting at grid barriers measured slower:
// 0.167 vs 0.132 ms/step, the sampling phases themselves slowed down.)
// Warp-uniform.
__device__ __forceinline__ bool claim_rows(WsHeader *hdr, bool front, int cnt, int64_t n, int64_t *r0, int64_t *r1) {
  unsigned long long old = 0;
  if ((threadIdx.x & 31) == 0)
    old = atomicAdd(&hdr->gcur, front ? (unsigned long long)cnt : (unsigned long long)cnt << 32);
  old = __shfl_sync(FULL_MASK, old, 0);
  const int64_t f = (int64_t)(uint32_t)old, b = (int64_t)(old >> 32);
  if (front) {
    *r0 = f;
    *r1 = min(f + cnt, n - b);
  } else {
    *r0 = max(f, n - b - cnt);
    *r1 = n - b;
  }
  return *r1 > *r0;
}

#ifndef DSP_HELPER_UNROLL
#define DSP_HELPER_UNROLL 4
#endif
// Rows [r0, r1) of the previous call's gather by one warp with 16-byte
// register loads, HU loads in flight per lane.  MULTI (world > 1): rows of
// every rank, read from the owner's shard (local or peer-mapped).
template <bool MULTI = false>
__device__ __forceinline__ void gather_rows_regs(const PersistArgs &a, int64_t r0, int64_t r1) {
  constexpr int HU = DSP_HELPER_UNROLL;
  const int lane = threadIdx.x & 31;
  const GatherArgs &g = a.gp;
  const uint32_t dim4 = (uint32_t)g.dim4, head4 = (uint32_t)g.head4;
  const unsigned long long pol = l2_policy_evict_first(), pol_t = head4 ? l2_policy_tail() : pol;
  const uint32_t total = (uint32_t)((r1 - r0) * dim4);
  for (uint32_t e0 = lane; e0 < total; e0 += 32 * HU) {
    float4 v[HU];
    int32_t id[HU];
    uint32_t col[HU];
#pragma unroll
    for (int u = 0; u < HU; ++u) {
      const uint32_t e = e0 + 32u * u;
      id[u] = -1;
      col[u] = 0;
      if (e < total) {
        const uint32_t r = e / dim4;
        col[u] = e - r * dim4;
        id[u] = __ldg(g.ids + r0 + r);
      }
    }
    const int32_t N = (int32_t)g.bd.b[MULTI ? g.bd.world : 1];
#pragma unroll
    for (int u = 0; u < HU; ++u)
      if (id[u] >= 0 && id[u] < N)
        v[u] = ld_f4_hint(row_col(feature_row(g, MULTI ? owner_of(g.bd, id[u]) : 0, id[u]), col[u], head4),
                          col[u] < head4 ? pol : pol_t);
#pragma unroll
    for (int u = 0; u < HU; ++u) {
      const uint32_t e = e0 + 32u * u;
      if (e < total) {
        if (id[u] >= 0 && id[u] < N)
          st_f4_hint(g.out + r0 * dim4 + e, v[u], pol);
        else
          latch(g.err, E_RANGE);
      }
    }
  }
}

// Loader warp of a pipelined launch: gathers chunks of R consecutive output
// rows of the previous call with TMA bulk copies (one cp.async.bulk per row
// into a shared-memory ring slot, completion counted on the slot's mbarrier,
// then one bulk store of the R contiguous output rows).  Chunks come from a
// grid-wide cursor, so the sampling warps can join when they are done.
// LOADER_WARPS warps per SM sustain ~5 TB/s on random 400-byte rows
// (tools/micro/tma_gather_bench.cu), leaving the other warps for the sampling.
// MULTI (world > 1): rows of every rank, the bulk copy reading the owner's
// shard (local, or a peer's over NVLink through its mapping).
// STATIC: chunks gw, gw + nw, ... instead of the grid-wide cursor (the
// standalone k_gather_tma, whose warps all gather).
template <bool MULTI = false, bool STATIC = false, int SLOTS = LOADER_SLOTS>
__device__ DSP_PHASE void loader_warp(const PersistArgs &a, char *ring, uint64_t *bars, int64_t n,
                                            int64_t gw = 0, int64_t nw = 1) {
  const int lane = threadIdx.x & 31;
  const GatherArgs &g = a.gp;
  const int R = a.rows_per_chunk;
  const uint32_t row_bytes = (uint32_t)g.dim4 * 16u, head_bytes = (uint32_t)g.head4 * 16u;
  const uint32_t tail_bytes = row_bytes - head_bytes;
  char *out = reinterpret_cast<char *>(g.out);
  const unsigned long long pol = l2_policy_evict_first(), pol_t = head_bytes ? l2_policy_tail() : pol;
  int issued = 0, done = 0;
  int64_t start[SLOTS];  // first row held by each ring slot
  int nrows[SLOTS];      // and its row count
  bool exhausted = false;
  while (true) {
    while (!exhausted && issued - done < SLOTS) {
      int64_t r0 = 0, r1 = 0;
      if (STATIC) {
        const int64_t c = gw + (int64_t)issued * nw;
        r0 = min(n, c * R);
        r1 = min(n, r0 + R);
      } else {
        claim_rows(a.hdr, true, R, n, &r0, &r1);
      }
      if (r1 <= r0) {
        exhausted = true;
        break;
      }
      const int s = issued % SLOTS;
      if (issued >= SLOTS) {  // the slot's previous store must have read its smem
        if (lane == 0) bulk_wait_read<SLOTS - 1>();
        __syncwarp();
      }
      const int rows = (int)(r1 - r0);
      if (lane == 0) mbar_expect_tx(&bars[s], (uint32_t)rows * row_bytes);
      __syncwarp();
      if (lane < rows) {
        const int32_t id = __ldg(g.ids + r0 + lane);
        if (id >= 0 && id < (int32_t)g.bd.b[MULTI ? g.bd.world : 1]) {  // cold rows: host memory over UVA
          // head (whole 128-byte lines, streamed) and tail (L2-resident array) into one slot row
          const RowRef r = feature_row(g, MULTI ? owner_of(g.bd, id) : 0, id);
          char *dst = ring + (size_t)s * a.slot_bytes + (size_t)lane * row_bytes;
          if (head_bytes) bulk_g2s_hint(dst, r.head, head_bytes, &bars[s], pol);
          if (tail_bytes) bulk_g2s_hint(dst + head_bytes, r.tail, tail_bytes, &bars[s], pol_t);
        } else {  // keep the byte count consistent; the error is reported
          latch(g.err, E_RANGE);
        }
      }
#pragma unroll
      for (int q = 0; q < SLOTS; ++q)
        if (q == s) {
          start[q] = r0;
          nrows[q] = rows;
        }
      ++issued;
    }
    if (done == issued) break;
    if (!STATIC && lane == 0) atomicAdd(&a.hdr->chunks_loader, 1u);
    const int s = done % SLOTS;
    int64_t r0 = 0;
    int rows = 0;
#pragma unroll
    for (int q = 0; q < SLOTS; ++q)
      if (q == s) {
        r0 = start[q];
        rows = nrows[q];
      }
    bool bad = false;
    if (lane == 0) {
      // an out-of-range id never delivers its bytes: do not wait forever on it
      const unsigned long long t0 = globaltimer_ns();
      while (!mbar_try_wait(&bars[s], (uint32_t)(done / SLOTS) & 1u)) {
        if (*(volatile int *)g.err != 0 && globaltimer_ns() - t0 > 1000000ull) {
          bad = true;
          break;
        }
      }
      if (!bad) {
        bulk_s2g_hint(out + (size_t)r0 * row_bytes, ring + (size_t)s * a.slot_bytes, (uint32_t)rows * row_bytes, pol);
        bulk_commit();
      }
    }
    bad = __shfl_sync(FULL_MASK, bad, 0);
    __syncwarp();
    ++done;
    if (bad) break;
  }
  if (lane == 0) bulk_wait_all();
}

// A sampling warp that finished its phases takes remaining chunks of the
// previous call's gather from the front, with 16-byte register loads.
template <bool MULTI = false>
__device__ DSP_PHASE void helper_warp(const PersistArgs &a, int64_t n) {
  const int lane = threadIdx.x & 31;
  int64_t r0, r1;
  while (claim_rows(a.hdr, true, a.rows_per_chunk, n, &r0, &r1)) {
    if (lane == 0) atomicAdd(&a.hdr->chunks_helper, 1u);
    gather_rows_regs<MULTI>(a, r0, r1);
  }
}

// Standalone gather (dsp_gather_features, pending pipelined gathers): every
// warp a TMA loader (loader_warp) over a static share of the 32-row chunks:
// one cp.async.bulk per row part (head, tail) into a shared-memory ring slot,
// one bulk store of the chunk's contiguous output rows.  GTMA_WARPS x 2 slots of <= 16 KB.
#ifndef DSP_GTMA_WARPS
#define DSP_GTMA_WARPS 6
#endif
constexpr int GTMA_WARPS = DSP_GTMA_WARPS;
template <bool MULTI>
__global__ void __launch_bounds__(32 * GTMA_WARPS) k_gather_tma(const __grid_constant__ PersistArgs a, int64_t n_host) {
  __shared__ __align__(8) uint64_t bars[GTMA_WARPS][GTMA_SLOTS];
  extern __shared__ __align__(128) char ring_smem[];
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) == 0)
    for (int s2 = 0; s2 < GTMA_SLOTS; ++s2) mbar_init(&bars[w][s2], 1);
  mbar_init_fence();
  __syncwarp();
  const int64_t n = a.gp.n_dev ? (int64_t)ld_volatile_i32(a.gp.n_dev) : n_host;
  loader_warp<MULTI, true, GTMA_SLOTS>(a, ring_smem + (size_t)w * GTMA_SLOTS * a.slot_bytes, bars[w], n,
                           (int64_t)blockIdx.x * GTMA_WARPS + w, (int64_t)gridDim.x * GTMA_WARPS);
}

// The whole CSP call for world == 1 in one launch: per layer sample(l) +
// indices(l-1) | scan pass 1 | scan pass 2, separated by grid barriers; then
// indices(L-1) and either this call's gather (all warps) or, pipelined, the
// previous call's gather by the loader warps running alongside the sampling
// (the paper's loader(t-1) || sampler(t)).  No host round trip,
// no map clearing (epochs).
template <int TEAM, bool PIPE, bool BIASED, int BLK = PNT>
__global__ void __launch_bounds__(BLK, 1) k_csp_persistent(const __grid_constant__ PersistArgs a) {
#ifndef DSP_W1_GROUPS
#define DSP_W1_GROUPS 1
#endif
  constexpr int SG = DSP_W1_GROUPS;  // scan groups per round: 1 keeps pass 1's rows in registers (2 / 4: 0.130 vs 0.127 ms/step)
  __shared__ Scan2Smem<TEAM, SG> sm;
  __shared__ __align__(8) uint64_t bars[LOADER_WARPS][LOADER_SLOTS];
  extern __shared__ __align__(128) char ring_smem[];
  const int blk = blockIdx.x, nblk = gridDim.x;

  if (PIPE && threadIdx.x >= TEAM) {  // ------------------------------ loader warps
    const int w = (threadIdx.x - TEAM) >> 5;
    if ((threadIdx.x & 31) == 0)
      for (int s2 = 0; s2 < LOADER_SLOTS; ++s2) mbar_init(&bars[w][s2], 1);
    mbar_init_fence();
    __syncwarp();
    if (a.prev) {
      const int64_t n = ld_volatile_i32(a.gp.n_dev);
      if (a.gp.tiered == 1)  // cold tier read with register loads (DSP_COLD_REGLOADS=1)
        helper_warp(a, n);
      else
        loader_warp(a, ring_smem + (size_t)w * LOADER_SLOTS * a.slot_bytes, bars[w], n);
    }
    if (blockIdx.x == 0 && threadIdx.x == TEAM) a.hdr->t[22] = globaltimer_ns();  // loader warp 0 of block 0 done
    return;
  }

  // ------------------------------------------------------------ sampling team
  const int64_t tid = blockIdx.x * (int64_t)TEAM + threadIdx.x;
  const int64_t nthreads = (int64_t)gridDim.x * TEAM;
  uint32_t bar = 0;  // grid barrier target
  uint32_t e0 = *(volatile const uint32_t *)&a.persist->epoch;
  if (a.buf[0].first32) e0 = dwin_start(e0, (uint32_t)a.L);
  const bool hclear = hash_clear_due(a.persist, e0, (uint32_t)a.L, a.buf[0].mask, a.buf[0].first);
  const bool dclear = a.buf[0].first32 && dclear_due(a.persist, e0);
  if (hclear || dclear) {  // zero the relabel map (once per ~255 / L calls)
    map_zero(a.buf[0], tid, nthreads);
    grid_barrier<TEAM>(a.hdr, bar);
  }
  if (tid == 0) {  // the host cleared the header just before the launch
    a.hdr->t[0] = globaltimer_ns();
    a.hdr->F[0] = a.B;
  }
  int F = a.B;  // frontier size of layer l, tracked in every block
  int Fprev = 0;
  for (int l = 0; l < a.L; ++l) {
    const uint32_t epoch = e0 + 1 + l;
    const int32_t *frontier = l == 0 ? a.seeds : a.out.src_ids[l - 1];
    const int k = a.k[l];
    persist_sample<TEAM, BIASED>(a, frontier, F, l, epoch);
    if (l > 0)
      phase_indices_dups(Fprev, a.k[l - 1], a.buf[(l - 1) & 1], a.out.indptr[l - 1], a.out.indices[l - 1],
                         block_span<TEAM>((int64_t)Fprev * a.k[l - 1]));
    grid_barrier<TEAM>(a.hdr, bar);
    // scan over the F*k edge slots: each block one contiguous chunk of <= TEAM*IPT slots per round
    constexpr int64_t TILE = (int64_t)TEAM * SCAN2_IPT * SG;
    const int64_t total = (int64_t)F * k;
    const int64_t rounds = total > 0 ? (total + (int64_t)nblk * TILE - 1) / ((int64_t)nblk * TILE) : 1;
    const int64_t per_round = (total + rounds - 1) / rounds;
    const int64_t chunk = (per_round + nblk - 1) / nblk;
    unsigned long long carry = 0;
    for (int64_t r = 0; r < rounds; ++r) {
      Scan2Regs R;
      const int64_t r0 = r * per_round, r1 = min(total, r0 + per_round);
      const int64_t tile0 = min(r1, r0 + (int64_t)blk * chunk), tile_end = min(r1, tile0 + chunk);
      unsigned long long *agg = a.agg + (r & 1) * MAX_PERSIST_BLOCKS;
      scan2_pass1<TEAM, SG>(F, k, a.buf[l & 1], epoch, tile0, tile_end, R, agg + blk, sm);
      grid_barrier<TEAM>(a.hdr, bar);
      unsigned long long prefix, round_total;
      scan2_prefix<TEAM, SG>(agg, nblk, blk, sm, &prefix, &round_total);
      scan2_pass2<TEAM, SG>(F, k, a.buf[l & 1], tile0, tile_end, R, carry + prefix, sm, a.out.indptr[l],
                        a.out.indices[l], a.out.src_ids[l]);
      carry += round_total;
      if (r + 1 < rounds) grid_barrier<TEAM>(a.hdr, bar);
    }
    const int32_t E = (int32_t)(carry & 0x7fffffffull);
    const int32_t nnew = (int32_t)((carry >> 31) & 0x7fffffffull);
    if (tid == 0) {
      a.out.indptr[l][F] = E;
      a.hdr->E[l] = E;
      a.hdr->S[l] = F + nnew;
      a.hdr->F[l + 1] = F + nnew;
      a.hdr->sizes[3 * l + 0] = F;
      a.hdr->sizes[3 * l + 1] = F + nnew;
      a.hdr->sizes[3 * l + 2] = E;
    }
    Fprev = F;
    F = F + nnew;
    grid_barrier<TEAM>(a.hdr, bar);
  }
  // last layer's indices (F = num_src of the last block)
  const int l = a.L - 1;
  phase_indices_dups(Fprev, a.k[l], a.buf[l & 1], a.out.indptr[l], a.out.indices[l],
                     block_span<TEAM>((int64_t)Fprev * a.k[l]));
  if (PIPE) {
    if (tid == 0) *a.pend_n = F;  // this call's rows, gathered by the next pipelined call / flush
    if (a.prev) helper_warp(a, ld_volatile_i32(a.gp.n_dev));
  } else if (a.gather) {
    phase_gather<GATHER_UNROLL>(a.g, F, tid, nthreads);
  }
  // the last sampling block to finish advances the workspace epoch and stamps the end
  team_sync<TEAM>();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(&a.hdr->done, 1u) == gridDim.x - 1) {
      a.persist->epoch = e0 + (uint32_t)a.L;
      if (hclear) hash_cleared(a.persist, e0, a.buf[0].mask, a.buf[0].first);
      if (dclear) a.persist->dwin = e0 / DWIN + 1u;
      a.hdr->t[23] = globaltimer_ns();
      a.hdr->done = 0u;
    }
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
#ifdef DSP_EXPERIMENT_GPU_FENCE  // cost measurement on virtual ranks only (not valid across GPUs)
  __threadfence();
#else
  __threadfence_system();
#endif
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

// fp32 edge weights -> 16.16 fixed point a = floor(w * 2^16), w = 0 or
// w in [2^-16, 2^16) (R24); an invalid weight is counted in *bad:
// negative, NaN, >= 2^16, or positive but below 2^-16 (it would quantize to 0
// and never be sampled, silently departing from w_u / sum w).
__global__ void k_weights_fixed(const float *w, int64_t n, uint32_t *out, int *bad) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
    const float x = w[e];
    const uint32_t a = (x >= 0.0f && x < 65536.0f) ? (uint32_t)floorf(x * 65536.0f) : 0u;
    if (!(x >= 0.0f) || x >= 65536.0f || (x > 0.0f && a == 0u)) {
      atomicAdd(bad, 1);
      out[e] = 0;
    } else {
      out[e] = a;
    }
  }
}

// Random walks: step l from node v takes the fan-out-1 node-wise
// sample of v at layer l (no draw when deg <= 1); a node without neighbours
// ends the walk (-1 for the remaining steps).  One thread per walk; each step
// is two dependent random loads (indptr pair, adjacency entry).
// independent = 1 (DSP_WALK_INDEPENDENT, R35): the draw of walk i is keyed by
// i instead of slot 0, so walks from the same start are independent.
__global__ void __launch_bounds__(NT) k_random_walk(const int32_t *starts, int64_t n, int32_t length, uint2 key,
                                                    const int64_t *__restrict__ indptr,
                                                    const int32_t *__restrict__ indices, int64_t N,
                                                    int32_t *traces, int *err, int independent) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t v = __ldg(starts + i);
    int32_t *tr = traces + i * (int64_t)(length + 1);
    if (v < 0 || v >= N) {
      latch(err, E_RANGE);
      v = -1;
    }
    tr[0] = v;
    for (int l = 0; l < length; ++l) {
      if (v >= 0) {
        const int64_t s = __ldg(indptr + v);
        const int64_t d = __ldg(indptr + v + 1) - s;
        if (d == 0) {
          v = -1;
        } else {
          const uint32_t pos = d == 1        ? 0u
                               : independent ? walk_draw(key, (uint32_t)i, v, l, (uint32_t)d)
                                             : draw_range(key, 0u, v, l, (uint32_t)d);
          v = __ldg(indices + s + pos);
        }
      }
      tr[l + 1] = v;
    }
  }
}

}  // namespace dsp
