// dsp_device.cuh -- device primitives for the CSP hot path on sm_100a:
// counter-based Philox draws, warp-cooperative Floyd sampling, the relabel
// hash table, peer-memory flags.  Written for B200 from PAPER.md + DESIGN.md;
// shares nothing with oracle/.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace dsp {

constexpr unsigned FULL_MASK = 0xffffffffu;
constexpr unsigned long long EMPTY_SLOT = ~0ull;

// ---------------------------------------------------------------- errors
enum : int {
  E_OK = 0, E_INVALID = -1, E_RANGE = -2, E_DUP = -3, E_CAP = -4, E_STATE = -5,
};

__device__ __forceinline__ void latch(int *err, int code) {
  atomicCAS(err, 0, code);
}

// ---------------------------------------------------------------- Philox
// Philox4x32-10 (Salmon et al., SC'11).  Counter/key layout: DESIGN.md R5.
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
  for (int round = 0; round < 10; ++round) {
    if (round) {
      k.x += 0x9E3779B9u;
      k.y += 0xBB67AE85u;
    }
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
  }
  return c;
}

// draw(slot, v, l) in [0, m): high 64 bits of (x1:x0) * m   (R6)
__device__ __forceinline__ uint32_t draw_range(uint2 key, uint32_t slot, int32_t v, int32_t l,
                                               uint32_t m) {
  const uint4 x = philox4x32_10(make_uint4(slot, (uint32_t)v, (uint32_t)l, 0x44535031u), key);
  const unsigned long long w = ((unsigned long long)x.y << 32) | x.x;
  return (uint32_t)__umul64hi(w, (unsigned long long)m);
}

// independent random walks (R35): walk i's draw at step l from v
__device__ __forceinline__ uint32_t walk_draw(uint2 key, uint32_t walk, int32_t v, int32_t l, uint32_t m) {
  const uint4 x = philox4x32_10(make_uint4(walk, (uint32_t)v, (uint32_t)l, 0x44535057u), key);
  const unsigned long long w = ((unsigned long long)x.y << 32) | x.x;
  return (uint32_t)__umul64hi(w, (unsigned long long)m);
}

// ------------------------------------------------------------ hash table
// Open addressing, linear probing, one 64-bit word per slot:
//   word = key << 32 | val,  EMPTY = all ones (keys are < 2^31).
// val is the minimum "order key" inserted for that key: dst index i (< F)
// or F + i*k + slot for a sampled edge, so after all insertions val < F
// means "is a dst" and val == F + q means "edge slot q is the first
// occurrence".
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16;
  x *= 0x85EBCA6Bu;
  x ^= x >> 13;
  x *= 0xC2B2AE35u;
  x ^= x >> 16;
  return x;
}

// Inserts (key, val) keeping the minimum val, probing from slot `idx`.
// Returns the slot index and the previous val of the key in *old
// (0xffffffff if the key was new).
__device__ __forceinline__ uint32_t table_insert_min_from(unsigned long long *tbl, uint32_t mask, uint32_t idx,
                                                          uint32_t key, uint32_t val, uint32_t *old) {
  const unsigned long long want = ((unsigned long long)key << 32) | val;
  while (true) {
    unsigned long long cur = *(volatile unsigned long long *)&tbl[idx];
    if (cur == EMPTY_SLOT) {
      const unsigned long long prev = atomicCAS(&tbl[idx], EMPTY_SLOT, want);
      if (prev == EMPTY_SLOT) {
        *old = 0xffffffffu;
        return idx;
      }
      cur = prev;
    }
    if ((uint32_t)(cur >> 32) == key) {
      uint32_t o = (uint32_t)cur;
      if (o > val) o = (uint32_t)atomicMin(&tbl[idx], want);
      *old = o;
      return idx;
    }
    idx = (idx + 1) & mask;
  }
}

__device__ __forceinline__ uint32_t table_insert_min(unsigned long long *tbl, uint32_t mask, uint32_t key,
                                                     uint32_t val, uint32_t *old) {
  return table_insert_min_from(tbl, mask, hash32(key) & mask, key, val, old);
}

// Completion of an insertion whose first CAS at its home slot `idx` (issued
// speculatively, expecting an empty slot) returned `prev` != EMPTY.
__device__ __forceinline__ uint32_t table_insert_finish(unsigned long long *tbl, uint32_t mask, uint32_t idx,
                                                        uint32_t key, uint32_t val, unsigned long long prev,
                                                        uint32_t *old) {
  if ((uint32_t)(prev >> 32) == key) {
    uint32_t o = (uint32_t)prev;
    if (o > val) o = (uint32_t)atomicMin(&tbl[idx], ((unsigned long long)key << 32) | val);
    *old = o;
    return idx;
  }
  return table_insert_min_from(tbl, mask, (idx + 1) & mask, key, val, old);
}

// ------------------------------------------------------ peer-memory flags
__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_gpu(unsigned long long *p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// release store of a flag: system scope when a peer may sit on another device
__device__ __forceinline__ void st_release_flag(unsigned long long *p, unsigned long long v, int sys) {
  if (sys) st_release_sys(p, v); else st_release_gpu(p, v);
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// ------------------------------------------- TMA bulk copies + mbarriers
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_init_fence() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}
// L2 eviction policies: the streamed feature rows are marked evict-first so the
// sampling working set (indptr, relabel map, edge slots) stays L2-resident.
__device__ __forceinline__ unsigned long long l2_policy_evict_first() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long l2_policy_evict_last() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long l2_policy_evict_normal() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// L2 policy of the feature tails (16-byte tails of 400-byte rows: a 16 B-per-node
// array kept resident so a row costs its three head lines of DRAM)
#ifndef DSP_TAIL_POLICY
#define DSP_TAIL_POLICY 1
#endif
__device__ __forceinline__ unsigned long long l2_policy_tail() {
  return DSP_TAIL_POLICY == 0 ? l2_policy_evict_first() : DSP_TAIL_POLICY == 2 ? l2_policy_evict_normal() : l2_policy_evict_last();
}
__device__ __forceinline__ float4 ld_f4_hint(const float4 *p, unsigned long long pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_f4_hint(float4 *p, float4 v, unsigned long long pol) {
  asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
               "f"(v.w), "l"(pol) : "memory");
}
// global -> shared, completion counted in bytes on the mbarrier, with an L2 policy
__device__ __forceinline__ void bulk_g2s_hint(void *dst, const void *src, uint32_t bytes, uint64_t *bar,
                                              unsigned long long pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
      ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void bulk_s2g_hint(void *dst, const void *src, uint32_t bytes, unsigned long long pol) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
               "r"(smem_u32(src)), "r"(bytes), "l"(pol) : "memory");
}
// global -> shared, completion counted in bytes on the mbarrier
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
// shared -> global, tracked by bulk groups
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
               "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ------------------------------------------------------------- owner map
struct Bounds {
  int64_t b[9];  // DSP_MAX_WORLD + 1
  int32_t world;
};
__device__ __forceinline__ int owner_of(const Bounds &bd, int64_t g) {
  int o = 0;
#pragma unroll
  for (int r = 1; r < 8; ++r) o += (r < bd.world && g >= bd.b[r]) ? 1 : 0;
  return o;
}

// adjacency read: streamed at random, never reused within a call (L2 evict_first)
__device__ __forceinline__ int32_t adj_ld(const int32_t *p) {
  int32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(l2_policy_evict_first()));
  return v;
}

// Row extent [s, s + d) of local row lv: one 16-byte load when the pair is
// 16-byte aligned (lv even), else two 8-byte loads.
__device__ __forceinline__ void row_extent(const int64_t *__restrict__ indptr, int64_t lv, int64_t *s, int64_t *d) {
#ifdef DSP_INDPTR_EVICT_LAST
  // experiment: keep the (degree-biased) indptr working set L2-resident
  const unsigned long long pol = l2_policy_evict_last();
  long long a, b;
  if ((lv & 1) == 0) {
    asm volatile("ld.global.nc.L2::cache_hint.v2.s64 {%0,%1}, [%2], %3;" : "=l"(a), "=l"(b) : "l"(indptr + lv), "l"(pol));
  } else {
    asm volatile("ld.global.nc.L2::cache_hint.s64 %0, [%1], %2;" : "=l"(a) : "l"(indptr + lv), "l"(pol));
    asm volatile("ld.global.nc.L2::cache_hint.s64 %0, [%1], %2;" : "=l"(b) : "l"(indptr + lv + 1), "l"(pol));
  }
  *s = a;
  *d = b - a;
  return;
#endif
  if ((lv & 1) == 0) {
    const longlong2 p = __ldg(reinterpret_cast<const longlong2 *>(indptr + lv));
    *s = p.x;
    *d = p.y - p.x;
  } else {
    const int64_t a = __ldg(indptr + lv);
    *s = a;
    *d = __ldg(indptr + lv + 1) - a;
  }
}

// ------------------------------------------------------- one node's sample
// Lane group of G lanes (G = next pow2 >= k) samples node v.  Returns, per
// lane t: whether slot `*slot` of the node holds sampled neighbour *u, and
// the node's count min(deg, k).  Warp-uniform control flow (every lane of the
// warp calls it): full rows and inactive groups run the same instructions.
//
// Floyd's algorithm (R7): lane t < k draws r_t in [0, d-k+t];
// step t takes j_t = d-k+t if r_t equals an earlier choice, else r_t.  The
// positions are then ranked (sorted ascending) by pairwise comparison, so
// slot = rank and neighbours come out in row order.
template <int G>
__device__ __forceinline__ void sample_node(bool ok, int32_t v, int64_t row_start, int64_t deg,
                                            int k, int layer, uint2 key,
                                            const int32_t *__restrict__ indices, bool *valid,
                                            int *slot, int32_t *u, int *count) {
  const int lane = threadIdx.x & 31;
  const int t = lane & (G - 1);
  const int gbase = lane & ~(G - 1);
  const unsigned gmask = (G == 32) ? FULL_MASK : (((1u << G) - 1u) << gbase);
  const bool full = deg <= k;
  uint32_t chosen = (uint32_t)t;
  if (ok && !full && t < k) {
    const uint32_t j = (uint32_t)(deg - k + t);
    chosen = draw_range(key, (uint32_t)t, v, layer, j + 1u);
  }
  // Floyd resolution, slot by slot
  for (int tt = 1; tt < k; ++tt) {
    const uint32_t x = __shfl_sync(FULL_MASK, chosen, tt, G);
    const bool hit = (t < tt) && (chosen == x);
    const unsigned m = __ballot_sync(FULL_MASK, hit) & gmask;
    if (t == tt && m != 0u) chosen = (uint32_t)(deg - k + tt);
  }
  // rank = number of chosen positions smaller than mine (they are distinct)
  int rank = 0;
  for (int s = 0; s < k; ++s) {
    const uint32_t c = __shfl_sync(FULL_MASK, chosen, s, G);
    rank += (c < chosen) ? 1 : 0;
  }
  const int cnt = ok ? (int)(full ? deg : k) : 0;
  *count = cnt;
  *valid = t < cnt;
  *slot = full ? t : rank;
  *u = *valid ? adj_ld(indices + row_start + chosen) : -1;
}

// -------------------------------------------------- one node's biased sample
__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(FULL_MASK, x, off);
  return x;
}
__device__ __forceinline__ unsigned long long warp_incl_scan_u64(unsigned long long x) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const unsigned long long y = __shfl_up_sync(FULL_MASK, x, off);
    if (lane >= off) x += y;
  }
  return x;
}

// Biased sample of node v by a whole warp (R24-R26): with
// a[p] the 16.16 fixed-point weight of row position p, successive sampling
// without replacement: k times, r = mulhi(Philox{t, v, l, "DSPB"}, W) with W
// the total weight of the positions not yet picked, and the pick is the first
// position (row order) whose running weight exceeds r.  When at most k
// positions have a positive weight they are all taken, no draw.  Lanes t <
// cnt return a position in *pos and its output slot in *slot (the rank of the
// position among the cnt returned, so slot order is row order).  Warp-uniform.
//
// Draw words: lane (wbase + t) of `wordg` holds the word of draw t of this
// node (callers compute the words of several nodes in one Philox pass:
// biased_group_word).
//
// Rows of up to 256 positions whose weights are all <= 2^24 (the common
// case; every running weight then fits 32 bits) are sampled by lane groups,
// 32 / G nodes per warp at once (biased_group_pass).  This warp-wide sampler
// takes the rest: the row is read in 128-byte-aligned chunks of 32 weights
// (chunk c, lane l: weight index A + 32c + l, A = the row start rounded down
// to 32; slots outside the row hold 0), one line per coalesced load.  Rows of
// up to 32 * HSEG chunks keep the chunk sums in registers (lane l: chunks
// 32j + l) with their running weights (row order) of the positions not yet
// picked, 64-bit: a round counts the chunks whose running weight is <= r (one
// REDUX over the lanes' counts: running weights are non-decreasing and a
// picked position's interval is empty), which is the crossing chunk; it is
// re-read (earlier picks in it masked out) and scanned; removing the pick
// subtracts its weight from the running weights behind it.  The pick's rank
// among the earlier picks is kept on the fly (no sort).  Longer rows re-read
// the row every round.
constexpr int HSEG = 4;   // chunk sums per lane of the chunk-sum path

// Lanes t < k hold distinct picks; lane r returns the pick of rank r (ascending):
// each lane ranks its own pick with k shuffles, then one ballot + shuffle per
// rank moves it to its lane (3k warp ops instead of k^2).
__device__ __forceinline__ uint32_t biased_sort_picks(uint32_t pick, int k) {
  const int lane = threadIdx.x & 31;
  int rank = 0;
  for (int j = 0; j < k; ++j) rank += __shfl_sync(FULL_MASK, pick, j) < pick ? 1 : 0;
  uint32_t mine = 0xffffffffu;
  for (int r = 0; r < k; ++r) {
    const uint32_t b = __ballot_sync(FULL_MASK, lane < k && rank == r);
    const uint32_t v = __shfl_sync(FULL_MASK, pick, __ffs(b) - 1);
    if (lane == r) mine = v;
  }
  return mine;
}

__device__ __forceinline__ unsigned long long biased_word(uint2 key, int t, int32_t v, int layer) {
  const uint4 x = philox4x32_10(make_uint4((uint32_t)t, (uint32_t)v, (uint32_t)layer, 0x44535042u), key);
  return ((unsigned long long)x.y << 32) | x.x;
}

// Draw words of up to G = 32 / k nodes in one Philox pass: lane t (< G * k)
// computes draw t % k of the node held (as vl) by lane j0 + t / k of the
// warp.  tq = lane / k and tr = lane % k are precomputed by the caller.
__device__ __forceinline__ unsigned long long biased_group_word(uint2 key, int layer, int32_t vl, int j0, int G,
                                                                int tq, int tr) {
  const int src = min(j0 + tq, 31);
  const int32_t v = __shfl_sync(FULL_MASK, vl, src);
  return tq < G ? biased_word(key, tr, v, layer) : 0ull;
}

// Round t picked position p (warp-uniform): lane t keeps it, and every pick
// so far keeps its rank among the picks.
__device__ __forceinline__ void biased_track(int t, uint32_t p, uint32_t &pick, int &rank) {
  const int lane = threadIdx.x & 31;
  const uint32_t below = __ballot_sync(FULL_MASK, lane < t && pick < p);
  if (lane < t && pick > p) ++rank;
  if (lane == t) {
    pick = p;
    rank = __popc(below);
  }
}

// Every positive-weight position of the row (at most k of them), in row
// order: lane t gets the t-th one.  m(j) is the ballot of chunk j.
template <typename Mask>
__device__ __forceinline__ uint32_t biased_all_positive(int nch, int off, Mask m) {
  const int lane = threadIdx.x & 31;
  int base = 0;
  uint32_t mine = 0xffffffffu;
  for (int j = 0; j < nch; ++j) {
    const uint32_t b = m(j);
    const int want = lane - base;
    if (want >= 0 && want < __popc(b)) mine = (uint32_t)(32 * j - off) + __fns(b, 0, want + 1);
    base += __popc(b);
  }
  return mine;
}

// Sum over the warp of 32-bit values as a 64-bit total (two 32-bit REDUX).
__device__ __forceinline__ unsigned long long warp_sum_w(uint32_t x) {
  return (unsigned long long)__reduce_add_sync(FULL_MASK, x & 0xffffu) +
         ((unsigned long long)__reduce_add_sync(FULL_MASK, x >> 16) << 16);
}

// Rows of up to 32 * HSEG aligned chunks: lane l holds the sum of chunk
// 32j + l in cs[j] and the chunk's running weight (inclusive, row order) in
// CP[j], 64-bit.  A round finds the crossing chunk by counting as above,
// re-reads it (earlier picks in it masked out) and scans it.
__device__ __forceinline__ int biased_chunks(const uint32_t *__restrict__ al, int off, int d, int nch, int k,
                                             unsigned long long wordg, int wbase, uint32_t *pos, int *slot) {
  using U = unsigned long long;
  const int lane = threadIdx.x & 31;
  U cs[HSEG], CP[HSEG];
  // lane l sums chunk 32j + l: one aligned 128-byte line, 8 vector loads, all
  // lanes' lines in flight at once (slots outside the row masked to 0)
  uint32_t np = 0;
#pragma unroll
  for (int j = 0; j < HSEG; ++j) {
    cs[j] = 0;
    const int c = 32 * j + lane;
    if (32 * j < nch && c < nch) {
      const uint4 *line = reinterpret_cast<const uint4 *>(al + 32 * c);
      uint4 q4[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) q4[e] = __ldg(line + e);
      const int lo = max(0, off - 32 * c), hi = min(32, off + d - 32 * c);  // valid slots [lo, hi)
      U s = 0;
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const uint32_t v4[4] = {q4[e].x, q4[e].y, q4[e].z, q4[e].w};
#pragma unroll
        for (int f = 0; f < 4; ++f) {
          const int i = 4 * e + f;
          const uint32_t x = (i >= lo && i < hi) ? v4[f] : 0u;
          s += x;
          np += x > 0u ? 1u : 0u;
        }
      }
      cs[j] = s;
    }
  }
  const int npos = (int)__reduce_add_sync(FULL_MASK, np);
  if (npos <= k) {
    *pos = biased_all_positive(nch, off, [&](int j) {
      const int q = 32 * j + lane;
      return __ballot_sync(FULL_MASK, q >= off && q < off + d && __ldg(al + q) > 0u);
    });
    return npos;
  }
  U base = 0;
#pragma unroll
  for (int j = 0; j < HSEG; ++j) {
    U s = cs[j];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const U y = __shfl_up_sync(FULL_MASK, s, o);
      if (lane >= o) s += y;
    }
    CP[j] = base + s;
    base = __shfl_sync(FULL_MASK, CP[j], 31);
  }
  U W = base;
  uint32_t pick = 0xffffffffu;
  int rank = 0;
  for (int t = 0; t < k; ++t) {
    const U r = __umul64hi(__shfl_sync(FULL_MASK, wordg, wbase + t), W);
    uint32_t c = 0;
#pragma unroll
    for (int j = 0; j < HSEG; ++j) c += CP[j] <= r ? 1u : 0u;
    const int cst = (int)__reduce_add_sync(FULL_MASK, c);  // the crossing chunk
    const int js = cst >> 5, Lc = cst & 31;
    U csel = cs[0], psel = CP[0];
#pragma unroll
    for (int j = 1; j < HSEG; ++j)
      if (j == js) {
        csel = cs[j];
        psel = CP[j];
      }
    const U before = __shfl_sync(FULL_MASK, psel, Lc) - __shfl_sync(FULL_MASK, csel, Lc);
    const int q = 32 * cst + lane;
    uint32_t x = (q >= off && q < off + d) ? __ldg(al + q) : 0u;
    // earlier picks inside this chunk (usually none)
    uint32_t M = __ballot_sync(FULL_MASK, lane < t && ((pick + (uint32_t)off) >> 5) == (uint32_t)cst);
    uint32_t taken = 0;
    while (M) {
      const int s = __ffs(M) - 1;
      M &= M - 1;
      taken |= 1u << ((__shfl_sync(FULL_MASK, pick, s) + (uint32_t)off) & 31u);
    }
    if ((taken >> lane) & 1u) x = 0u;
    U incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const U y = __shfl_up_sync(FULL_MASK, incl, o);
      if (lane >= o) incl += y;
    }
    const int Lp = __ffs(__ballot_sync(FULL_MASK, before + incl > r)) - 1;
    const uint32_t ap = __shfl_sync(FULL_MASK, x, Lp);
    if (lane == Lc) {
#pragma unroll
      for (int j = 0; j < HSEG; ++j)
        if (j == js) cs[j] -= ap;
    }
    const int jt = js + (lane < Lc ? 1 : 0);
#pragma unroll
    for (int j = 0; j < HSEG; ++j) CP[j] -= j >= jt ? (U)ap : 0ull;
    W -= ap;
    biased_track(t, (uint32_t)(32 * cst + Lp - off), pick, rank);
  }
  *pos = pick;
  *slot = rank;
  return k;
}

__device__ __forceinline__ int sample_node_biased(bool ok, int32_t v, int64_t row_start, int64_t deg, int k,
                                                  int layer, uint2 key, const uint32_t *__restrict__ w,
                                                  unsigned long long wordg, int wbase, uint32_t *pos, int *slot) {
  const int lane = threadIdx.x & 31;
  *slot = lane;
  if (!ok) return 0;
  const int d = (int)deg;
  const int off = (int)(row_start & 31);
  const uint32_t *al = w + (row_start - off);  // 128-byte aligned
  const int nch = (off + d + 31) >> 5;
  if (nch <= 32 * HSEG) return biased_chunks(al, off, d, nch, k, wordg, wbase, pos, slot);
  const uint32_t *a = w + row_start;
  // ---------------------------------------------------------- very long rows
  int npos = 0;
  for (int c0 = 0; c0 < d; c0 += 32) npos += __popc(__ballot_sync(FULL_MASK, c0 + lane < d && a[c0 + lane] > 0u));
  if (npos <= k) {
    int base = 0;
    uint32_t mine = 0xffffffffu;
    for (int c0 = 0; c0 < d; c0 += 32) {
      const bool f = c0 + lane < d && a[c0 + lane] > 0u;
      const uint32_t b = __ballot_sync(FULL_MASK, f);
      const int want = lane - base;
      if (want >= 0 && want < __popc(b)) mine = c0 + (__fns(b, 0, want + 1));
      base += __popc(b);
    }
    *pos = mine;
    return npos;
  }
  uint32_t pick = 0xffffffffu;
  for (int t = 0; t < k; ++t) {
    unsigned long long part = 0;
    for (int c0 = 0; c0 < d; c0 += 32) {
      const int p = c0 + lane;
      bool taken = p >= d;
      for (int j = 0; j < t; ++j) taken |= __shfl_sync(FULL_MASK, pick, j) == (uint32_t)p;
      if (!taken) part += a[p];
    }
    const unsigned long long W = warp_sum_u64(part);
    const unsigned long long r = __umul64hi(__shfl_sync(FULL_MASK, wordg, wbase + t), W);
    unsigned long long acc = 0;
    uint32_t found = 0xffffffffu;
    for (int c0 = 0; c0 < d && found == 0xffffffffu; c0 += 32) {
      const int p = c0 + lane;
      bool taken = p >= d;
      for (int j = 0; j < t; ++j) taken |= __shfl_sync(FULL_MASK, pick, j) == (uint32_t)p;
      const unsigned long long val = taken ? 0ull : (unsigned long long)a[p];
      const unsigned long long incl = warp_incl_scan_u64(val);
      const uint32_t cross = __ballot_sync(FULL_MASK, acc + incl > r);
      if (cross) found = (uint32_t)(c0 + __ffs(cross) - 1);
      acc += __shfl_sync(FULL_MASK, incl, 31);
    }
    if (lane == t) pick = found;
  }
  *pos = biased_sort_picks(pick, k);
  return k;
}

// ------------------------------------------------ biased sampling by lane groups
// A group of G lanes samples one node whose row has d <= 8G positions and
// whose weights are all <= 2^24 (so the row's total, <= 256 * 2^24, fits 32
// bits unless it is exactly 2^32, which is detected), with k <= G: lane g
// holds positions [8g, 8g + 8) in registers and their running weights (row
// order, of the positions not yet picked) P[i].  The successive-sampling
// round of sample_node_biased then costs one group reduction: the pick p is
// the number of positions whose running weight is <= r, its weight comes
// from the lane holding it, and the running weights behind it drop by that
// weight.  32 / G nodes per warp at once, every collective over the whole
// warp with width G, the k rounds uniform over the warp (k is the layer's).
// Lane t < k of a group draws word t.  Out receives the results:
//   Out::Ctx ctx(int jn)                      (all lanes; jn = claim-local node)
//   void node(const Ctx &, int32_t v, bool ok, int cnt)   (one lane per node)
//   void edge(const Ctx &, int slot, int32_t u)           (one lane per edge)
// Returns the claim-local nodes of cmask that need the warp-wide sampler
// (a weight above 2^24): their results are not written.
constexpr uint32_t BGROUP_WMAX = 1u << 24;

// the bits of lane group grp (G lanes) of a warp ballot
template <int G>
__device__ __forceinline__ uint32_t bslice(uint32_t b, int grp) {
  return G == 32 ? b : (b >> (grp * G)) & ((1u << G) - 1u);
}

// the sums of x over each group of G lanes with one warp REDUX: group q's
// values shifted into their own 32 / (32 / G)-bit field (the sums must fit it)
template <int G>
__device__ __forceinline__ uint32_t group_sum_redux(uint32_t x, int grp) {
  if constexpr (G == 32) {
    return __reduce_add_sync(FULL_MASK, x);
  } else {
    constexpr int SH = G;  // 32 / (32 / G) bits per group
    const uint32_t tot = __reduce_add_sync(FULL_MASK, x << (SH * grp));
    return (tot >> (SH * grp)) & ((1u << SH) - 1u);
  }
}

#ifdef DSP_BPROF
#define BPROF_T(var) const long long var = clock64()
#define BPROF_ADD(idx, val) do { if (bprof && (threadIdx.x & 31) == 0) atomicAdd(bprof + (idx), (unsigned long long)(val)); } while (0)
#else
#define BPROF_T(var)
#define BPROF_ADD(idx, val) do { } while (0)
#endif
template <int G, class Out>
__device__ __forceinline__ uint32_t biased_group_pass(uint32_t cmask, int32_t vl, bool okl, int64_t sl, int dl, int k,
                                                      int layer, uint2 key, const uint32_t *__restrict__ w,
                                                      const int32_t *__restrict__ indices, const Out &out,
                                                      unsigned long long *bprof = nullptr) {
  constexpr int NPW = 32 / G;
  const int lane = threadIdx.x & 31, grp = lane / G, g = lane & (G - 1);
  uint32_t redo = 0;
  while (cmask) {
    int jn = -1;
#pragma unroll
    for (int q = 0; q < NPW; ++q) {
      if (cmask) {
        if (q == grp) jn = __ffs(cmask) - 1;
        cmask &= cmask - 1;
      }
    }
    BPROF_T(s0);
    const bool act = jn >= 0;
    const int src = act ? jn : 0;
    const int32_t v = __shfl_sync(FULL_MASK, vl, src);
    const bool ok = __shfl_sync(FULL_MASK, okl, src) && act;
    const int64_t s = __shfl_sync(FULL_MASK, sl, src);
    const int dsh = __shfl_sync(FULL_MASK, dl, src);
    const int d = act && ok ? dsh : 0;
    const typename Out::Ctx c = out.ctx(src);
    const unsigned long long word = (g < k && d > 0) ? biased_word(key, g, v, layer) : 0ull;
    BPROF_T(s1);
    uint32_t x[8], P[8];
    bool heavy = false;
    uint32_t np = 0, T = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int p = 8 * g + i;
      x[i] = p < d ? __ldg(w + s + p) : 0u;
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      heavy |= x[i] > BGROUP_WMAX;
      np += x[i] > 0u ? 1u : 0u;
      T += x[i];
      P[i] = T;
    }
    // group scan of the lane totals; the group's positive count by a packed REDUX
    uint32_t incl = T;
#pragma unroll
    for (int o = 1; o < G; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL_MASK, incl, o, G);
      if (g >= o) incl += y;
    }
    uint32_t W = __shfl_sync(FULL_MASK, incl, G - 1, G);
    const uint32_t npos = group_sum_redux<G>(np, grp);
    const uint32_t hb = __ballot_sync(FULL_MASK, heavy);
    heavy = bslice<G>(hb, grp) != 0u || (W == 0u && npos > 0u);
#pragma unroll
    for (int i = 0; i < 8; ++i) P[i] += incl - T;
    const bool allpos = npos <= (uint32_t)k;
    BPROF_T(s2);
    uint32_t pick = 0xffffffffu;
    int rank = 0;
    unsigned long long wt = __shfl_sync(FULL_MASK, word, 0, G);
    for (int t = 0; t < k; ++t) {
      // mulhi(word, W) for W < 2^32 (as sample_node_biased's rounds)
      const uint32_t r = (uint32_t)(((unsigned long long)(uint32_t)(wt >> 32) * W + __umulhi((uint32_t)wt, W)) >> 32);
      wt = __shfl_sync(FULL_MASK, word, min(t + 1, G - 1), G);  // the next round's word, off the chain
      // count of the lane's positions whose running weight is <= r (adder tree)
      const uint32_t c01 = (P[0] <= r ? 1u : 0u) + (P[1] <= r ? 1u : 0u), c23 = (P[2] <= r ? 1u : 0u) + (P[3] <= r ? 1u : 0u);
      const uint32_t c45 = (P[4] <= r ? 1u : 0u) + (P[5] <= r ? 1u : 0u), c67 = (P[6] <= r ? 1u : 0u) + (P[7] <= r ? 1u : 0u);
      const uint32_t cnt = (c01 + c23) + (c45 + c67);
      // running weights are non-decreasing along the group's positions and a
      // picked position's interval is empty, so the pick is the group's count
      // (one packed REDUX for all groups of the warp: 48 cycles, vs 3 dependent
      // shuffles; a chain-length win measured 0.2125 -> 0.2085 ms/step)
      const uint32_t p = group_sum_redux<G>(cnt, grp);
      const int io = (int)(p & 7u);
      // x[io] by a 3-level select tree (depth 3 instead of a chain of 7)
      const uint32_t s01 = (io & 1) ? x[1] : x[0], s23 = (io & 1) ? x[3] : x[2];
      const uint32_t s45 = (io & 1) ? x[5] : x[4], s67 = (io & 1) ? x[7] : x[6];
      const uint32_t s03 = (io & 2) ? s23 : s01, s47 = (io & 2) ? s67 : s45;
      const uint32_t xs = (io & 4) ? s47 : s03;
      const uint32_t ap = __shfl_sync(FULL_MASK, xs, (int)(p >> 3), G);
#pragma unroll
      for (int i = 0; i < 8; ++i) P[i] -= (uint32_t)(8 * g + i) >= p ? ap : 0u;
      W -= ap;
      const uint32_t below = bslice<G>(__ballot_sync(FULL_MASK, g < t && pick < p), grp);
      if (g < t && pick > p) ++rank;
      if (g == t) {
        pick = p;
        rank = __popc(below);
      }
    }
    BPROF_T(s3);
    if (act && !heavy) {
      const int cnt = allpos ? (int)npos : k;
      if (g == 0) out.node(c, v, ok, cnt);
      if (allpos) {  // every positive-weight position, in row order
        // the group's lanes are all here (act, heavy and allpos are per group)
        const unsigned gm = G == 32 ? FULL_MASK : ((1u << G) - 1u) << (grp * G);
        uint32_t ipos = np;
#pragma unroll
        for (int o = 1; o < G; o <<= 1) {
          const uint32_t z = __shfl_up_sync(gm, ipos, o, G);
          if (g >= o) ipos += z;
        }
        uint32_t sl2 = ipos - np;
#pragma unroll
        for (int i = 0; i < 8; ++i)
          if (x[i] > 0u) out.edge(c, (int)sl2++, __ldg(indices + s + 8 * g + i));
      } else if (g < k) {
        out.edge(c, rank, __ldg(indices + s + pick));
      }
    }
    redo |= __reduce_or_sync(FULL_MASK, (act && heavy && g == 0) ? 1u << jn : 0u);
    BPROF_T(s4);
    if (G == 8) {
      BPROF_ADD(11, s1 - s0); BPROF_ADD(12, s2 - s1); BPROF_ADD(13, s3 - s2); BPROF_ADD(14, s4 - s3);
      BPROF_ADD(15, 1);
    }
  }
  return redo;
}

// The G of a node's lane group (8, 16 or 32: d <= 8G and k <= G), or 0 for
// the warp-wide sampler (d > 256).
__device__ __forceinline__ int biased_group_of(int64_t d, int k) {
  const int gd = d <= 64 ? 8 : d <= 128 ? 16 : d <= 256 ? 32 : 0;
  const int gk = k <= 8 ? 8 : k <= 16 ? 16 : 32;
  return gd == 0 ? 0 : max(gd, gk);
}

// One claim of nn <= 32 nodes (lane j < nn holds node j's id vl, okl, row
// start sl and degree dl): the grouped passes, then the warp-wide sampler for
// long or heavy rows, node by node.
template <class Out>
__device__ __forceinline__ void biased_claim(int nn, int32_t vl, bool okl, int64_t sl, int64_t dl, int k, int layer,
                                             uint2 key, const uint32_t *__restrict__ w,
                                             const int32_t *__restrict__ indices, const Out &out,
                                             unsigned long long *bprof = nullptr) {
  const int lane = threadIdx.x & 31;
  const int gl = lane < nn ? (okl ? biased_group_of(dl, k) : 8) : -1;
  const int dg = (int)min(dl, (int64_t)256);
  BPROF_T(c0);
  uint32_t redo = biased_group_pass<8>(__ballot_sync(FULL_MASK, gl == 8), vl, okl, sl, dg, k, layer, key, w, indices, out, bprof);
  BPROF_T(c1);
  redo |= biased_group_pass<16>(__ballot_sync(FULL_MASK, gl == 16), vl, okl, sl, dg, k, layer, key, w, indices, out);
  BPROF_T(c2);
  redo |= biased_group_pass<32>(__ballot_sync(FULL_MASK, gl == 32), vl, okl, sl, dg, k, layer, key, w, indices, out);
  BPROF_T(c3);
  BPROF_ADD(1, c1 - c0); BPROF_ADD(2, c2 - c1); BPROF_ADD(3, c3 - c2);
#ifdef DSP_BPROF
  const int n8 = __popc(__ballot_sync(FULL_MASK, gl == 8)), n16 = __popc(__ballot_sync(FULL_MASK, gl == 16)),
            n32 = __popc(__ballot_sync(FULL_MASK, gl == 32));
  BPROF_ADD(5, n8); BPROF_ADD(6, n16); BPROF_ADD(7, n32);
#endif
  uint32_t rest = redo | __ballot_sync(FULL_MASK, gl == 0);
  BPROF_ADD(8, __popc(rest));
  while (rest) {
    const int j = __ffs(rest) - 1;
    rest &= rest - 1;
    const int32_t v = __shfl_sync(FULL_MASK, vl, j);
    const bool ok = __shfl_sync(FULL_MASK, okl, j);
    const int64_t s = __shfl_sync(FULL_MASK, sl, j), d = __shfl_sync(FULL_MASK, dl, j);
    const typename Out::Ctx c = out.ctx(j);
    const unsigned long long word = lane < k ? biased_word(key, lane, v, layer) : 0ull;
    uint32_t pos;
    int slot;
    const int cnt = sample_node_biased(ok, v, s, d, k, layer, key, w, word, 0, &pos, &slot);
    if (lane == 0) out.node(c, v, ok, cnt);
    if (lane < cnt) out.edge(c, slot, __ldg(indices + s + pos));
  }
  BPROF_T(c4);
  BPROF_ADD(4, c4 - c3);
}

}  // namespace dsp
