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
// positions have a positive weight they are all taken, no draw.  Lane t < cnt
// returns the t-th position in ascending row order in *pos.  Warp-uniform.
//
// Rows of up to 32 positions hold one weight per lane and a round's crossing
// lane is the pick.  Rows of up to 32*BSEG positions keep their weights in registers, lane l
// holding the contiguous segment [l*S, (l+1)*S): a round is one warp sum, one
// warp scan of the lane totals and a scan inside the crossing lane's segment,
// and the pick is removed by zeroing one register.  Longer rows re-read the
// weights and test membership against the picks so far.
constexpr int BSEG = 8;

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

// The k rounds of the register path (below): lane t's draw word is myword of
// lane t, incl the inclusive scan of the lane totals tot, W their sum; the pick
// of round t is left in lane t.  (The same rounds in 32-bit arithmetic when
// W < 2^32, as a second copy of this loop, measured 8 % slower: 0.331 vs 0.308
// ms/step, the larger kernel.)
__device__ __forceinline__ uint32_t biased_reg_rounds(uint32_t (&reg)[BSEG], unsigned long long myword,
                                                      unsigned long long incl, unsigned long long tot,
                                                      unsigned long long W, int k, int S) {
  using U = unsigned long long;
  const int lane = threadIdx.x & 31;
  uint32_t pick = 0xffffffffu;
  for (int t = 0; t < k; ++t) {
    const U r = __umul64hi(__shfl_sync(FULL_MASK, myword, t), W);
    const uint32_t cross = __ballot_sync(FULL_MASK, incl > r);
    const int L = __ffs(cross) - 1;
    uint32_t found = 0, wrem = 0;
    if (lane == L) {
      U acc = incl - tot;
      bool done = false;
#pragma unroll
      for (int j = 0; j < BSEG; ++j) {
        if (!done && acc + reg[j] > r) {
          found = (uint32_t)(lane * S + j);
          wrem = reg[j];
          reg[j] = 0u;  // remove the pick
          done = true;
        }
        acc += reg[j];
      }
      tot -= wrem;
    }
    found = __shfl_sync(FULL_MASK, found, L);
    wrem = __shfl_sync(FULL_MASK, wrem, L);
    if (lane >= L) incl -= wrem;
    W -= wrem;
    if (lane == t) pick = found;
  }
  return pick;
}

__device__ __forceinline__ int sample_node_biased(bool ok, int32_t v, int64_t row_start, int64_t deg, int k,
                                                  int layer, uint2 key, const uint32_t *__restrict__ w,
                                                  uint32_t *pos) {
  const int lane = threadIdx.x & 31;
  if (!ok) return 0;
  const uint32_t *a = w + row_start;
  const int d = (int)deg;
  if (d <= 32) {
    // ------------------------------------------ one weight per lane (lane = position)
    // the crossing lane of a round is the pick itself (no in-lane scan), and the
    // picks as a lane mask are already in row order
    const uint32_t x = lane < d ? __ldg(a + lane) : 0u;
    const uint32_t posm = __ballot_sync(FULL_MASK, x > 0u);
    const int npos = __popc(posm);
    if (npos <= k) {
      *pos = lane < npos ? (uint32_t)__fns(posm, 0, lane + 1) : 0xffffffffu;
      return npos;
    }
    const unsigned long long myword = lane < k ? biased_word(key, lane, v, layer) : 0ull;  // all draws at once
    unsigned long long incl = warp_incl_scan_u64(x);
    unsigned long long W = __shfl_sync(FULL_MASK, incl, 31);
    uint32_t pm = 0;
    for (int t = 0; t < k; ++t) {
      const unsigned long long r = __umul64hi(__shfl_sync(FULL_MASK, myword, t), W);
      const int L = __ffs(__ballot_sync(FULL_MASK, incl > r)) - 1;
      const uint32_t wrem = __shfl_sync(FULL_MASK, x, L);
      if (lane >= L) incl -= wrem;  // L's interval becomes empty
      W -= wrem;
      pm |= 1u << L;
    }
    *pos = lane < k ? (uint32_t)__fns(pm, 0, lane + 1) : 0xffffffffu;
    return k;
  }
  if (d <= 32 * BSEG) {
    // ------------------------------------------------ weights in registers
    const int S = (d + 31) >> 5;
    uint32_t reg[BSEG];
    int mypos = 0;
#pragma unroll
    for (int j = 0; j < BSEG; ++j) {
      const int p = lane * S + j;
      reg[j] = (j < S && p < d) ? __ldg(a + p) : 0u;
      mypos += reg[j] > 0u ? 1 : 0;
    }
    int npos = mypos;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) npos += __shfl_xor_sync(FULL_MASK, npos, off);
    if (npos <= k) {  // every positive-weight position, in row order
      int excl = mypos;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const int y = __shfl_up_sync(FULL_MASK, excl, off);
        if (lane >= off) excl += y;
      }
      excl -= mypos;
      uint32_t mine = 0xffffffffu;
      // lane t needs the position of rank t: owner lanes hand it over one rank at a time
      for (int t = 0; t < npos; ++t) {
        const bool own = t >= excl && t < excl + mypos;
        uint32_t cand = 0;
        if (own) {
          int r = excl;
#pragma unroll
          for (int j = 0; j < BSEG; ++j)
            if (reg[j] > 0u) {
              if (r == t) cand = (uint32_t)(lane * S + j);
              ++r;
            }
        }
        const uint32_t b = __ballot_sync(FULL_MASK, own);
        const uint32_t got = __shfl_sync(FULL_MASK, cand, __ffs(b) - 1);
        if (lane == t) mine = got;
      }
      *pos = mine;
      return npos;
    }
    uint32_t pick = 0xffffffffu;
    const unsigned long long myword = lane < k ? biased_word(key, lane, v, layer) : 0ull;  // all draws at once
    // lane totals, their inclusive scan and the remaining weight W, scanned once and
    // then updated in place: removing weight w at lane L lowers incl of lanes >= L by w
    unsigned long long tot = 0;
#pragma unroll
    for (int j = 0; j < BSEG; ++j) tot += reg[j];
    const unsigned long long incl = warp_incl_scan_u64(tot);
    const unsigned long long W = __shfl_sync(FULL_MASK, incl, 31);
    pick = biased_reg_rounds(reg, myword, incl, tot, W, k, S);
    *pos = biased_sort_picks(pick, k);
    return k;
  }
  // ------------------------------------------- long rows: chunk sums in registers
  // chunk c = positions [32c, 32c+32); lane l holds the sums of chunks
  // [l*T, (l+1)*T).  A round finds the crossing chunk from the chunk sums, then
  // the crossing position inside it (picks already in that chunk masked out).
  if (d <= 32 * 32 * BSEG) {
    const int nch = (d + 31) >> 5, T = (nch + 31) >> 5;
    unsigned long long cs[BSEG];
    int npos = 0;
#pragma unroll
    for (int j = 0; j < BSEG; ++j) cs[j] = 0;
    for (int c = 0; c < nch; ++c) {
      const int p = c * 32 + lane;
      const uint32_t x = p < d ? __ldg(a + p) : 0u;
      npos += __popc(__ballot_sync(FULL_MASK, x > 0u));
      const unsigned long long sum = warp_sum_u64(x);
      if (lane == c / T) {
#pragma unroll
        for (int j = 0; j < BSEG; ++j)
          if (j == c - lane * T) cs[j] = sum;
      }
    }
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
    const unsigned long long myword = lane < k ? biased_word(key, lane, v, layer) : 0ull;  // all draws at once
    unsigned long long tot = 0;  // scanned once, then updated in place (as above)
#pragma unroll
    for (int j = 0; j < BSEG; ++j) tot += cs[j];
    unsigned long long incl = warp_incl_scan_u64(tot);
    unsigned long long W = __shfl_sync(FULL_MASK, incl, 31);
    for (int t = 0; t < k; ++t) {
      const unsigned long long r = __umul64hi(__shfl_sync(FULL_MASK, myword, t), W);
      const int L = __ffs(__ballot_sync(FULL_MASK, incl > r)) - 1;
      int cstar = 0;
      unsigned long long before = 0;  // weight of the chunks before the crossing one
      if (lane == L) {
        unsigned long long acc = incl - tot;
        bool done = false;
#pragma unroll
        for (int j = 0; j < BSEG; ++j) {
          if (!done && acc + cs[j] > r) {
            cstar = lane * T + j;
            before = acc;
            done = true;
          }
          acc += cs[j];
        }
      }
      cstar = __shfl_sync(FULL_MASK, cstar, L);
      before = __shfl_sync(FULL_MASK, before, L);
      const int p = cstar * 32 + lane;
      bool taken = p >= d;
      for (int j = 0; j < t; ++j) taken |= __shfl_sync(FULL_MASK, pick, j) == (uint32_t)p;
      const unsigned long long val = taken ? 0ull : (unsigned long long)__ldg(a + min(p, d - 1));
      const unsigned long long pin = warp_incl_scan_u64(val);
      const int P2 = __ffs(__ballot_sync(FULL_MASK, before + pin > r)) - 1;
      const uint32_t found = (uint32_t)(cstar * 32 + P2);
      const unsigned long long wfound = __shfl_sync(FULL_MASK, val, P2);
      if (lane == L) {
#pragma unroll
        for (int j = 0; j < BSEG; ++j)
          if (j == cstar - lane * T) cs[j] -= wfound;  // remove the pick
        tot -= wfound;
      }
      if (lane >= L) incl -= wfound;
      W -= wfound;
      if (lane == t) pick = found;
    }
    *pos = biased_sort_picks(pick, k);
    return k;
  }
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
    const unsigned long long r = __umul64hi(biased_word(key, t, v, layer), W);
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

}  // namespace dsp
