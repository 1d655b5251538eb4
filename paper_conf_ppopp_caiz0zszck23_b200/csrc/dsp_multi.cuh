// dsp_multi.cuh -- world > 1: the whole CSP call of one rank in ONE persistent
// cooperative kernel (sm_100a), the exchanges done inside it over NVLink peer
// memory.
//
// Per layer l (Fig. 5), with grid barriers (GB) between phases:
//   A  shuffle   : group the frontier by owner (contiguous id ranges),
//                  write each id straight into the owner's inbox (peer store),
//                  perm[i] = its inbox slot;  [indices of layer l-1 meanwhile]
//                  -- GB with fence.sys, block 0 publishes counts + header and the
//                  inbox flag of every owner (count notification)
//   B  sample    : wait for every rank's inbox flag; sample every received
//                  task (one phase over all tasks) and write the row
//                  straight into the requester's return slot (reshuffle)
//                  -- GB with fence.sys, block 0 releases the return flags
//   C  unpermute : wait for every owner's return flag; frontier node i takes
//                  its row from slot perm[i] of its owner, writes the edge
//                  slots and marks the relabel map (as the local sampler does)
//                  -- GB
//   D  scan      : the two-pass relabel scan of the world-1 kernel -- GB
// then the last layer's indices and the gather (fused, or pipelined: loader
// warps read the PREVIOUS call's rows from the owners' shards while this
// call samples -- the paper's loader(t-1) || sampler(t)).
//
// Compared with the stage-by-stage path (k_bucket_scatter .. k_write_indices,
// 5 launches per layer) this removes the per-kernel launch / drain / refill
// and the system fence of every block of every stage kernel: one launch per
// call, 148 fences per exchange.  Waiting inside a kernel on a peer's kernel
// is safe because every rank's kernel is fully resident (cooperative launch on
// its own GPU; virtual ranks sharing a GPU each get 1/P of the SMs on their
// own stream), and every wait is bounded (20 s, then E_STATE and an abort
// word that ends every later wait of the call at once: never a hung GPU).
//
// The results are the same as the staged path's (same draws, same slots,
// same relabel), checked against the oracle in tests/test_gpu_parity.py.
#pragma once
#include "dsp_kernels.cuh"

namespace dsp {

struct MultiArgs {
  PersistArgs p;            // the world-1 persistent kernel's arguments
  int32_t rank;
  unsigned long long seq0;  // exchange sequence number before this call (layer l uses seq0 + 1 + l)
  Bounds bd;
  XchLayout X;
  XchPeers peers;
  int32_t *perm;            // [F] inbox slot of frontier node i at its owner
  int32_t *abort_word;      // set when a wait timed out: later waits of this call end at once
  uint32_t call_tag;        // low byte of the ctx's collective call count: ranks must agree
};

// Thread 0 of each block waits until flags[s] >= seq for every rank s; the
// block then proceeds (bar.sync after the acquire).  Bounded: E_STATE + abort.
template <int TEAM>
__device__ __forceinline__ void multi_wait(unsigned long long *flags0, int world, unsigned long long seq, int *err,
                                           int32_t *abort_word) {
  if (threadIdx.x == 0) {
    const unsigned long long t0 = globaltimer_ns();
    for (int s = 0; s < world; ++s) {
      while (ld_acquire_sys(flags0 + s) < seq) {
        if (*(volatile int32_t *)abort_word) return;
        if (globaltimer_ns() - t0 > WAIT_TIMEOUT_NS) {
          latch(err, E_STATE);
          *(volatile int32_t *)abort_word = 1;
          break;
        }
        __nanosleep(32);
      }
    }
  }
}

// A: shuffle.  Each block scatters its contiguous chunk of the frontier,
// TEAM ids per round: a shared-memory owner histogram and one global counter
// add per owner and round give every id its inbox slot; the round's ids are
// then staged in shared memory grouped by owner, so the peer stores go out as
// contiguous runs (coalesced NVLink writes) instead of one scattered 4-byte
// store per id.
template <int TEAM>
__device__ __forceinline__ void multi_scatter(const MultiArgs &m, const int32_t *frontier, int F, int par,
                                              uint32_t *s_cnt, uint32_t *s_base) {
  __shared__ int32_t s_stage[TEAM];
  __shared__ uint32_t s_pre[9];
  const PersistArgs &a = m.p;
  const Span sp = block_span<TEAM>(F);
  const int64_t b0 = sp.first - threadIdx.x;
  const int world = m.bd.world;
  const int32_t N = (int32_t)m.bd.b[world];
  for (int64_t r0 = b0; r0 < sp.end; r0 += TEAM) {
    if (threadIdx.x < 8) s_cnt[threadIdx.x] = 0;
    team_sync<TEAM>();
    const int64_t i = r0 + threadIdx.x;
    int o = -1;
    uint32_t local = 0;
    int32_t v = 0;
    if (i < sp.end) {
      v = ldw_i32(frontier + i);
      if (v < 0 || v >= N) {
        latch(a.err, E_RANGE);
      } else {
        o = owner_of(m.bd, v);
        local = atomicAdd(&s_cnt[o], 1u);
      }
    }
    team_sync<TEAM>();
    if (threadIdx.x < world && s_cnt[threadIdx.x])
      s_base[threadIdx.x] = atomicAdd(&a.hdr->bucket[threadIdx.x], s_cnt[threadIdx.x]);
    if (threadIdx.x == 32) {  // staging offsets of the owners' runs
      uint32_t acc = 0;
      for (int q = 0; q < world; ++q) {
        s_pre[q] = acc;
        acc += s_cnt[q];
      }
      s_pre[world] = acc;
    }
    team_sync<TEAM>();
    if (o >= 0) {
      s_stage[s_pre[o] + local] = v;
      m.perm[i] = (int32_t)(s_base[o] + local);
    }
    team_sync<TEAM>();
    const uint32_t t = threadIdx.x;
    if (t < s_pre[world]) {  // staged position t -> owner q, slot s_base[q] + (t - s_pre[q])
      int q = 0;
      while (q + 1 < world && t >= s_pre[q + 1]) ++q;
      xch_inbox(m.peers.base[q], m.X, par, m.rank)[s_base[q] + (t - s_pre[q])] = s_stage[t];
    }
  }
}

// B: the owner's sample of every received task.  Tasks are numbered over the
// senders (s_off = prefix of the per-sender counts); thread per task for
// k <= KB (draws, Floyd and ranking in registers, as phase_sample_tpn).  The
// count goes straight to the requester's return slot j; the row (slot order,
// row j of the requester's return rows at stride k) is staged in shared
// memory for the block's round of TEAM tasks and then copied out as one
// contiguous run per requester (coalesced NVLink stores).
template <int KB, int TEAM>
__device__ __forceinline__ void multi_sample_tpn(const MultiArgs &m, int T, const uint32_t *s_off, int layer, int k,
                                                 int par) {
  constexpr bool STAGE = KB <= 8;  // k <= 8 (the largest layer): staged; k <= 16: direct stores
  __shared__ int32_t s_rows[STAGE ? TEAM * KB : 1];
  const PersistArgs &a = m.p;
  const int world = m.bd.world;
  char *self = m.peers.base[m.rank];
  const Span sp = block_span<TEAM>(T);
  const int64_t b0 = sp.first - threadIdx.x;
  for (int64_t r0 = b0; r0 < sp.end; r0 += TEAM) {  // block-uniform rounds
    const int q = (int)(r0 + threadIdx.x);
    if (q < sp.end) {
      int s = 0;
      while (s + 1 < world && (uint32_t)q >= s_off[s + 1]) ++s;
      const int j = q - (int)s_off[s];
      const int32_t v = __ldcv(xch_inbox(self, m.X, par, s) + j);
      const int64_t lv = (int64_t)v - a.lo;
      char *req = m.peers.base[s];
      if (lv < 0 || lv >= a.n_local) {  // routed to the wrong owner: protocol error
        latch(a.err, E_STATE);
        xch_ret_cnt(req, m.X, par, m.rank)[j] = 0;
      } else {
        int64_t rs, d;
        row_extent(a.indptr, lv, &rs, &d);
        const bool full = d <= k;
        const int cnt = full ? (int)d : k;
        uint32_t pos[KB];
#pragma unroll
        for (int t = 0; t < KB; ++t) pos[t] = (uint32_t)t;
        if (!full) {
#pragma unroll
          for (int t = 0; t < KB; ++t)
            if (t < k) pos[t] = draw_range(a.key, (uint32_t)t, v, layer, (uint32_t)(d - k + t + 1));
#pragma unroll
          for (int t = 1; t < KB; ++t) {
            if (t < k) {
              bool hit = false;
#pragma unroll
              for (int qx = 0; qx < t; ++qx) hit |= (pos[qx] == pos[t]);
              if (hit) pos[t] = (uint32_t)(d - k + t);
            }
          }
        }
        int32_t u[KB];
        unsigned long long slots = 0;
#pragma unroll
        for (int t = 0; t < KB; ++t) {
          uint32_t r = 0;
#pragma unroll
          for (int qx = 0; qx < KB; ++qx) r += (qx < cnt && pos[qx] < pos[t]) ? 1u : 0u;
          slots |= (unsigned long long)r << (4 * t);
          u[t] = (t < cnt) ? adj_ld(a.indices + rs + pos[t]) : 0;
        }
        xch_ret_cnt(req, m.X, par, m.rank)[j] = cnt;
        int32_t *row = STAGE ? s_rows + (int64_t)threadIdx.x * k : xch_ret_rows(req, m.X, par, m.rank) + (int64_t)j * k;
#pragma unroll
        for (int t = 0; t < KB; ++t)
          if (t < cnt) row[(slots >> (4 * t)) & 15u] = u[t];
      }
    }
    if (!STAGE) continue;
    team_sync<TEAM>();
    // copy-out: the round's tasks [r0, r1) split into one contiguous run per requester
    const int64_t r1 = min(sp.end, r0 + TEAM);
    for (int s = 0; s < world; ++s) {
      const int64_t q0 = max(r0, (int64_t)s_off[s]), q1 = min(r1, (int64_t)s_off[s + 1]);
      if (q0 >= q1) continue;
      int32_t *dst = xch_ret_rows(m.peers.base[s], m.X, par, m.rank) + (q0 - (int64_t)s_off[s]) * k;
      const int32_t *src = s_rows + (q0 - r0) * k;
      const int64_t len = (q1 - q0) * k;
      for (int64_t e = threadIdx.x; e < len; e += TEAM) dst[e] = src[e];
    }
    team_sync<TEAM>();
  }
}

// B with a lane group of G lanes per task (G = next pow2 >= k): k > 16, and
// small task counts (the first layers), where a thread per task would run its
// k Philox draws back to back with few warps busy.  Biased: warp per task.
template <int G, int TEAM>
__device__ __forceinline__ void multi_sample_lanes(const MultiArgs &m, int T, const uint32_t *s_off, int layer, int k,
                                                   int par) {
  const PersistArgs &a = m.p;
  const int world = m.bd.world;
  char *self = m.peers.base[m.rank];
  constexpr int NPW = 32 / G;
  const int lane = threadIdx.x & 31;
  const bool leader = (lane & (G - 1)) == 0;
  const Span sp = block_span<TEAM>(T);
  const int64_t b0 = sp.first - threadIdx.x;
  const int wib = threadIdx.x >> 5, wpb = TEAM >> 5;
  for (int64_t base = b0 + (int64_t)wib * NPW; base < sp.end; base += (int64_t)wpb * NPW) {
    const int q = (int)(base + lane / G);
    const bool active = q < sp.end;
    int s = 0;
    if (active)
      while (s + 1 < world && (uint32_t)q >= s_off[s + 1]) ++s;
    const int j = q - (int)s_off[s];
    const int32_t v = active ? __ldcv(xch_inbox(self, m.X, par, s) + j) : 0;
    const int64_t lv = (int64_t)v - a.lo;
    const bool ok = active && lv >= 0 && lv < a.n_local;
    if (active && !ok && leader) latch(a.err, E_STATE);
    int64_t rs = 0, d = 0;
    if (ok) row_extent(a.indptr, lv, &rs, &d);
    bool valid;
    int slot, cnt;
    int32_t u;
    if (G == 32 && a.biased) {
      uint32_t pos;
      const unsigned long long word = lane < k ? biased_word(a.key, lane, v, layer) : 0ull;
      cnt = sample_node_biased(ok, v, rs, d, k, layer, a.key, a.weights, word, 0, &pos, &slot);
      valid = lane < cnt;
      u = valid ? __ldg(a.indices + rs + pos) : -1;
    } else {
      sample_node<G>(ok, v, rs, d, k, layer, a.key, a.indices, &valid, &slot, &u, &cnt);
    }
    char *req = m.peers.base[s];
    if (active && leader) xch_ret_cnt(req, m.X, par, m.rank)[j] = cnt;
    if (valid) xch_ret_rows(req, m.X, par, m.rank)[(int64_t)j * k + slot] = u;
  }
}

// B for biased sampling: as phase_sample_biased (biased_claim on
// runs of 32 tasks of the block's share, lane groups for rows of <= 256
// positions), the rows written into the requesters' return slots.
struct BiasedOutMulti {
  const MultiArgs &m;
  int par, k, sl, jl;  // this lane's task of the claim: requester rank, index in its list
  struct Ctx {
    int32_t *rows;
    int32_t *cnt;
  };
  __device__ __forceinline__ Ctx ctx(int jn) const {
    const int s = __shfl_sync(FULL_MASK, sl, jn), j = __shfl_sync(FULL_MASK, jl, jn);
    char *req = m.peers.base[s];
    return Ctx{xch_ret_rows(req, m.X, par, m.rank) + (int64_t)j * k, xch_ret_cnt(req, m.X, par, m.rank) + j};
  }
  __device__ __forceinline__ void node(const Ctx &c, int32_t, bool, int cnt) const { *c.cnt = cnt; }
  __device__ __forceinline__ void edge(const Ctx &c, int slot, int32_t u) const { c.rows[slot] = u; }
};

template <int TEAM>
__device__ __forceinline__ void multi_sample_biased(const MultiArgs &m, int T, const uint32_t *s_off, int layer,
                                                    int k, int par) {
  const PersistArgs &a = m.p;
  const int world = m.bd.world;
  char *self = m.peers.base[m.rank];
  const int lane = threadIdx.x & 31;
  const Span sp = block_span<TEAM>(T);
  const int64_t b0 = sp.first - threadIdx.x;
  const int wib = threadIdx.x >> 5, wpb = TEAM >> 5;
  for (int64_t g0 = b0 + wib; g0 < sp.end; g0 += (int64_t)wpb * 32) {
    const int64_t ql = g0 + (int64_t)lane * wpb;
    int sl = 0, jl = 0;
    int32_t vl = 0;
    bool okl = false;
    int64_t rsl = 0, dl = 0;
    if (ql < sp.end) {
      while (sl + 1 < world && (uint32_t)ql >= s_off[sl + 1]) ++sl;
      jl = (int)ql - (int)s_off[sl];
      vl = __ldcv(xch_inbox(self, m.X, par, sl) + jl);
      const int64_t lv = (int64_t)vl - a.lo;
      okl = lv >= 0 && lv < a.n_local;
      if (!okl) latch(a.err, E_STATE);  // routed to the wrong owner
      else row_extent(a.indptr, lv, &rsl, &dl);
    }
    const int nn = (int)min((int64_t)32, (sp.end - g0 + wpb - 1) / wpb);
    const BiasedOutMulti out{m, par, k, sl, jl};
    biased_claim(nn, vl, okl, rsl, dl, k, layer, a.key, a.weights, a.indices, out);
  }
}

// C: frontier node i (thread per node) reads its row from its owner's return
// slot perm[i]: counts, edge slots, dst copy and relabel marks.
template <int TEAM>
__device__ __forceinline__ void multi_unpermute(const MultiArgs &m, const int32_t *frontier, int F, int layer, int k,
                                                int par, uint32_t epoch) {
  const PersistArgs &a = m.p;
  const LayerBufs &B = a.buf[layer & 1];
  int32_t *src_out = a.out.src_ids[layer];
  const int32_t N = (int32_t)m.bd.b[m.bd.world];
  const Span sp = block_span<TEAM>(F);
  for (int64_t ii = sp.first; ii < sp.end; ii += sp.step) {
    const int i = (int)ii;
    const int32_t v = ldw_i32(frontier + i);
    src_out[i] = v;  // dst copy (R17)
    if (v < 0 || v >= N) {  // latched by the shuffle
      B.cnt[i] = 0;
      continue;
    }
    const int o = owner_of(m.bd, v);
    const int j = ldw_i32(m.perm + i);
    int c = __ldcv(xch_ret_cnt(m.peers.base[m.rank], m.X, par, o) + j);
    c = c < 0 ? 0 : (c > k ? k : c);  // a failed exchange (E_STATE) leaves stale slots: never write past k
    const int32_t *row = xch_ret_rows(m.peers.base[m.rank], m.X, par, o) + (int64_t)j * k;  // rows at stride k
    B.cnt[i] = c;
    mark_dst(B, v, i, F, layer, epoch, a.err);
    const uint32_t q0 = (uint32_t)i * (uint32_t)k;
    if (k <= 16) {
      int32_t u[16];
#pragma unroll
      for (int t = 0; t < 16; ++t) u[t] = t < c ? __ldcv(row + t) : 0;
#pragma unroll
      for (int t = 0; t < 16; ++t)
        if (t < c) {
          B.rows[q0 + t] = u[t];
          mark(B, u[t], epoch, (uint32_t)F + q0 + (uint32_t)t);
        }
    } else {
      for (int t = 0; t < c; ++t) {
        const int32_t u = __ldcv(row + t);
        B.rows[q0 + t] = u;
        mark(B, u, epoch, (uint32_t)F + q0 + (uint32_t)t);
      }
    }
  }
}

template <int TEAM, bool PIPE, bool BIASED>
__global__ void __launch_bounds__(PNT, 1) k_csp_multi(const __grid_constant__ MultiArgs m) {
  __shared__ Scan2Smem<TEAM, SCAN2_GROUPS> sm;
  __shared__ uint32_t s_cnt[8], s_base[8], s_off[9];
  __shared__ __align__(8) uint64_t bars[LOADER_WARPS][LOADER_SLOTS];
  extern __shared__ __align__(128) char ring_smem[];
  const PersistArgs &a = m.p;
  const int blk = blockIdx.x, nblk = gridDim.x;
  const int world = m.bd.world;

  if (PIPE && threadIdx.x >= TEAM) {  // ------ loader warps: previous call's rows from every owner (TMA)
    const int w = (threadIdx.x - TEAM) >> 5;
    if ((threadIdx.x & 31) == 0)
      for (int s2 = 0; s2 < LOADER_SLOTS; ++s2) mbar_init(&bars[w][s2], 1);
    mbar_init_fence();
    __syncwarp();
    if (a.prev) loader_warp<true>(a, ring_smem + (size_t)w * LOADER_SLOTS * a.slot_bytes, bars[w],
                                  ld_volatile_i32(a.gp.n_dev));
    return;
  }

  const int64_t tid = blockIdx.x * (int64_t)TEAM + threadIdx.x;
  const int64_t nthreads = (int64_t)gridDim.x * TEAM;
  uint32_t bar = 0;
  uint32_t e0 = *(volatile const uint32_t *)&a.persist->epoch;
  if (a.buf[0].first32) e0 = dwin_start(e0, (uint32_t)a.L);
  const bool hclear = hash_clear_due(a.persist, e0, (uint32_t)a.L, a.buf[0].mask, a.buf[0].first);
  const bool dclear = a.buf[0].first32 && dclear_due(a.persist, e0);
  if (hclear || dclear) {  // zero the relabel map (once per ~255 / L calls)
    map_zero(a.buf[0], tid, nthreads);
    grid_barrier<TEAM>(a.hdr, bar);
  }
  if (tid == 0) {
    a.hdr->t[0] = globaltimer_ns();
    a.hdr->F[0] = a.B;
  }
  char *self = m.peers.base[m.rank];
  int F = a.B;
  int Fprev = 0;
  for (int l = 0; l < a.L; ++l) {
    const uint32_t epoch = e0 + 1 + l;
    const unsigned long long seq = m.seq0 + 1 + (unsigned long long)l;
    const int par = (int)(seq & 1ull);
    const int32_t *frontier = l == 0 ? a.seeds : a.out.src_ids[l - 1];
    const int k = a.k[l];
    const int Fs = F > m.X.cap ? 0 : F;  // capacity overflow: send nothing (latched below)
    if (F > m.X.cap && tid == 0) latch(a.err, E_CAP);

    // ---- A: shuffle (+ the previous layer's duplicate indices)
    multi_scatter<TEAM>(m, frontier, Fs, par, s_cnt, s_base);
    if (l > 0)
      phase_indices_dups(Fprev, a.k[l - 1], a.buf[(l - 1) & 1], a.out.indptr[l - 1], a.out.indices[l - 1],
                         block_span<TEAM>((int64_t)Fprev * a.k[l - 1]));
    grid_barrier<TEAM, true>(a.hdr, bar);  // + fence.sys: the block's peer stores precede the flag
    if (blk == 0 && threadIdx.x == 0) {
      for (int o = 0; o < world; ++o) {
        const uint32_t c = *(volatile uint32_t *)&a.hdr->bucket[o];
        a.hdr->bucket[o] = 0u;
        *xch_inbox_hdr(m.peers.base[o], m.X, par, m.rank) =
            make_uint4(c, (uint32_t)k | ((uint32_t)l << 8) | ((uint32_t)a.biased << 16) | (m.call_tag << 24), a.key.x,
                       a.key.y);
      }
      __threadfence_system();
      for (int o = 0; o < world; ++o) st_release_sys(xch_inbox_flag(m.peers.base[o], m.X, par, m.rank), seq);
    }

    // ---- B: sample every task received from any rank
    multi_wait<TEAM>(xch_inbox_flag(self, m.X, par, 0), world, seq, a.err, m.abort_word);
    if (threadIdx.x == 0) {
      uint32_t acc = 0;
      for (int s = 0; s < world; ++s) {
        const uint4 h = __ldcv(xch_inbox_hdr(self, m.X, par, s));
        if (h.y != ((uint32_t)k | ((uint32_t)l << 8) | ((uint32_t)a.biased << 16) | (m.call_tag << 24)) ||
            h.z != a.key.x || h.w != a.key.y)
          latch(a.err, E_STATE);  // ranks disagree on (call, layer, fan-out, seed, scheme)
        s_off[s] = acc;
        acc += (h.x <= (uint32_t)m.X.cap) ? h.x : 0u;
      }
      s_off[world] = *(volatile int32_t *)m.abort_word ? 0u : acc;
    }
    team_sync<TEAM>();
    const int T = (int)s_off[world];
    const int G = k <= 4 ? 4 : k <= 8 ? 8 : 16;
    if (BIASED)  // a template parameter: the uniform kernel carries no biased code
      multi_sample_biased<TEAM>(m, T, s_off, l, k, par);
    else if (k > 16)
      multi_sample_lanes<32, TEAM>(m, T, s_off, l, k, par);
    else if ((int64_t)T * G <= (int64_t)a.lane_rounds * nblk * TEAM)  // few tasks: lane groups
      (G == 4 ? multi_sample_lanes<4, TEAM> : G == 8 ? multi_sample_lanes<8, TEAM> : multi_sample_lanes<16, TEAM>)(
          m, T, s_off, l, k, par);
    else if (k <= 8)
      multi_sample_tpn<8, TEAM>(m, T, s_off, l, k, par);
    else
      multi_sample_tpn<16, TEAM>(m, T, s_off, l, k, par);
    grid_barrier<TEAM, true>(a.hdr, bar);
    if (blk == 0 && threadIdx.x == 0) {
      __threadfence_system();
      for (int s = 0; s < world; ++s) st_release_sys(xch_ret_flag(m.peers.base[s], m.X, par, m.rank), seq);
    }

    // ---- C: rows back in frontier order, relabel marks
    multi_wait<TEAM>(xch_ret_flag(self, m.X, par, 0), world, seq, a.err, m.abort_word);
    team_sync<TEAM>();
    multi_unpermute<TEAM>(m, frontier, Fs, l, k, par, epoch);
    grid_barrier<TEAM>(a.hdr, bar);

    // ---- D: relabel scan (as k_csp_persistent)
    constexpr int64_t TILE = (int64_t)TEAM * SCAN2_IPT * SCAN2_GROUPS;
    const int64_t total = (int64_t)Fs * k;
    const int64_t rounds = total > 0 ? (total + (int64_t)nblk * TILE - 1) / ((int64_t)nblk * TILE) : 1;
    const int64_t per_round = (total + rounds - 1) / rounds;
    const int64_t chunk = (per_round + nblk - 1) / nblk;
    unsigned long long carry = 0;
    for (int64_t r = 0; r < rounds; ++r) {
      Scan2Regs R;
      const int64_t r0 = r * per_round, r1 = min(total, r0 + per_round);
      const int64_t tile0 = min(r1, r0 + (int64_t)blk * chunk), tile_end = min(r1, tile0 + chunk);
      unsigned long long *agg = a.agg + (r & 1) * MAX_PERSIST_BLOCKS;
      scan2_pass1<TEAM, SCAN2_GROUPS>(Fs, k, a.buf[l & 1], epoch, tile0, tile_end, R, agg + blk, sm);
      grid_barrier<TEAM>(a.hdr, bar);
      unsigned long long prefix, round_total;
      scan2_prefix<TEAM, SCAN2_GROUPS>(agg, nblk, blk, sm, &prefix, &round_total);
      scan2_pass2<TEAM, SCAN2_GROUPS>(Fs, k, a.buf[l & 1], tile0, tile_end, R, carry + prefix, sm, a.out.indptr[l],
                        a.out.indices[l], a.out.src_ids[l]);
      carry += round_total;
      if (r + 1 < rounds) grid_barrier<TEAM>(a.hdr, bar);
    }
    const int32_t E = (int32_t)(carry & 0x7fffffffull);
    const int32_t nnew = (int32_t)((carry >> 31) & 0x7fffffffull);
    if (tid == 0) {
      a.out.indptr[l][Fs] = E;
      a.hdr->E[l] = E;
      a.hdr->S[l] = Fs + nnew;
      a.hdr->F[l] = Fs;
      a.hdr->F[l + 1] = Fs + nnew;
      a.hdr->sizes[3 * l + 0] = Fs;
      a.hdr->sizes[3 * l + 1] = Fs + nnew;
      a.hdr->sizes[3 * l + 2] = E;
    }
    Fprev = Fs;
    F = Fs + nnew;
    grid_barrier<TEAM>(a.hdr, bar);
  }
  const int l = a.L - 1;
  phase_indices_dups(Fprev, a.k[l], a.buf[l & 1], a.out.indptr[l], a.out.indices[l],
                     block_span<TEAM>((int64_t)Fprev * a.k[l]));
  if (PIPE) {
    if (tid == 0) *a.pend_n = F;
    if (a.prev) helper_warp<true>(a, ld_volatile_i32(a.gp.n_dev));
  } else if (a.gather) {
    phase_gather<GATHER_UNROLL>(a.g, F, tid, nthreads);
  }
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

}  // namespace dsp
