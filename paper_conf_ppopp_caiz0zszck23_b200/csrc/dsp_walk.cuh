// dsp_walk.cuh -- random walks over a partitioned graph (world > 1).
//
// P:L184 (Sec. 4.2): "random walk can be implemented as a special case of
// node-wise sampling, whose fan-out is 1 for all layers.  Termination
// conditions can be introduced to determine whether a random walk should
// continue in the shuffle stage, and the reshuffle stage can be removed."
//
// CSP push without reshuffle: a walker (walk id, current node v) is moved to
// the owner of v (shuffle, through the owner's peer-mapped inbox); the owner
// takes the step -- the fan-out-1 node-wise pick of v at step l (DESIGN.md
// R27), identical to the world-1 kernel -- writes the new node straight into
// the trace row of the walk's ORIGIN rank (peer store, no reshuffle round),
// and keeps the walker for the next shuffle.  A walker whose node has no
// neighbours terminates (its trace rows stay -1).  Per step one exchange
// round: counts + header + release flag per (parity, sender), as the CSP
// shuffle.
#pragma once
#include "dsp_kernels.cuh"

namespace dsp {

constexpr int WALK_RANK_SHIFT = 27;  // walk id = origin rank << 27 | walk index
constexpr int32_t WALK_MAX = 1 << WALK_RANK_SHIFT;

// Peer-visible walk region of a rank (library-owned, CUDA-IPC mapped by every peer).
struct WalkLayout {
  int64_t cap;            // walkers per (parity, sender) inbox = world * max_walks
  int64_t max_walks;      // per origin
  int32_t max_len;        // steps (trace row = max_len + 1 entries)
  size_t off_flag;        // u64 [2][8]  inbox flags (parity, sender)
  size_t off_done;        // u64 [8]     "all my steps are done" flags (sender)
  size_t off_hdr;         // uint4 [2][8] {count, length, seed lo, seed hi}
  size_t off_inbox;       // int2 [2][8][cap]
  size_t off_trace;       // i32 [max_walks][max_len + 1] traces of this rank's walks
  size_t off_list;        // int2 [2][cap] walkers kept at this rank (local use only)
  size_t off_ctr;         // u32 [16]  list counts [2], bucket counters [8], done counter
  size_t bytes;
};

struct WalkPeers {
  char *base[8];
};

__device__ __forceinline__ unsigned long long *walk_flag(char *b, const WalkLayout &L, int p, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_flag) + p * 8 + s;
}
__device__ __forceinline__ unsigned long long *walk_done(char *b, const WalkLayout &L, int s) {
  return reinterpret_cast<unsigned long long *>(b + L.off_done) + s;
}
__device__ __forceinline__ uint4 *walk_hdr(char *b, const WalkLayout &L, int p, int s) {
  return reinterpret_cast<uint4 *>(b + L.off_hdr) + p * 8 + s;
}
__device__ __forceinline__ int2 *walk_inbox(char *b, const WalkLayout &L, int p, int s) {
  return reinterpret_cast<int2 *>(b + L.off_inbox) + ((int64_t)p * 8 + s) * L.cap;
}
__device__ __forceinline__ int32_t *walk_trace(char *b, const WalkLayout &L) {
  return reinterpret_cast<int32_t *>(b + L.off_trace);
}
__device__ __forceinline__ int2 *walk_list(char *b, const WalkLayout &L, int p) {
  return reinterpret_cast<int2 *>(b + L.off_list) + (int64_t)p * L.cap;
}
__device__ __forceinline__ uint32_t *walk_ctr(char *b, const WalkLayout &L) {
  return reinterpret_cast<uint32_t *>(b + L.off_ctr);
}
// counters: [0..1] list count per parity, [2..9] bucket per owner, [10] last-block counter

struct WalkArgs {
  const int32_t *starts;
  int64_t n;
  int32_t length, step, rank, parity;
  unsigned long long seq;   // flag value of this round
  uint2 key;
  const int64_t *indptr;
  const int32_t *indices;
  int64_t lo, n_local;
  Bounds bd;
  WalkLayout L;
  WalkPeers peers;
  int32_t *traces;          // caller's output (finish)
  int *err;
  int32_t independent;      // DSP_WALK_INDEPENDENT: draws keyed by the walk index (R35)
};

// Origin: trace rows := -1, column 0 := start, walkers of step 0 := the
// valid starts (list parity 0).
__device__ __forceinline__ void walk_init_body(const WalkArgs &a) {
  char *self = a.peers.base[a.rank];
  int32_t *tr = walk_trace(self, a.L);
  uint32_t *ctr = walk_ctr(self, a.L);
  const int64_t W = a.L.max_len + 1;
  const int64_t N = a.bd.b[a.bd.world];
  for (int64_t e = blockIdx.x * (int64_t)NT + threadIdx.x; e < a.n * (a.length + 1); e += (int64_t)gridDim.x * NT) {
    const int64_t i = e / (a.length + 1), c = e - i * (a.length + 1);
    int32_t v = -1;
    if (c == 0) {
      v = __ldg(a.starts + i);
      if (v < 0 || v >= N) {
        latch(a.err, E_RANGE);
        v = -1;
      } else {
        const uint32_t slot = atomicAdd(&ctr[0], 1u);
        walk_list(self, a.L, 0)[slot] = make_int2((int32_t)(((uint32_t)a.rank << WALK_RANK_SHIFT) | (uint32_t)i), v);
      }
    }
    tr[i * W + c] = v;
  }
}

// Shuffle of step l: every walker kept here goes to the owner of its node
// (inbox slot order irrelevant); the last block publishes counts + header,
// then the flags.  The list is consumed (its count reset for step l + 1).
// round of a call: step, flag value, parity (per-launch in the stage kernels, per
// iteration in k_walk_multi, whose WalkArgs stay in the grid-constant parameter space)
struct WalkRound {
  int32_t step, parity;
  unsigned long long seq;
};

__device__ __forceinline__ void walk_scatter_body(const WalkArgs &a, const WalkRound rd) {
  __shared__ uint32_t s_cnt[8], s_base[8];
  char *self = a.peers.base[a.rank];
  uint32_t *ctr = walk_ctr(self, a.L);
  const int lp = rd.step & 1;
  const uint32_t n = *(volatile uint32_t *)&ctr[lp];
  const int2 *list = walk_list(self, a.L, lp);
  for (uint32_t b0 = blockIdx.x * NT; b0 < ((n + NT - 1) / NT) * NT; b0 += gridDim.x * NT) {
    if (threadIdx.x < 8) s_cnt[threadIdx.x] = 0;
    __syncthreads();
    const uint32_t i = b0 + threadIdx.x;
    int o = -1;
    uint32_t local = 0;
    int2 w = make_int2(0, 0);
    if (i < n) {
      w = list[i];
      o = owner_of(a.bd, w.y);
      local = atomicAdd(&s_cnt[o], 1u);
    }
    __syncthreads();
    if (threadIdx.x < a.bd.world) s_base[threadIdx.x] = atomicAdd(&ctr[2 + threadIdx.x], s_cnt[threadIdx.x]);
    __syncthreads();
    if (o >= 0) walk_inbox(a.peers.base[o], a.L, rd.parity, a.rank)[s_base[o] + local] = w;
    __syncthreads();
  }
  if (last_block_done(&ctr[10])) {
    ctr[lp] = 0u;
    for (int o = 0; o < a.bd.world; ++o) {
      const uint32_t c = *(volatile uint32_t *)&ctr[2 + o];
      ctr[2 + o] = 0u;
      *walk_hdr(a.peers.base[o], a.L, rd.parity, a.rank) =
          make_uint4(c, (uint32_t)a.length | ((uint32_t)rd.step << 16) | ((uint32_t)a.independent << 30), a.key.x,
                     a.key.y);
    }
    __threadfence_system();
    for (int o = 0; o < a.bd.world; ++o) st_release_sys(walk_flag(a.peers.base[o], a.L, rd.parity, a.rank), rd.seq);
  }
}

// Step l at the owner: every received walker takes its fan-out-1 step; the
// new node goes to trace[l + 1] of the walk at its origin (peer store); a
// walker that can continue stays here (list parity l + 1).
__device__ __forceinline__ void walk_step_body(const WalkArgs &a, const WalkRound rd) {
  __shared__ uint32_t s_off[9];
  char *self = a.peers.base[a.rank];
  const int world = a.bd.world;
  uint32_t *ctr = walk_ctr(self, a.L);
  if (wait_flags(walk_flag(self, a.L, rd.parity, 0), world, rd.seq, a.err)) {
    if (threadIdx.x == 0) {
      uint32_t acc = 0;
      for (int s = 0; s < world; ++s) {
        const uint4 h = __ldcv(walk_hdr(self, a.L, rd.parity, s));
        if (h.y != ((uint32_t)a.length | ((uint32_t)rd.step << 16) | ((uint32_t)a.independent << 30)) ||
            h.z != a.key.x || h.w != a.key.y)
          latch(a.err, E_STATE);
        s_off[s] = acc;
        acc += h.x <= (uint32_t)a.L.cap ? h.x : 0u;
      }
      s_off[world] = acc;
    }
    __syncthreads();
    const uint32_t total = s_off[world];
    const int64_t W = a.L.max_len + 1;
    const int lane = threadIdx.x & 31;
    int2 *next = walk_list(self, a.L, (rd.step + 1) & 1);
    for (uint32_t b0 = blockIdx.x * NT; b0 < ((total + NT - 1) / NT) * NT; b0 += gridDim.x * NT) {
      const uint32_t q = b0 + threadIdx.x;
      bool keep = false;
      int2 w = make_int2(0, -1);
      if (q < total) {
        int s = 0;
        while (s + 1 < world && q >= s_off[s + 1]) ++s;
        w = __ldcv(walk_inbox(self, a.L, rd.parity, s) + (q - s_off[s]));
        const int64_t lv = (int64_t)w.y - a.lo;
        int32_t u = -1;
        if (lv < 0 || lv >= a.n_local) {
          latch(a.err, E_STATE);  // routed to the wrong owner
        } else {
          int64_t rs, d;
          row_extent(a.indptr, lv, &rs, &d);
          const uint32_t wi = (uint32_t)w.x & (uint32_t)(WALK_MAX - 1);  // index in the origin's starts
          if (d > 0)
            u = __ldg(a.indices + rs +
                      (d == 1          ? 0u
                       : a.independent ? walk_draw(a.key, wi, w.y, rd.step, (uint32_t)d)
                                       : draw_range(a.key, 0u, w.y, rd.step, (uint32_t)d)));
        }
        const int origin = (int)((uint32_t)w.x >> WALK_RANK_SHIFT);
        const int64_t i = (int64_t)((uint32_t)w.x & (uint32_t)(WALK_MAX - 1));
        walk_trace(a.peers.base[origin], a.L)[i * W + rd.step + 1] = u;
        keep = u >= 0;
        w.y = u;
      }
      // warp-aggregated append of the walkers that continue
      const unsigned m = __ballot_sync(FULL_MASK, keep);
      uint32_t base = 0;
      if (lane == 0 && m) base = atomicAdd(&ctr[(rd.step + 1) & 1], (uint32_t)__popc(m));
      base = __shfl_sync(FULL_MASK, base, 0);
      if (keep) next[base + __popc(m & ((1u << lane) - 1u))] = w;
    }
  }
  __threadfence_system();  // this step's peer trace stores before the next round's flags
}

// After the last step: tell every rank that this rank's trace stores are done.
__device__ __forceinline__ void walk_done_body(const WalkArgs &a, const WalkRound rd) {
  if (threadIdx.x == 0) {
    uint32_t *ctr = walk_ctr(a.peers.base[a.rank], a.L);
    ctr[0] = ctr[1] = 0u;  // walkers left after the last step are dropped
    __threadfence_system();
    for (int o = 0; o < a.bd.world; ++o) st_release_sys(walk_done(a.peers.base[o], a.L, a.rank), rd.seq);
  }
}

// Origin: once every rank is done, copy the trace rows to the caller.
__device__ __forceinline__ void walk_finish_body(const WalkArgs &a, const WalkRound rd) {
  char *self = a.peers.base[a.rank];
  if (!wait_flags(walk_done(self, a.L, 0), a.bd.world, rd.seq, a.err)) return;
  const int32_t *tr = walk_trace(self, a.L);
  const int64_t W = a.L.max_len + 1, w = a.length + 1;
  for (int64_t e = blockIdx.x * (int64_t)NT + threadIdx.x; e < a.n * w; e += (int64_t)gridDim.x * NT) {
    const int64_t i = e / w, c = e - i * w;
    a.traces[e] = __ldcv(tr + i * W + c);
  }
}


// The whole multi-rank walk call in ONE cooperative launch per rank: init,
// then per step the shuffle (its last block publishes the inbox flags) and the
// step at the owners (waiting on every rank's flag inside the kernel: all
// ranks' kernels are resident), a grid barrier before the next step's shuffle
// reads the list the step appended to, then done flags and the trace copy.
struct WalkPersistArgs {
  WalkArgs a;
  unsigned long long seq0;
  WsHeader *hdr;            // grid-barrier counter (zeroed by the host before the launch)
};

__global__ void __launch_bounds__(NT) k_walk_multi(const __grid_constant__ WalkPersistArgs p) {
  const WalkArgs &a = p.a;
  uint32_t bar = 0;
  walk_init_body(a);
  grid_barrier<NT>(p.hdr, bar);
  for (int l = 0; l < a.length; ++l) {
    const unsigned long long seq = p.seq0 + 1 + (unsigned long long)l;
    const WalkRound rd{l, (int32_t)(seq & 1ull), seq};
    walk_scatter_body(a, rd);
    walk_step_body(a, rd);
    grid_barrier<NT>(p.hdr, bar);
  }
  const WalkRound fin{a.length, 0, p.seq0 + 1 + (unsigned long long)a.length};
  if (blockIdx.x == 0) walk_done_body(a, fin);
  walk_finish_body(a, fin);
}

}  // namespace dsp
