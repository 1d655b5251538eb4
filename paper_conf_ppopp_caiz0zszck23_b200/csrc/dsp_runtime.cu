// dsp_runtime.cu -- host runtime behind the C ABI of include/dsp.h:
// context, partition load (padded feature rows), peer mapping (CUDA IPC /
// P2P), workspace planning, and the CSP driver that issues the kernels of
// dsp_kernels.cuh.  sm_100a only.
#include <cuda_runtime.h>
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/dsp.h"
#include "dsp_layerwise.cuh"
#include "dsp_multi.cuh"
#include "dsp_walk.cuh"

using namespace dsp;

namespace {

// Every adjacency entry must be a global id in [0, N): the relabel map is
// indexed by it.
__global__ void k_validate_indices(const int32_t *indices, int64_t nnz, int64_t N, int *bad) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t u = indices[e];
    if (u < 0 || u >= N) {
      atomicAdd(bad, 1);
      return;
    }
  }
}

constexpr uint32_t HANDLE_MAGIC = 0x44535048u;  // "DSPH"

// Feature row layout (dsp_kernels.cuh GatherArgs).  Packed (default): a
// region of `slots` rows is one array of rows at stride dim * 4.  Split
// (DSP_OPT_SPLIT_ROWS): each row is cut at its last 128-byte boundary, head =
// dim * 4 rounded down to a multiple of 128 in a packed head array, then
// (256-aligned) the tail (< 128 B) in a packed tail array.
int head_bytes_of(bool split, int dim) { return split ? dim * 4 / 128 * 128 : 0; }
int tail_bytes_of(bool split, int dim) { return dim * 4 - head_bytes_of(split, dim); }
size_t tail_offset(bool split, int64_t slots, int dim) {
  return ((size_t)std::max<int64_t>(1, slots) * (size_t)head_bytes_of(split, dim) + 255) / 256 * 256;
}
size_t region_bytes(bool split, int64_t slots, int dim) {
  return tail_offset(split, slots, dim) + (size_t)std::max<int64_t>(1, slots) * (size_t)tail_bytes_of(split, dim);
}
thread_local std::string g_create_error;

struct PeerHandle {  // fits in DSP_HANDLE_BYTES
  uint32_t magic;
  int32_t rank, world, device;
  int64_t pid;
  uint64_t boot_id;  // distinguishes processes of different hosts / boots
  uint64_t feat_ptr, xch_ptr;
  int64_t feat_bytes, xch_bytes;
  int32_t has_feat, has_xch;
  cudaIpcMemHandle_t feat_ipc, xch_ipc;
  int64_t bounds[DSP_MAX_WORLD + 1];
  int32_t dim, max_seeds, head_bytes, tiered;
  int64_t feat_slots, cold_slots;  // rows of the HBM shard / of the cold region (their tail arrays' offsets)
  cudaIpcMemHandle_t fpos_ipc;
  uint64_t fpos_ptr, cold_ptr;
  int64_t cold_bytes;
  char cold_shm[48];  // POSIX shm name of the cold rows (cross-process access)
  // layer-wise exchange region + this rank's indptr (degree lookups)
  cudaIpcMemHandle_t lxch_ipc, indptr_ipc;
  uint64_t lxch_ptr, indptr_ptr;
  int32_t has_lxch, lw_max_seeds, lw_L, lw_sizes[DSP_MAX_LAYERS];
  // random-walk region (dsp_reserve_walks)
  cudaIpcMemHandle_t wxch_ipc;
  uint64_t wxch_ptr;
  int64_t walk_max;
  int32_t has_wxch, walk_len;
  int32_t channels;  // node-wise exchange channels (DSP_OPT_EXCHANGE_CHANNELS)
};
static_assert(sizeof(PeerHandle) <= DSP_HANDLE_BYTES, "handle too large");

uint64_t boot_id() {
  static uint64_t id = [] {
    uint64_t h = 1469598103934665603ull;
    FILE *f = fopen("/proc/sys/kernel/random/boot_id", "r");
    if (f) {
      int c;
      while ((c = fgetc(f)) != EOF) h = (h ^ (uint64_t)c) * 1099511628211ull;
      fclose(f);
    }
    char host[256] = {0};
    gethostname(host, sizeof(host) - 1);
    for (char *p = host; *p; ++p) h = (h ^ (uint64_t)*p) * 1099511628211ull;
    return h;
  }();
  return id;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

int64_t next_pow2(int64_t x) {
  int64_t p = 1;
  while (p < x) p <<= 1;
  return p;
}

// Per-layer bounds (dsp_sample_bounds) and the workspace plan:
//   persist | hdr | first[2][N] (| first32[2][N] | hash[2][cap]) | agg[2][MAX_PERSIST_BLOCKS]
//   | cnt[2][max_F] | perm[max_F] | rows[2][max_slots]
struct Plan {
  int L;
  int64_t F[DSP_MAX_LAYERS + 1];   // max frontier per layer
  int64_t E[DSP_MAX_LAYERS];       // max edges
  int64_t S[DSP_MAX_LAYERS];       // max src
  int64_t max_F, max_slots;
  size_t off_hdr, off_agg, off_cnt[2], off_perm, off_rows[2], off_first[2], bytes;
  size_t off_first32;               // compact direct map [N] (N <= DIRECT_MAP_MAX_N), else 0
  bool direct32;                    // node-wise relabel through the compact direct map
  int64_t hash_cap;                 // > 0: relabel hash table of hash_cap slots per parity (else direct map)
  size_t off_hash;                  // relabel hash table [hash_cap]
  // layer-wise scheme (make_plan_lw)
  int64_t ncap, big_cap;
  size_t off_P, off_c, off_off, off_slot_node, off_excl, off_newid, off_big;
  size_t off_lxch;                  // world 1: the layer-wise inbox / return slots in the workspace (else 0)
};

}  // namespace

struct dsp_ctx {
  int rank = 0, world = 1, device = 0;
  std::string err;
  bool loaded = false, reserved = false, imported = false, broken = false;
  int64_t bounds[DSP_MAX_WORLD + 1] = {0};
  int64_t N = 0, lo = 0, n_local = 0, nnz = 0;
  int32_t dim = 0;                  // feature row length (floats)
  bool split_rows = false;          // DSP_OPT_SPLIT_ROWS: rows stored split head / tail (head_bytes_of)
  int64_t feat_slots = 0, cold_slots = 0;  // rows in the HBM shard / cold region
  int64_t *d_indptr = nullptr;
  int32_t *d_indices = nullptr;
  uint32_t *d_weights = nullptr;  // 16.16 edge weights (biased sampling)
  float *d_feat = nullptr;
  int64_t feat_bytes = 0;
  // cold-feature tier
  bool tiered = false;
  bool cold_regloads = false;         // DSP_OPT_GATHER_REGLOADS: cold rows by register loads
  int32_t *d_fpos = nullptr;          // feature position list [n_local]
  float *h_cold = nullptr;            // cold rows (pinned host, UVA-mapped)
  int64_t cold_bytes = 0;
  char cold_shm[48] = {0};            // non-empty: h_cold is a registered POSIX shm mapping
  const int32_t *peer_fpos[DSP_MAX_WORLD] = {nullptr};
  const float *peer_cold[DSP_MAX_WORLD] = {nullptr};
  const float *peer_cold_tail[DSP_MAX_WORLD] = {nullptr};
  void *peer_cold_map[DSP_MAX_WORLD] = {nullptr};  // shm mappings opened in this process
  int64_t peer_cold_bytes[DSP_MAX_WORLD] = {0};
  int *d_err = nullptr;  // latched device error of this ctx
  // exchange
  int32_t max_seeds = 0, L = 0, kmax = 0;
  int32_t fanouts[DSP_MAX_LAYERS] = {0};
  XchLayout xl{};
  char *d_xch = nullptr;           // channels x chan_stride bytes, peer-mapped
  // node-wise exchange channels (DSP_OPT_EXCHANGE_CHANNELS): collective call n of
  // this ctx uses channel n % channels with its own exchange region and sequence
  // numbers, so up to `channels` calls can be in flight on different streams; the
  // calls of one channel are ordered by an event (the call issue order, identical
  // on every rank, is the fixed collective order CCC provides)
  int channels = 1;
  size_t chan_stride = 0;
  unsigned long long ncalls = 0;
  unsigned long long chan_seq[DSP_MAX_CHANNELS] = {0};
  cudaEvent_t chan_ev[DSP_MAX_CHANNELS] = {nullptr};
  bool chan_used[DSP_MAX_CHANNELS] = {false};
  // peers
  const float *peer_feat[DSP_MAX_WORLD] = {nullptr};       // head arrays of the ranks' shards
  const float *peer_feat_tail[DSP_MAX_WORLD] = {nullptr};  // tail arrays
  char *peer_xch[DSP_MAX_WORLD] = {nullptr};
  void *ipc_opened[6 * DSP_MAX_WORLD] = {nullptr};  // feat, xch | fpos | lxch | indptr | walk region per peer
  unsigned long long seq = 0;
  // layer-wise scheme (dsp_reserve_layerwise)
  bool lw_reserved = false;
  int32_t lw_max_seeds = 0, lw_L = 0;
  int32_t lw_sizes[DSP_MAX_LAYERS] = {0};
  LwLayout lxl{};
  char *d_lxch = nullptr;
  char *peer_lxch[DSP_MAX_WORLD] = {nullptr};
  const int64_t *peer_indptr[DSP_MAX_WORLD] = {nullptr};
  // random walks over a partitioned graph (dsp_reserve_walks)
  bool walk_reserved = false;
  int64_t walk_max = 0;
  int32_t walk_len = 0;
  WalkLayout wl{};
  char *d_wxch = nullptr;
  char *peer_wxch[DSP_MAX_WORLD] = {nullptr};
  unsigned long long wseq = 0;
  // host staging (pinned)
  WsHeader *h_hdr = nullptr;
  int *h_err = nullptr;
  int num_sms = 148;
  int persist_blocks_per_sm = 1;
  // dsp_set_option (performance only; results are identical for every value)
  int lane_rounds = 8;  // DSP_OPT_LANE_ROUNDS (8 measured best with 4 streams)
  int relabel_mode = 0; // DSP_OPT_RELABEL_MAP: 0 by N, 1 compact direct, 2 hash, 3 8-byte direct
  int loader_rows = 32;  // DSP_OPT_LOADER_ROWS: rows per TMA chunk, <= 32
  int persist_blocks = 0;  // blocks of the persistent kernel (0 = one per SM x occupancy)
  bool gather_reg = false;    // DSP_OPT_GATHER_REGLOADS: standalone gathers with register loads
  bool tma_unavailable = false;  // the TMA gather's shared memory could not be configured
  WsHeader *d_walk_hdr = nullptr;  // grid-barrier counter of k_walk_multi
  int walk_blocks_per_sm = 2;
  // virtual ranks sharing a GPU: each rank's persistent launch on its own
  // stream, one per exchange channel (concurrent group calls)
  cudaStream_t aux[DSP_MAX_CHANNELS] = {nullptr};
  cudaEvent_t aux_ev[DSP_MAX_CHANNELS][2] = {{nullptr}};
  cudaEvent_t flush_ev = nullptr;  // dsp_pipeline_flush: orders a pending gather after its call's stream
  int gather_blocks_per_sm = 1;
  // pipelined steps: per workspace, the gather owed by its previous
  // DSP_PIPELINED call (row count in the workspace's WsPersist::pend_n[parity])
  struct Pending {
    const char *ws = nullptr;
    const int32_t *ids = nullptr;  // its last block's src_ids
    float *out = nullptr;          // its feature output
    void *stream = nullptr;
    uint32_t calls = 0;            // pipelined calls made with this workspace
    bool active = false;
  } pend[8];
  Pending *pending_of(const char *ws) {
    for (auto &p : pend)
      if (p.ws == ws) return &p;
    for (auto &p : pend)
      if (!p.ws || !p.active) {
        p = Pending{};
        p.ws = ws;
        return &p;
      }
    return nullptr;
  }
};

namespace {

dsp_status fail(dsp_ctx *c, dsp_status s, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  if (c)
    c->err = buf;
  else
    g_create_error = buf;
  return s;
}

#define CUDA_TRY(ctx, call)                                                                  \
  do {                                                                                       \
    cudaError_t e_ = (call);                                                                 \
    if (e_ != cudaSuccess) {                                                                 \
      cudaGetLastError();                                                                    \
      return fail((ctx), e_ == cudaErrorMemoryAllocation ? DSP_ERR_OOM : DSP_ERR_CUDA,       \
                  "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));         \
    }                                                                                        \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

dsp_status check_fanouts(dsp_ctx *c, const int32_t *fanouts, int32_t L) {
  if (L < 1 || L > DSP_MAX_LAYERS || !fanouts)
    return fail(c, DSP_ERR_INVALID_ARG, "num_layers must be in [1, %d]", DSP_MAX_LAYERS);
  for (int l = 0; l < L; ++l)
    if (fanouts[l] < 1 || fanouts[l] > DSP_MAX_FANOUT)
      return fail(c, DSP_ERR_INVALID_ARG, "fanouts[%d] = %d not in [1, %d]", l, fanouts[l], DSP_MAX_FANOUT);
  return DSP_OK;
}

// The node-wise relabel map is a hash table sized to the batch (north star:
// "dedup and relabel through a GPU hash table") when a direct map over all N
// ids is too large to stay in L2; x = F + slot must fit the 25-bit field of a
// hash word.  Otherwise it is the compact direct map (4 B per node and parity,
// x < 2^24), or the 8-byte epoch-word direct map beyond that (and for the
// layer-wise scheme).
constexpr int64_t DIRECT_MAP_MAX_N = 3 * 1000 * 1000;
constexpr int64_t HASH_MAX_X = 1ll << 25;
constexpr int64_t DIRECT32_MAX_X = 1ll << 24;

// persist | hdr | first[2][N] (| first32[N] for direct-map sizes) at fixed
// offsets for every plan, so that one workspace can serve calls of any size
// and either scheme (the relabel maps' epoch words stay valid across them).
// Node-wise calls use ONE relabel map for all layers: layer l + 1 marks with
// a newer epoch tag, which beats every word of layer l, and no phase reads
// layer l's map once layer l + 1 starts marking (the duplicates of layer l are
// resolved through its edge slots, not the map), so half the L2 footprint of a
// map per layer parity.
size_t plan_common(Plan &p, int64_t N) {
  size_t o = align_up(sizeof(WsPersist), 256);
  p.off_hdr = o;
  o = align_up(o + sizeof(WsHeader), 256);
  for (int b = 0; b < 2; ++b) {
    p.off_first[b] = o;
    o = align_up(o + sizeof(unsigned long long) * std::max<int64_t>(1, N), 256);
  }
  p.off_first32 = 0;
  if (N <= DIRECT_MAP_MAX_N) {
    p.off_first32 = o;
    o = align_up(o + sizeof(uint32_t) * std::max<int64_t>(1, N), 256);
  }
  return o;
}

Plan make_plan(int64_t N, int64_t num_seeds, const int32_t *fanouts, int L, int relabel_mode = 0) {
  Plan p{};
  p.L = L;
  p.F[0] = num_seeds;
  p.max_F = std::max<int64_t>(1, num_seeds);
  p.max_slots = 1;
  for (int l = 0; l < L; ++l) {
    p.E[l] = p.F[l] * fanouts[l];
    p.S[l] = std::max<int64_t>(p.F[l], std::min<int64_t>(N, p.F[l] + p.E[l]));
    p.F[l + 1] = p.S[l];
    p.max_F = std::max(p.max_F, p.F[l]);
    p.max_slots = std::max(p.max_slots, p.E[l]);
  }
  size_t o = plan_common(p, N);
  // relabel_mode: 0 = by N, 1 = direct, 2 = hashed (DSP_RELABEL)
  int64_t max_keys = 0;
  for (int l = 0; l < L; ++l) max_keys = std::max(max_keys, p.F[l] + p.E[l]);
  const bool hashed = max_keys < HASH_MAX_X && (relabel_mode == 2 || (relabel_mode == 0 && N > DIRECT_MAP_MAX_N));
  p.direct32 = !hashed && relabel_mode != 3 && p.off_first32 != 0 && max_keys < DIRECT32_MAX_X;
  p.hash_cap = 0;
  if (hashed) {
    p.hash_cap = 1024;
    while (p.hash_cap < max_keys + max_keys / 2) p.hash_cap <<= 1;  // load factor <= 2/3
    p.off_hash = o;
    o = align_up(o + sizeof(unsigned long long) * (size_t)p.hash_cap, 256);
  }
  p.off_agg = o;
  o = align_up(o + sizeof(unsigned long long) * 2 * MAX_PERSIST_BLOCKS, 256);
  for (int b = 0; b < 2; ++b) {
    p.off_cnt[b] = o;
    o = align_up(o + sizeof(int32_t) * p.max_F, 256);
  }
  p.off_perm = o;
  o = align_up(o + sizeof(int32_t) * p.max_F, 256);
  for (int b = 0; b < 2; ++b) {
    p.off_rows[b] = o;
    o = align_up(o + sizeof(int32_t) * p.max_slots, 256);
  }
  p.bytes = o;
  return p;
}

// Layer-wise (R28): E_l <= n_l, max_src[l] = min(N, F_l + n_l).
LwLayout make_lw_layout(int64_t cap, int32_t ncap);

// own_xch (world 1): the inbox / return slots live in the workspace, so calls
// on different workspaces can run concurrently (no flags: k_lw_persistent)
Plan make_plan_lw(int64_t N, int64_t num_seeds, const int32_t *sizes, int L, bool own_xch) {
  Plan p{};
  p.L = L;
  p.F[0] = num_seeds;
  p.max_F = std::max<int64_t>(1, num_seeds);
  p.ncap = 1;
  for (int l = 0; l < L; ++l) {
    p.E[l] = sizes[l];
    p.S[l] = std::max<int64_t>(p.F[l], std::min<int64_t>(N, p.F[l] + p.E[l]));
    p.F[l + 1] = p.S[l];
    p.max_F = std::max(p.max_F, p.F[l]);
    p.ncap = std::max<int64_t>(p.ncap, sizes[l]);
  }
  p.big_cap = 8 * (p.ncap / 32) + 8;
  size_t o = plan_common(p, N);
  auto take = [&](size_t &off, size_t bytes) {
    off = o;
    o = align_up(o + bytes, 256);
  };
  take(p.off_P, sizeof(unsigned long long) * (size_t)(p.max_F + 1));
  take(p.off_c, sizeof(int32_t) * (size_t)p.max_F);
  take(p.off_off, sizeof(int32_t) * (size_t)(p.max_F + 1));
  take(p.off_slot_node, sizeof(int32_t) * (size_t)p.ncap);
  take(p.off_excl, sizeof(int32_t) * (size_t)(p.ncap + 1));
  take(p.off_newid, sizeof(int32_t) * (size_t)p.ncap);
  take(p.off_big, sizeof(int2) * (size_t)p.big_cap);
  p.off_lxch = 0;
  if (own_xch) take(p.off_lxch, make_lw_layout(std::max<int64_t>(1, p.max_F), (int32_t)p.ncap).bytes);
  p.bytes = o;
  return p;
}

LwLayout make_lw_layout(int64_t cap, int32_t ncap) {
  LwLayout x{};
  x.cap = cap;
  x.ncap = ncap;
  size_t o = 0;
  auto take = [&](size_t &off, size_t bytes) {
    off = o;
    o = align_up(o + bytes, 256);
  };
  take(x.off_inbox_flag, sizeof(unsigned long long) * 16);
  take(x.off_ret_flag, sizeof(unsigned long long) * 16);
  take(x.off_inbox_hdr, sizeof(uint4) * 16);
  take(x.off_inbox, sizeof(int4) * 16 * (size_t)cap);
  take(x.off_ret_cnt, sizeof(int32_t) * 2 * (size_t)cap);
  take(x.off_ret_rows, sizeof(int32_t) * 2 * (size_t)ncap);
  x.bytes = o;
  return x;
}

WalkLayout make_walk_layout(int world, int64_t max_walks, int32_t max_len) {
  WalkLayout x{};
  x.max_walks = max_walks;
  x.max_len = max_len;
  x.cap = std::max<int64_t>(1, (int64_t)world * max_walks);
  size_t o = 0;
  auto take = [&](size_t &off, size_t bytes) {
    off = o;
    o = align_up(o + bytes, 256);
  };
  take(x.off_flag, sizeof(unsigned long long) * 16);
  take(x.off_done, sizeof(unsigned long long) * 8);
  take(x.off_hdr, sizeof(uint4) * 16);
  take(x.off_inbox, sizeof(int2) * 16 * (size_t)x.cap);
  take(x.off_trace, sizeof(int32_t) * (size_t)std::max<int64_t>(1, max_walks) * (size_t)(max_len + 1));
  take(x.off_list, sizeof(int2) * 2 * (size_t)x.cap);
  take(x.off_ctr, sizeof(uint32_t) * 16);
  x.bytes = o;
  return x;
}

XchLayout make_xch_layout(int64_t cap, int kmax) {
  XchLayout x{};
  x.cap = cap;
  x.kmax = kmax;
  size_t o = 0;
  x.off_inbox_flag = o;
  o += sizeof(unsigned long long) * 16;
  x.off_ret_flag = o;
  o += sizeof(unsigned long long) * 16;
  x.off_inbox_hdr = o;
  o += sizeof(uint4) * 16;
  o = align_up(o, 256);
  x.off_inbox = o;
  o = align_up(o + sizeof(int32_t) * 16 * (size_t)cap, 256);
  x.off_ret_cnt = o;
  o = align_up(o + sizeof(int32_t) * 16 * (size_t)cap, 256);
  x.off_ret_rows = o;
  o = align_up(o + sizeof(int32_t) * 16 * (size_t)cap * kmax, 256);
  x.bytes = o;
  return x;
}

Bounds make_bounds(const dsp_ctx *c) {
  Bounds b{};
  for (int r = 0; r <= DSP_MAX_WORLD; ++r) b.b[r] = r <= c->world ? c->bounds[r] : c->N;
  b.world = c->world;
  return b;
}

int grid_for(const dsp_ctx *c, int blocks_per_sm) { return c->num_sms * blocks_per_sm; }

GatherArgs make_gather(const dsp_ctx *c, const int32_t *ids, int64_t n, const int32_t *n_dev, float *out) {
  GatherArgs a{};
  a.ids = ids;
  a.n = n;
  a.n_dev = n_dev;
  a.dim4 = c->dim / 4;
  a.head4 = head_bytes_of(c->split_rows, c->dim) / 16;
  a.out = reinterpret_cast<float4 *>(out);
  for (int r = 0; r < DSP_MAX_WORLD; ++r) {
    a.base[r] = r < c->world ? reinterpret_cast<const float4 *>(c->peer_feat[r]) : nullptr;
    a.tail[r] = r < c->world ? reinterpret_cast<const float4 *>(c->peer_feat_tail[r]) : nullptr;
    a.cold_tail[r] = r < c->world ? reinterpret_cast<const float4 *>(c->peer_cold_tail[r]) : nullptr;
    a.fpos[r] = r < c->world ? c->peer_fpos[r] : nullptr;
    a.cold[r] = r < c->world ? reinterpret_cast<const float4 *>(c->peer_cold[r]) : nullptr;
  }
  // 2: loader warps bulk-copy cold rows from host memory too; 1: register loads
  a.tiered = c->tiered ? (c->cold_regloads ? 1 : 2) : 0;
  a.bd = make_bounds(c);
  a.err = c->d_err;
  return a;
}

// ---------------------------------------------------------------- driver
// One dsp_sample call for one ctx, split into stages so that
// dsp_sample_group can interleave several ctxs stage by stage.
struct Call {
  dsp_ctx *c;
  const int32_t *seeds;
  int32_t num_seeds;
  const int32_t *fanouts;
  int32_t L;
  uint64_t rng_seed;
  dsp_block *blocks;
  char *ws;
  cudaStream_t stream;
  Plan plan;
  WsHeader *hdr;
  unsigned long long seq0;
  float *feat_out;     // fused gather (or nullptr)
  int64_t *sizes_out;  // async sizes destination (or nullptr)
  bool async;
  bool pipelined;      // gather this call's rows in the next pipelined call / flush
  bool biased;         // DSP_BIASED
  bool layerwise;      // DSP_LAYERWISE: fanouts are layer sizes
  int channel;         // node-wise world > 1: exchange channel of this call
  uint32_t call_tag;   // low byte of the ctx's collective call count (checked in the exchange header)
};

LayerBufs bufs_of(const Call &k, int parity) {
  LayerBufs b{};
  b.cnt = reinterpret_cast<int32_t *>(k.ws + k.plan.off_cnt[parity]);
  b.rows = reinterpret_cast<int32_t *>(k.ws + k.plan.off_rows[parity]);
  b.first = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_first[0]);  // one map for all layers
  b.mask = 0;
  b.first32 = nullptr;
  b.n32 = 0;
  if (k.plan.direct32) {
    b.first32 = reinterpret_cast<uint32_t *>(k.ws + k.plan.off_first32);
    b.n32 = (uint32_t)k.c->N;
  }
  if (k.plan.hash_cap > 0) {
    b.first = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_hash);
    b.mask = (uint32_t)(k.plan.hash_cap - 1);
  }
  return b;
}

WsPersist *persist_of(const Call &k) { return reinterpret_cast<WsPersist *>(k.ws); }

dsp_status check_sizes(dsp_ctx *c, const int32_t *sizes, int32_t L) {
  if (L < 1 || L > DSP_MAX_LAYERS || !sizes)
    return fail(c, DSP_ERR_INVALID_ARG, "num_layers must be in [1, %d]", DSP_MAX_LAYERS);
  for (int l = 0; l < L; ++l)
    if (sizes[l] < 1 || sizes[l] > DSP_MAX_LAYER_SIZE)
      return fail(c, DSP_ERR_INVALID_ARG, "layer size %d = %d not in [1, %d]", l, sizes[l], DSP_MAX_LAYER_SIZE);
  return DSP_OK;
}

dsp_status check_blocks(dsp_ctx *c, const Plan &p, const dsp_block *blocks, int L) {
  for (int l = 0; l < L; ++l) {
    if ((uint64_t)p.F[l] + (uint64_t)p.E[l] >= (1ull << 31))
      return fail(c, DSP_ERR_CAPACITY, "layer %d: frontier + edges exceeds 2^31", l);
    if (!blocks[l].indptr || !blocks[l].indices || !blocks[l].src_ids)
      return fail(c, DSP_ERR_INVALID_ARG, "blocks[%d] has a NULL array", l);
    if (blocks[l].cap_indptr < p.F[l] + 1 || blocks[l].cap_edges < p.E[l] || blocks[l].cap_src < p.S[l])
      return fail(c, DSP_ERR_CAPACITY, "blocks[%d] capacities (%lld, %lld, %lld) < bounds (%lld, %lld, %lld)", l,
                  (long long)blocks[l].cap_indptr, (long long)blocks[l].cap_edges, (long long)blocks[l].cap_src,
                  (long long)(p.F[l] + 1), (long long)p.E[l], (long long)p.S[l]);
  }
  return DSP_OK;
}

// DSP_LAYERWISE: needs dsp_reserve_layerwise with the same sizes.
dsp_status prepare_call_lw(Call &k, dsp_ctx *c, const int32_t *seeds, int32_t num_seeds, const int32_t *sizes,
                           int32_t L, uint64_t rng_seed, dsp_block *blocks, void *workspace, size_t ws_bytes,
                           void *stream) {
  if (k.biased) return fail(c, DSP_ERR_INVALID_ARG, "DSP_LAYERWISE with DSP_BIASED is not supported");
  if (c->broken) return fail(c, DSP_ERR_STATE, "ctx unusable after an earlier exchange failure");
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition not called");
  if (!c->lw_reserved) return fail(c, DSP_ERR_STATE, "DSP_LAYERWISE needs dsp_reserve_layerwise first");
  if (c->world > 1 && !c->imported) return fail(c, DSP_ERR_STATE, "world_size > 1 needs dsp_import_handles first");
  dsp_status st = check_sizes(c, sizes, L);
  if (st != DSP_OK) return st;
  if (num_seeds < 0 || (num_seeds > 0 && !seeds)) return fail(c, DSP_ERR_INVALID_ARG, "bad seeds / num_seeds");
  if (!blocks || !workspace) return fail(c, DSP_ERR_INVALID_ARG, "blocks / workspace is NULL");
  if (num_seeds > c->lw_max_seeds)
    return fail(c, DSP_ERR_CAPACITY, "num_seeds %d > reserved max_seeds %d", num_seeds, c->lw_max_seeds);
  if (L != c->lw_L) return fail(c, DSP_ERR_STATE, "num_layers %d != reserved %d", L, c->lw_L);
  for (int l = 0; l < L; ++l)
    if (sizes[l] != c->lw_sizes[l])
      return fail(c, DSP_ERR_STATE, "layer size %d = %d != reserved %d", l, sizes[l], c->lw_sizes[l]);
  k.plan = make_plan_lw(c->N, c->lw_max_seeds, sizes, L, c->world == 1);
  if (ws_bytes < k.plan.bytes)
    return fail(c, DSP_ERR_CAPACITY, "workspace %zu B < required %zu B", ws_bytes, k.plan.bytes);
  if (((uintptr_t)workspace & 255u) != 0) return fail(c, DSP_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
  if ((st = check_blocks(c, k.plan, blocks, L)) != DSP_OK) return st;
  k.seeds = seeds;
  k.num_seeds = num_seeds;
  k.fanouts = sizes;
  k.L = L;
  k.rng_seed = rng_seed;
  k.blocks = blocks;
  k.ws = static_cast<char *>(workspace);
  k.stream = static_cast<cudaStream_t>(stream);
  k.hdr = reinterpret_cast<WsHeader *>(k.ws + k.plan.off_hdr);
  k.seq0 = c->seq;
  return DSP_OK;
}

dsp_status prepare_call(Call &k, dsp_ctx *c, const int32_t *seeds, int32_t num_seeds,
                        const int32_t *fanouts, int32_t L, uint64_t rng_seed, dsp_block *blocks,
                        void *workspace, size_t ws_bytes, uint32_t flags, void *stream) {
  k = Call{};
  k.c = c;
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if ((flags & ~(DSP_ASYNC | DSP_PIPELINED | DSP_BIASED | DSP_LAYERWISE)) != 0)
    return fail(c, DSP_ERR_INVALID_ARG, "unknown flags 0x%x", flags);
  k.biased = (flags & DSP_BIASED) != 0;
  k.layerwise = (flags & DSP_LAYERWISE) != 0;
  if (k.layerwise) return prepare_call_lw(k, c, seeds, num_seeds, fanouts, L, rng_seed, blocks, workspace,
                                          ws_bytes, stream);
  if (k.biased && !c->d_weights) return fail(c, DSP_ERR_STATE, "DSP_BIASED needs dsp_load_weights first");
  if (c->broken) return fail(c, DSP_ERR_STATE, "ctx unusable after an earlier exchange failure");
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition not called");
  if (c->world > 1 && (!c->reserved || !c->imported))
    return fail(c, DSP_ERR_STATE, "world_size > 1 needs dsp_reserve + dsp_import_handles first");
  dsp_status st = check_fanouts(c, fanouts, L);
  if (st != DSP_OK) return st;
  if (num_seeds < 0 || (num_seeds > 0 && !seeds))
    return fail(c, DSP_ERR_INVALID_ARG, "bad seeds / num_seeds");
  if (!blocks || !workspace) return fail(c, DSP_ERR_INVALID_ARG, "blocks / workspace is NULL");
  if (c->reserved) {
    if (num_seeds > c->max_seeds)
      return fail(c, DSP_ERR_CAPACITY, "num_seeds %d > reserved max_seeds %d", num_seeds, c->max_seeds);
    if (L != c->L) return fail(c, DSP_ERR_STATE, "num_layers %d != reserved %d", L, c->L);
    for (int l = 0; l < L; ++l)
      if (fanouts[l] != c->fanouts[l])
        return fail(c, DSP_ERR_STATE, "fanouts[%d] = %d != reserved %d", l, fanouts[l], c->fanouts[l]);
  }
  // workspace and exchange capacities are planned for the reserved maximum so
  // that every rank derives the same sizes
  const int64_t plan_seeds = c->reserved ? c->max_seeds : num_seeds;
  k.plan = make_plan(c->N, plan_seeds, fanouts, L, c->relabel_mode);
  if (ws_bytes < k.plan.bytes)
    return fail(c, DSP_ERR_CAPACITY, "workspace %zu B < required %zu B", ws_bytes, k.plan.bytes);
  if (((uintptr_t)workspace & 255u) != 0) return fail(c, DSP_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
  for (int l = 0; l < L; ++l) {
    if ((uint64_t)k.plan.F[l] + (uint64_t)k.plan.E[l] >= (1ull << 31))
      return fail(c, DSP_ERR_CAPACITY, "layer %d: frontier * (1 + fanout) exceeds 2^31", l);
    if (!blocks[l].indptr || !blocks[l].indices || !blocks[l].src_ids)
      return fail(c, DSP_ERR_INVALID_ARG, "blocks[%d] has a NULL array", l);
    if (blocks[l].cap_indptr < k.plan.F[l] + 1 || blocks[l].cap_edges < k.plan.E[l] ||
        blocks[l].cap_src < k.plan.S[l])
      return fail(c, DSP_ERR_CAPACITY,
                  "blocks[%d] capacities (%lld, %lld, %lld) < bounds (%lld, %lld, %lld)", l,
                  (long long)blocks[l].cap_indptr, (long long)blocks[l].cap_edges,
                  (long long)blocks[l].cap_src, (long long)(k.plan.F[l] + 1),
                  (long long)k.plan.E[l], (long long)k.plan.S[l]);
  }
  k.seeds = seeds;
  k.num_seeds = num_seeds;
  k.fanouts = fanouts;
  k.L = L;
  k.rng_seed = rng_seed;
  k.blocks = blocks;
  k.ws = static_cast<char *>(workspace);
  k.stream = static_cast<cudaStream_t>(stream);
  k.hdr = reinterpret_cast<WsHeader *>(k.ws + k.plan.off_hdr);
  k.channel = (int)(c->ncalls % (unsigned long long)c->channels);
  k.call_tag = (uint32_t)(c->ncalls & 0xffu);
  k.seq0 = c->world > 1 ? c->chan_seq[k.channel] : 0;
  return DSP_OK;
}

dsp_status stage_begin(Call &k) {
  DeviceGuard g(k.c->device);
  CUDA_TRY(k.c, cudaMemsetAsync(k.hdr, 0, sizeof(WsHeader), k.stream));
  return DSP_OK;
}

const int32_t *frontier_of(const Call &k, int l) { return l == 0 ? k.seeds : k.blocks[l - 1].src_ids; }

uint2 key_of(uint64_t rng_seed) { return make_uint2((uint32_t)rng_seed, (uint32_t)(rng_seed >> 32)); }

// world == 1: the whole call (+ optional gather) in one cooperative kernel

dsp_status stage_persistent(Call &k) {
  dsp_ctx *c = k.c;
  DeviceGuard g(c->device);
  PersistArgs a{};
  a.seeds = k.seeds;
  a.B = k.num_seeds;
  a.L = k.L;
  for (int l = 0; l < k.L; ++l) {
    a.k[l] = k.fanouts[l];
    a.out.indptr[l] = k.blocks[l].indptr;
    a.out.indices[l] = k.blocks[l].indices;
    a.out.src_ids[l] = k.blocks[l].src_ids;
  }
  a.agg = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_agg);
  a.persist = persist_of(k);
  a.key = key_of(k.rng_seed);
  a.indptr = c->d_indptr;
  a.indices = c->d_indices;
  a.weights = c->d_weights;
  a.biased = k.biased ? 1 : 0;
  a.lo = c->lo;
  a.n_local = c->n_local;
  a.buf[0] = bufs_of(k, 0);
  a.buf[1] = bufs_of(k, 1);
  a.hdr = k.hdr;
  a.err = c->d_err;
  a.lane_rounds = c->lane_rounds;
  a.gather = k.feat_out != nullptr && !k.pipelined;
  if (a.gather) a.g = make_gather(c, k.blocks[k.L - 1].src_ids, 0, nullptr, k.feat_out);
  const dim3 grid(c->persist_blocks > 0 ? c->persist_blocks : c->num_sms * c->persist_blocks_per_sm), block(PNT);
  void *args[] = {&a};
  if (!k.pipelined) {
    CUDA_TRY(c, cudaLaunchCooperativeKernel(k.biased ? (const void *)k_csp_persistent<BIASED_BLK, false, true, BIASED_BLK>
                                                     : (const void *)k_csp_persistent<PNT, false, false>,
                                            grid, k.biased ? dim3(BIASED_BLK) : block, args, 0, k.stream));
    return DSP_OK;
  }
  dsp_ctx::Pending *pd = c->pending_of(k.ws);
  if (!pd) return fail(c, DSP_ERR_STATE, "more than 8 workspaces with pending pipelined gathers");
  WsPersist *ps = persist_of(k);
  a.prev = pd->active ? 1 : 0;
  if (a.prev) a.gp = make_gather(c, pd->ids, 0, &ps->pend_n[(pd->calls + 1) & 1], pd->out);
  a.pend_n = &ps->pend_n[pd->calls & 1];
  const int row_bytes = c->dim * 4;
  // ring slots sized to the chunk (rows_per_chunk rows of <= 12.8 KB in all): the ring's
  // shared memory is taken from the L1 the sampling phases use
  a.rows_per_chunk = std::max(1, std::min(c->loader_rows, 12800 / std::max(1, row_bytes)));
  a.slot_bytes = (int)align_up((size_t)a.rows_per_chunk * row_bytes, 128);
  const size_t smem = (size_t)(k.biased ? BIASED_LOADER_WARPS : LOADER_WARPS) * LOADER_SLOTS * a.slot_bytes;
  CUDA_TRY(c, cudaLaunchCooperativeKernel(k.biased ? (const void *)k_csp_persistent<BIASED_PIPE_TEAM, true, true, BIASED_BLK>
                                                   : (const void *)k_csp_persistent<PIPE_TEAM, true, false>,
                                          grid, k.biased ? dim3(BIASED_BLK) : block, args, smem, k.stream));
  pd->ids = k.blocks[k.L - 1].src_ids;
  pd->out = k.feat_out;
  pd->stream = k.stream;
  pd->active = true;
  pd->calls += 1;
  return DSP_OK;
}

XchPeers peers_of(const dsp_ctx *c, int channel);

// Virtual ranks sharing a GPU: fork the caller's stream onto the ctx's own
// stream of channel ch (created on first use), so that every rank of a group
// call is launched before any is joined (all of them resident at once).
dsp_status fork_aux(dsp_ctx *c, int ch, cudaStream_t from, cudaStream_t *out) {
  if (!c->aux[ch]) {
    CUDA_TRY(c, cudaStreamCreateWithFlags(&c->aux[ch], cudaStreamNonBlocking));
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->aux_ev[ch][0], cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventCreateWithFlags(&c->aux_ev[ch][1], cudaEventDisableTiming));
  }
  CUDA_TRY(c, cudaEventRecord(c->aux_ev[ch][0], from));
  CUDA_TRY(c, cudaStreamWaitEvent(c->aux[ch], c->aux_ev[ch][0], 0));
  *out = c->aux[ch];
  return DSP_OK;
}
dsp_status join_aux(dsp_ctx *c, int ch, cudaStream_t to) {
  CUDA_TRY(c, cudaEventRecord(c->aux_ev[ch][1], c->aux[ch]));
  CUDA_TRY(c, cudaStreamWaitEvent(to, c->aux_ev[ch][1], 0));
  return DSP_OK;
}

// world > 1, node-wise: the whole call in one cooperative kernel per rank
// (dsp_multi.cuh).  `share` = ranks of this call group on the same GPU
// (virtual ranks): each launch gets 1/share of the SMs, on the ctx's own
// stream forked from / joined to the caller's, so all of them are resident.
dsp_status stage_persistent_multi(Call &k, int share) {
  dsp_ctx *c = k.c;
  DeviceGuard g(c->device);
  MultiArgs m{};
  PersistArgs &a = m.p;
  a.seeds = k.seeds;
  a.B = k.num_seeds;
  a.L = k.L;
  for (int l = 0; l < k.L; ++l) {
    a.k[l] = k.fanouts[l];
    a.out.indptr[l] = k.blocks[l].indptr;
    a.out.indices[l] = k.blocks[l].indices;
    a.out.src_ids[l] = k.blocks[l].src_ids;
  }
  a.agg = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_agg);
  a.persist = persist_of(k);
  a.key = key_of(k.rng_seed);
  a.indptr = c->d_indptr;
  a.indices = c->d_indices;
  a.weights = c->d_weights;
  a.biased = k.biased ? 1 : 0;
  a.lo = c->lo;
  a.n_local = c->n_local;
  a.buf[0] = bufs_of(k, 0);
  a.buf[1] = bufs_of(k, 1);
  a.hdr = k.hdr;
  a.err = c->d_err;
  a.lane_rounds = c->lane_rounds;
  a.gather = k.feat_out != nullptr && !k.pipelined;
  if (a.gather) a.g = make_gather(c, k.blocks[k.L - 1].src_ids, 0, nullptr, k.feat_out);
  m.rank = c->rank;
  m.seq0 = k.seq0;
  m.bd = make_bounds(c);
  m.X = c->xl;
  m.peers = peers_of(c, k.channel);
  m.call_tag = k.call_tag;
  m.perm = reinterpret_cast<int32_t *>(k.ws + k.plan.off_perm);
  m.abort_word = &k.hdr->abort_wait;
  int blocks = c->persist_blocks > 0 ? c->persist_blocks : c->num_sms * c->persist_blocks_per_sm;
  if (share > 1) blocks = std::max(1, std::min(blocks, c->num_sms * c->persist_blocks_per_sm / share));
  const dim3 grid(blocks), block(PNT);
  cudaStream_t st = k.stream;
  if (share > 1) {  // fork onto the ctx's own stream
    dsp_status fs = fork_aux(c, k.channel, k.stream, &st);
    if (fs != DSP_OK) return fs;
  }
  void *args[] = {&m};
  cudaEvent_t &cev = c->chan_ev[k.channel];
  if (c->channels > 1 && c->chan_used[k.channel])  // the channel's previous call (possibly on another stream)
    CUDA_TRY(c, cudaStreamWaitEvent(st, cev, 0));
  if (!k.pipelined) {
    CUDA_TRY(c, cudaLaunchCooperativeKernel(k.biased ? (const void *)k_csp_multi<PNT, false, true>
                                                     : (const void *)k_csp_multi<PNT, false, false>,
                                            grid, block, args, 0, st));
  } else {
    dsp_ctx::Pending *pd = c->pending_of(k.ws);
    if (!pd) return fail(c, DSP_ERR_STATE, "more than 8 workspaces with pending pipelined gathers");
    WsPersist *ps = persist_of(k);
    a.prev = pd->active ? 1 : 0;
    if (a.prev) a.gp = make_gather(c, pd->ids, 0, &ps->pend_n[(pd->calls + 1) & 1], pd->out);
    a.pend_n = &ps->pend_n[pd->calls & 1];
    const int row_bytes = c->dim * 4;
    a.slot_bytes = (int)align_up((size_t)std::max(12800, row_bytes), 128);
    a.rows_per_chunk = std::max(1, std::min(c->loader_rows, a.slot_bytes / std::max(1, row_bytes)));
    const size_t smem = (size_t)LOADER_WARPS * LOADER_SLOTS * a.slot_bytes;
    CUDA_TRY(c, cudaLaunchCooperativeKernel(k.biased ? (const void *)k_csp_multi<PIPE_TEAM, true, true>
                                                     : (const void *)k_csp_multi<PIPE_TEAM, true, false>,
                                            grid, block, args, smem, st));
    pd->ids = k.blocks[k.L - 1].src_ids;
    pd->out = k.feat_out;
    pd->stream = k.stream;
    pd->active = true;
    pd->calls += 1;
  }
  if (c->channels > 1) {
    CUDA_TRY(c, cudaEventRecord(cev, st));
    c->chan_used[k.channel] = true;
  }
  return DSP_OK;
}

// the caller's stream waits for the rank's own stream (after ALL ranks of the
// group were launched: joining earlier would serialise the virtual ranks)
dsp_status join_persistent_multi(Call &k, int share) {
  dsp_ctx *c = k.c;
  if (share <= 1) return DSP_OK;
  DeviceGuard g(c->device);
  return join_aux(c, k.layerwise ? 0 : k.channel, k.stream);
}

// A standalone gather: TMA loader warps (k_gather_tma) by default, 16-byte
// register loads (k_gather) with DSP_GATHER_REG=1 or for register-loaded cold rows.
// n_host: the row count, or ignored when g.n_dev gives it on the device.
dsp_status launch_gather(dsp_ctx *c, const GatherArgs &g, int64_t n_host, cudaStream_t st) {
  if (c->gather_reg || (c->tiered && c->cold_regloads)) {
    int grid = grid_for(c, std::min(6, c->gather_blocks_per_sm));
    if (!g.n_dev) {  // resident blocks only (a partial extra wave costs more than it hides)
      const int64_t want = (n_host * g.dim4 + (int64_t)NT * GATHER_UNROLL - 1) / ((int64_t)NT * GATHER_UNROLL);
      grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, grid));
    }
    k_gather<<<grid, NT, 0, st>>>(g);
    CUDA_TRY(c, cudaGetLastError());
    return DSP_OK;
  }
  PersistArgs a{};
  a.gp = g;
  const int row_bytes = c->dim * 4;
  a.slot_bytes = (int)align_up((size_t)std::max(12800, row_bytes), 128);
  a.rows_per_chunk = std::max(1, std::min(c->loader_rows, a.slot_bytes / std::max(1, row_bytes)));
  int blocks = c->num_sms * (GTMA_WARPS <= 4 ? 2 : 1);
  if (!g.n_dev) {
    const int64_t chunks = (n_host + a.rows_per_chunk - 1) / a.rows_per_chunk;
    blocks = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, (chunks + 2 * GTMA_WARPS - 1) / (2 * GTMA_WARPS)));
  }
  const size_t smem = (size_t)GTMA_WARPS * GTMA_SLOTS * a.slot_bytes;
  if (c->world > 1)
    k_gather_tma<true><<<blocks, 32 * GTMA_WARPS, smem, st>>>(a, n_host);
  else
    k_gather_tma<false><<<blocks, 32 * GTMA_WARPS, smem, st>>>(a, n_host);
  CUDA_TRY(c, cudaGetLastError());
  return DSP_OK;
}

// Gather owed by a workspace's last pipelined call (the device row count),
// enqueued on `st`.  When the pipelined call ran on another stream, `st`
// first waits for everything issued there so far (event), so the gather reads
// that call's finished src_ids and row count on any stream.
dsp_status flush_one(dsp_ctx *c, dsp_ctx::Pending &pd, cudaStream_t st) {
  if (!pd.active) return DSP_OK;
  DeviceGuard g(c->device);
  if (static_cast<cudaStream_t>(pd.stream) != st) {
    if (!c->flush_ev) CUDA_TRY(c, cudaEventCreateWithFlags(&c->flush_ev, cudaEventDisableTiming));
    CUDA_TRY(c, cudaEventRecord(c->flush_ev, static_cast<cudaStream_t>(pd.stream)));
    CUDA_TRY(c, cudaStreamWaitEvent(st, c->flush_ev, 0));
  }
  const WsPersist *ps = reinterpret_cast<const WsPersist *>(pd.ws);
  GatherArgs a = make_gather(c, pd.ids, 0, &ps->pend_n[(pd.calls + 1) & 1], pd.out);
  dsp_status s = launch_gather(c, a, 0, st);
  if (s != DSP_OK) return s;
  pd.active = false;
  return DSP_OK;
}

dsp_status stage_flush(dsp_ctx *c, const char *ws, cudaStream_t st) {
  for (auto &p : c->pend)
    if (p.active && p.ws == ws) return flush_one(c, p, st);
  return DSP_OK;
}

XchPeers peers_of(const dsp_ctx *c, int channel) {
  XchPeers p{};
  for (int r = 0; r < DSP_MAX_WORLD; ++r)
    p.base[r] = r < c->world && c->peer_xch[r] ? c->peer_xch[r] + (size_t)channel * c->chan_stride : nullptr;
  return p;
}

// ------------------------------------------------ layer-wise stages
LwArgs lw_args(Call &k, int l) {
  dsp_ctx *c = k.c;
  LwArgs a{};
  a.seeds = k.seeds;
  a.frontier = frontier_of(k, l);
  a.F0 = k.num_seeds;
  a.layer = l;
  a.n = k.fanouts[l];
  a.rank = c->rank;
  a.seq = k.seq0 + 1 + l;
  a.parity = (int)(a.seq & 1);
  a.key = key_of(k.rng_seed);
  a.bd = make_bounds(c);
  for (int r = 0; r < DSP_MAX_WORLD; ++r) {
    a.peer_indptr[r] = r < c->world ? c->peer_indptr[r] : nullptr;
    a.peers.base[r] = r < c->world ? c->peer_lxch[r] : nullptr;
  }
  a.indptr = c->d_indptr;
  a.indices = c->d_indices;
  a.lo = c->lo;
  a.n_local = c->n_local;
  a.L = c->lxl;
  a.w.P = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_P);
  a.w.c = reinterpret_cast<int32_t *>(k.ws + k.plan.off_c);
  a.w.off = reinterpret_cast<int32_t *>(k.ws + k.plan.off_off);
  a.w.slot_node = reinterpret_cast<int32_t *>(k.ws + k.plan.off_slot_node);
  a.w.excl = reinterpret_cast<int32_t *>(k.ws + k.plan.off_excl);
  a.w.newid = reinterpret_cast<int32_t *>(k.ws + k.plan.off_newid);
  a.w.big = reinterpret_cast<int2 *>(k.ws + k.plan.off_big);
  a.w.big_cap = (int32_t)k.plan.big_cap;
  a.first = reinterpret_cast<unsigned long long *>(k.ws + k.plan.off_first[l & 1]);
  a.persist = persist_of(k);
  a.out.indptr[0] = k.blocks[l].indptr;
  a.out.indices[0] = k.blocks[l].indices;
  a.out.src_ids[0] = k.blocks[l].src_ids;
  a.hdr = k.hdr;
  a.err = c->d_err;
  a.sys = c->world > 1 ? 1 : 0;
  if (c->world == 1 && k.plan.off_lxch)  // world-1 call: its own exchange slots
    a.peers.base[0] = k.ws + k.plan.off_lxch;
  return a;
}

// layer-wise: every layer in one cooperative launch per rank (k_lw_persistent
// at world 1, k_lw_multi at world > 1; `share` = ranks of the call group on
// this GPU, each launched on its own stream with 1/share of the SMs)
dsp_status stage_lw_persistent(Call &k, int share = 1) {
  dsp_ctx *c = k.c;
  DeviceGuard g(c->device);
  LwPersistArgs p{};
  for (int l = 0; l < k.L; ++l) p.l[l] = lw_args(k, l);
  p.L = k.L;
  p.kp_max = (int)next_pow2(k.plan.ncap);
  p.hdr = k.hdr;
  p.persist = persist_of(k);
  p.gather = k.feat_out != nullptr && !k.pipelined;
  if (p.gather) p.g = make_gather(c, k.blocks[k.L - 1].src_ids, 0, nullptr, k.feat_out);
  dsp_ctx::Pending *pd = nullptr;
  if (k.feat_out && k.pipelined) {  // the previous call's rows are gathered during this call's first allocation
    pd = c->pending_of(k.ws);
    if (!pd) return fail(c, DSP_ERR_STATE, "more than 8 workspaces with pending pipelined gathers");
    WsPersist *ps = persist_of(k);
    p.prev = pd->active ? 1 : 0;
    if (p.prev) p.gp = make_gather(c, pd->ids, 0, &ps->pend_n[(pd->calls + 1) & 1], pd->out);
    p.pend_n = &ps->pend_n[pd->calls & 1];
  }
  const size_t smem = std::max(LW_ALLOC_SMEM, sizeof(int32_t) * 3 * (size_t)p.kp_max);
  int blocks = std::min(c->persist_blocks > 0 ? c->persist_blocks : c->num_sms, 64);
  if (share > 1) blocks = std::max(1, std::min(blocks, c->num_sms / share));
  const dim3 grid(blocks), block(LWT);
  cudaStream_t st = k.stream;
  if (share > 1) {  // fork onto the ctx's own stream (joined by join_persistent_multi)
    dsp_status fs = fork_aux(c, 0, k.stream, &st);
    if (fs != DSP_OK) return fs;
  }
  void *args[] = {&p};
  CUDA_TRY(c, cudaLaunchCooperativeKernel(c->world > 1 ? (const void *)k_lw_multi : (const void *)k_lw_persistent,
                                          grid, block, args, smem, st));
  if (pd) {
    pd->ids = k.blocks[k.L - 1].src_ids;
    pd->out = k.feat_out;
    pd->stream = k.stream;
    pd->active = true;
    pd->calls += 1;
  }
  return DSP_OK;
}

// ------------------------------------------------------------- end of call
dsp_status stage_end_async(Call &k) {
  dsp_ctx *c = k.c;
  DeviceGuard g(c->device);
  if (k.async) {
    if (k.sizes_out)
      CUDA_TRY(c, cudaMemcpyAsync(k.sizes_out, k.hdr->sizes, sizeof(int64_t) * 3 * k.L, cudaMemcpyDefault,
                                  k.stream));
  } else {
    CUDA_TRY(c, cudaMemcpyAsync(c->h_hdr, k.hdr, sizeof(WsHeader), cudaMemcpyDeviceToHost, k.stream));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_err, c->d_err, sizeof(int), cudaMemcpyDeviceToHost, k.stream));
  }
  return DSP_OK;
}

dsp_status stage_finish(Call &k) {
  dsp_ctx *c = k.c;
  DeviceGuard g(c->device);
  if (k.layerwise) {
    c->seq = k.seq0 + k.L;
  } else if (c->world > 1) {
    c->chan_seq[k.channel] = k.seq0 + k.L;
    c->ncalls += 1;
  }
  if (k.async) return DSP_OK;
  CUDA_TRY(c, cudaStreamSynchronize(k.stream));
  const int e = *c->h_err;
  if (e != 0) {
    CUDA_TRY(c, cudaMemset(c->d_err, 0, sizeof(int)));
    if (e == E_STATE && c->world > 1) c->broken = true;
    return fail(c, (dsp_status)e, "device-detected error %d (%s)", e, dsp_status_str(e));
  }
  const WsHeader &h = *c->h_hdr;
  for (int l = 0; l < k.L; ++l) {
    k.blocks[l].num_dst = h.F[l];
    k.blocks[l].num_src = h.S[l];
    k.blocks[l].num_edges = h.E[l];
  }
  if (k.sizes_out)
    for (int l = 0; l < k.L; ++l) {
      k.sizes_out[3 * l + 0] = h.F[l];
      k.sizes_out[3 * l + 1] = h.S[l];
      k.sizes_out[3 * l + 2] = h.E[l];
    }
  return DSP_OK;
}

dsp_status run_calls(std::vector<Call> &calls) {
  dsp_status st;
#define EACH(STAGE)                                   \
  for (auto &k : calls)                               \
    if ((st = (STAGE)) != DSP_OK) return st;
  // a non-pipelined call first settles a pending pipelined gather of its workspace
  for (auto &k : calls)
    if (!k.pipelined && (st = stage_flush(k.c, k.ws, k.stream)) != DSP_OK) return st;
  EACH(stage_begin(k));
  if (calls[0].c->world == 1 && !calls[0].layerwise) {
    EACH(stage_persistent(k));
  } else {
    // one cooperative launch per rank: k_csp_multi (node-wise, world > 1) or
    // k_lw_persistent / k_lw_multi (layer-wise); ranks sharing a device each
    // run on their own stream with 1/share of its SMs
    std::vector<int> share(calls.size(), 0);
    for (size_t i = 0; i < calls.size(); ++i)
      for (auto &o : calls) share[i] += o.c->device == calls[i].c->device ? 1 : 0;
    for (size_t i = 0; i < calls.size(); ++i)
      if ((st = calls[i].layerwise ? stage_lw_persistent(calls[i], share[i])
                                   : stage_persistent_multi(calls[i], share[i])) != DSP_OK)
        return st;
    for (size_t i = 0; i < calls.size(); ++i)
      if ((st = join_persistent_multi(calls[i], share[i])) != DSP_OK) return st;
  }
  EACH(stage_end_async(k));
#undef EACH
  dsp_status first = DSP_OK;
  for (auto &k : calls) {
    st = stage_finish(k);
    if (st != DSP_OK && first == DSP_OK) first = st;
  }
  return first;
}

void release(dsp_ctx *c) {
  DeviceGuard g(c->device);
  for (int r = 0; r < DSP_MAX_WORLD; ++r)
    if (c->peer_cold_map[r]) {
      cudaHostUnregister(c->peer_cold_map[r]);
      munmap(c->peer_cold_map[r], (size_t)c->peer_cold_bytes[r]);
      c->peer_cold_map[r] = nullptr;
    }
  if (c->h_cold) {
    if (c->cold_shm[0]) {
      cudaHostUnregister(c->h_cold);
      munmap(c->h_cold, (size_t)c->cold_bytes);
      shm_unlink(c->cold_shm);
    } else {
      cudaFreeHost(c->h_cold);
    }
    c->h_cold = nullptr;
  }
  cudaFree(c->d_fpos);
  for (int i = 0; i < 6 * DSP_MAX_WORLD; ++i)
    if (c->ipc_opened[i]) {
      cudaIpcCloseMemHandle(c->ipc_opened[i]);
      c->ipc_opened[i] = nullptr;
    }
  cudaFree(c->d_indptr);
  cudaFree(c->d_indices);
  cudaFree(c->d_weights);
  cudaFree(c->d_feat);
  cudaFree(c->d_xch);
  cudaFree(c->d_walk_hdr);
  for (int ch = 0; ch < DSP_MAX_CHANNELS; ++ch)
    if (c->aux[ch]) {
      cudaStreamSynchronize(c->aux[ch]);
      cudaStreamDestroy(c->aux[ch]);
      cudaEventDestroy(c->aux_ev[ch][0]);
      cudaEventDestroy(c->aux_ev[ch][1]);
      c->aux[ch] = nullptr;
    }
  if (c->flush_ev) {
    cudaEventDestroy(c->flush_ev);
    c->flush_ev = nullptr;
  }
  for (auto &e : c->chan_ev)
    if (e) {
      cudaEventDestroy(e);
      e = nullptr;
    }
  cudaFree(c->d_lxch);
  cudaFree(c->d_wxch);
  cudaFree(c->d_err);
  if (c->h_hdr) cudaFreeHost(c->h_hdr);
  if (c->h_err) cudaFreeHost(c->h_err);
  cudaGetLastError();
}

// Random walks over a partitioned graph: one stage of one rank.
// stage 0 = init, 1 = shuffle of step l, 2 = step l at the owner, 3 = done, 4 = finish.
WalkArgs walk_args(dsp_ctx *c, const int32_t *starts, int64_t n, int32_t length, uint64_t rng_seed,
                   int32_t *traces, uint32_t flags) {
  WalkArgs a{};
  a.starts = starts;
  a.n = n;
  a.length = length;
  a.rank = c->rank;
  a.key = key_of(rng_seed);
  a.indptr = c->d_indptr;
  a.indices = c->d_indices;
  a.lo = c->lo;
  a.n_local = c->n_local;
  a.bd = make_bounds(c);
  a.L = c->wl;
  for (int r = 0; r < DSP_MAX_WORLD; ++r) a.peers.base[r] = r < c->world ? c->peer_wxch[r] : nullptr;
  a.traces = traces;
  a.err = c->d_err;
  a.independent = (flags & DSP_WALK_INDEPENDENT) ? 1 : 0;
  return a;
}

dsp_status check_walk_call(dsp_ctx *c, const int32_t *starts, int64_t n, int32_t length, int32_t *traces) {
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  if (length < 1 || length > 1024) return fail(c, DSP_ERR_INVALID_ARG, "length %d not in [1, 1024]", length);
  if (n < 0 || (n > 0 && (!starts || !traces))) return fail(c, DSP_ERR_INVALID_ARG, "bad starts / traces / n");
  if (c->world > 1) {
    if (c->broken) return fail(c, DSP_ERR_STATE, "ctx unusable after an exchange failure");
    if (!c->walk_reserved) return fail(c, DSP_ERR_STATE, "random walks with world_size > 1 need dsp_reserve_walks");
    if (!c->imported) return fail(c, DSP_ERR_STATE, "dsp_import_handles first");
    if (n > c->walk_max) return fail(c, DSP_ERR_CAPACITY, "%lld walks > reserved %lld", (long long)n, (long long)c->walk_max);
    if (length > c->walk_len) return fail(c, DSP_ERR_CAPACITY, "length %d > reserved %d", length, c->walk_len);
  }
  return DSP_OK;
}

// all stages of a multi-rank walk call, stage by stage over the given ranks
dsp_status run_walks(std::vector<dsp_ctx *> &cs, std::vector<WalkArgs> &as, std::vector<cudaStream_t> &ss,
                     int32_t length) {
  const unsigned long long seq0 = cs[0]->wseq;
  for (auto *c : cs)
    if (c->wseq != seq0) return fail(cs[0], DSP_ERR_STATE, "ranks disagree on the number of walk calls");
  const size_t n = cs.size();
  // one cooperative launch per rank (k_walk_multi)
  std::vector<int> share(n, 0);
  for (size_t i = 0; i < n; ++i)
    for (auto *o : cs) share[i] += o->device == cs[i]->device ? 1 : 0;
  for (size_t i = 0; i < n; ++i) {
    dsp_ctx *c = cs[i];
    DeviceGuard g(c->device);
    CUDA_TRY(c, cudaMemsetAsync(c->d_walk_hdr, 0, sizeof(WsHeader), ss[i]));
    cudaStream_t st_i = ss[i];
    if (share[i] > 1) {  // virtual ranks: each on its own stream with 1/share of the SMs
      dsp_status fs = fork_aux(c, 0, ss[i], &st_i);
      if (fs != DSP_OK) return fs;
    }
    WalkPersistArgs p{};
    p.a = as[i];
    p.seq0 = seq0;
    p.hdr = c->d_walk_hdr;
    const dim3 grid(std::max(1, c->num_sms * c->walk_blocks_per_sm / share[i])), block(NT);
    void *args[] = {&p};
    CUDA_TRY(c, cudaLaunchCooperativeKernel((const void *)k_walk_multi, grid, block, args, 0, st_i));
  }
  for (size_t i = 0; i < n; ++i)
    if (share[i] > 1) {
      dsp_ctx *c = cs[i];
      DeviceGuard g(c->device);
      dsp_status js = join_aux(c, 0, ss[i]);
      if (js != DSP_OK) return js;
    }
  for (auto *c : cs) c->wseq = seq0 + 1 + (unsigned long long)length;
  return DSP_OK;
}

dsp_status check_gather_out(dsp_ctx *c, const float *out) {
  if (!c->d_feat) return fail(c, DSP_ERR_STATE, "no feature shard loaded");
  if (((uintptr_t)out & 15u) != 0) return fail(c, DSP_ERR_INVALID_ARG, "feature output must be 16-byte aligned");
  return DSP_OK;
}

}  // namespace

// ======================================================================= ABI
extern "C" {

int dsp_abi_version(void) { return DSP_ABI_VERSION; }

const char *dsp_status_str(int s) {
  switch (s) {
    case DSP_OK: return "DSP_OK";
    case DSP_ERR_INVALID_ARG: return "DSP_ERR_INVALID_ARG";
    case DSP_ERR_OUT_OF_RANGE: return "DSP_ERR_OUT_OF_RANGE";
    case DSP_ERR_DUPLICATE_SEED: return "DSP_ERR_DUPLICATE_SEED";
    case DSP_ERR_CAPACITY: return "DSP_ERR_CAPACITY";
    case DSP_ERR_STATE: return "DSP_ERR_STATE";
    case DSP_ERR_CUDA: return "DSP_ERR_CUDA";
    case DSP_ERR_PEER: return "DSP_ERR_PEER";
    case DSP_ERR_OOM: return "DSP_ERR_OOM";
    default: return "DSP_ERR_UNKNOWN";
  }
}

const char *dsp_last_error(const dsp_ctx *ctx) { return ctx ? ctx->err.c_str() : g_create_error.c_str(); }

dsp_status dsp_create(int32_t rank, int32_t world_size, int32_t cuda_device, dsp_ctx **out) {
  g_create_error.clear();
  if (!out) return fail(nullptr, DSP_ERR_INVALID_ARG, "out is NULL");
  *out = nullptr;
  if (world_size < 1 || world_size > DSP_MAX_WORLD || rank < 0 || rank >= world_size)
    return fail(nullptr, DSP_ERR_INVALID_ARG, "rank %d / world_size %d invalid (max %d)", rank,
                world_size, DSP_MAX_WORLD);
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || cuda_device < 0 || cuda_device >= ndev) {
    cudaGetLastError();
    return fail(nullptr, DSP_ERR_CUDA, "CUDA device %d not available (%d devices)", cuda_device, ndev);
  }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, cuda_device) != cudaSuccess)
    return fail(nullptr, DSP_ERR_CUDA, "cudaGetDeviceProperties failed");
  if (prop.major != 10)
    return fail(nullptr, DSP_ERR_CUDA, "device %d is sm_%d%d; libdsp is built for sm_100a only",
                cuda_device, prop.major, prop.minor);
  if (!prop.cooperativeLaunch)
    return fail(nullptr, DSP_ERR_CUDA, "device %d lacks cooperative launch", cuda_device);
  dsp_ctx *c = new dsp_ctx();
#ifdef DSP_SPLIT_DEFAULT  // experiment build (_build.build_variant): split feature rows by default
  c->split_rows = true;
#endif
  c->rank = rank;
  c->world = world_size;
  c->device = cuda_device;
  c->num_sms = prop.multiProcessorCount;
  DeviceGuard g(cuda_device);
  int occ = 0, occ_pipe = 0;
  const int pipe_smem = std::min(LOADER_WARPS * LOADER_SLOTS * 16384, 200 * 1024);  // largest ring (dim 4096)
  // each pipelined kernel may use up to the largest ring that fits beside its static shared memory
  auto ring_cap = [&](const void *f) {
    cudaFuncAttributes fa{};
    if (cudaFuncGetAttributes(&fa, f) != cudaSuccess) return -1;
    return std::min(pipe_smem, (int)prop.sharedMemPerBlockOptin - (int)fa.sharedSizeBytes);
  };
  const void *pk[4] = {(const void *)k_csp_persistent<PIPE_TEAM, true, false>,
                       (const void *)k_csp_persistent<BIASED_PIPE_TEAM, true, true, BIASED_BLK>,
                       (const void *)k_csp_multi<PIPE_TEAM, true, false>, (const void *)k_csp_multi<PIPE_TEAM, true, true>};
  bool attr_ok = true;
  for (const void *f : pk) {
    const int cap = ring_cap(f);
    attr_ok = attr_ok && cap > 0 && cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, cap) == cudaSuccess;
  }
  if (!attr_ok ||
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_csp_persistent<PNT, false, false>, PNT, 0) != cudaSuccess ||
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_pipe, k_csp_persistent<PIPE_TEAM, true, false>, PNT,
                                                    ring_cap(pk[0])) != cudaSuccess ||
      occ < 1 || occ_pipe < 1) {
    cudaGetLastError();
    delete c;
    return fail(nullptr, DSP_ERR_CUDA, "occupancy query for the persistent kernel failed");
  }
  if (cudaFuncSetAttribute((const void *)k_lw_persistent, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)std::max(LW_ALLOC_SMEM, sizeof(int32_t) * 3 * (size_t)LW_MAX_SIZE)) != cudaSuccess ||
      cudaFuncSetAttribute((const void *)k_lw_multi, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)std::max(LW_ALLOC_SMEM, sizeof(int32_t) * 3 * (size_t)LW_MAX_SIZE)) != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return fail(nullptr, DSP_ERR_CUDA, "shared-memory attribute of the layer-wise kernel failed");
  }
  c->persist_blocks_per_sm = std::min(occ, occ_pipe);
  if (cudaFuncSetAttribute((const void *)k_gather_tma<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           GTMA_WARPS * GTMA_SLOTS * 16384) != cudaSuccess ||
      cudaFuncSetAttribute((const void *)k_gather_tma<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           GTMA_WARPS * GTMA_SLOTS * 16384) != cudaSuccess) {
    cudaGetLastError();
    c->gather_reg = true;  // no TMA gather: register loads
    c->tma_unavailable = true;
  }
  {
    int ow = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ow, k_walk_multi, NT, 0) == cudaSuccess && ow >= 1)
      c->walk_blocks_per_sm = std::min(ow, 2);
    cudaGetLastError();
  }
  if (c->persist_blocks_per_sm * c->num_sms > MAX_PERSIST_BLOCKS) c->persist_blocks_per_sm = MAX_PERSIST_BLOCKS / c->num_sms;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_gather, NT, 0) != cudaSuccess || occ < 1) {
    cudaGetLastError();
    delete c;
    return fail(nullptr, DSP_ERR_CUDA, "occupancy query for the gather kernel failed");
  }
  c->gather_blocks_per_sm = occ;
  if (cudaMallocHost(&c->h_hdr, sizeof(WsHeader)) != cudaSuccess ||
      cudaMallocHost(&c->h_err, sizeof(int)) != cudaSuccess ||
      cudaMalloc(&c->d_err, sizeof(int)) != cudaSuccess || cudaMemset(c->d_err, 0, sizeof(int)) != cudaSuccess) {
    cudaGetLastError();
    release(c);
    delete c;
    return fail(nullptr, DSP_ERR_OOM, "host/device allocation failed in dsp_create");
  }
  *out = c;
  return DSP_OK;
}

void dsp_destroy(dsp_ctx *ctx) {
  if (!ctx) return;
  release(ctx);
  delete ctx;
}

dsp_status dsp_load_partition(dsp_ctx *c, const int64_t *bounds, const int64_t *indptr,
                              const int32_t *indices, const float *features, int32_t dim) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (c->loaded) return fail(c, DSP_ERR_STATE, "partition already loaded");
  if (!bounds || !indptr) return fail(c, DSP_ERR_INVALID_ARG, "bounds / indptr is NULL");
  if (bounds[0] != 0) return fail(c, DSP_ERR_INVALID_ARG, "bounds[0] must be 0");
  for (int r = 0; r < c->world; ++r)
    if (bounds[r + 1] < bounds[r]) return fail(c, DSP_ERR_INVALID_ARG, "bounds must be non-decreasing");
  if (bounds[c->world] >= (1ll << 31)) return fail(c, DSP_ERR_INVALID_ARG, "N must be < 2^31");
  if (features && (dim < 4 || dim > 4096 || dim % 4 != 0))
    return fail(c, DSP_ERR_INVALID_ARG, "dim %d must be a multiple of 4 in [4, 4096]", dim);
  DeviceGuard g(c->device);
  for (int r = 0; r <= c->world; ++r) c->bounds[r] = bounds[r];
  c->N = bounds[c->world];
  c->lo = bounds[c->rank];
  c->n_local = bounds[c->rank + 1] - c->lo;
  const size_t ip_bytes = sizeof(int64_t) * (size_t)(c->n_local + 1);
  CUDA_TRY(c, cudaMalloc(&c->d_indptr, ip_bytes));
  CUDA_TRY(c, cudaMemcpy(c->d_indptr, indptr, ip_bytes, cudaMemcpyDefault));
  int64_t first = 0;
  CUDA_TRY(c, cudaMemcpy(&first, c->d_indptr, sizeof(int64_t), cudaMemcpyDeviceToHost));
  CUDA_TRY(c, cudaMemcpy(&c->nnz, c->d_indptr + c->n_local, sizeof(int64_t), cudaMemcpyDeviceToHost));
  if (first != 0 || c->nnz < 0) return fail(c, DSP_ERR_INVALID_ARG, "indptr[0] must be 0");
  if (c->nnz > 0 && !indices) return fail(c, DSP_ERR_INVALID_ARG, "indices is NULL");
  CUDA_TRY(c, cudaMalloc(&c->d_indices, sizeof(int32_t) * (size_t)std::max<int64_t>(1, c->nnz)));
  if (c->nnz > 0) {
    CUDA_TRY(c, cudaMemcpy(c->d_indices, indices, sizeof(int32_t) * (size_t)c->nnz, cudaMemcpyDefault));
    CUDA_TRY(c, cudaMemset(c->d_err, 0, sizeof(int)));
    k_validate_indices<<<c->num_sms * 8, 256>>>(c->d_indices, c->nnz, c->N, c->d_err);
    int bad = 0;
    CUDA_TRY(c, cudaMemcpy(&bad, c->d_err, sizeof(int), cudaMemcpyDeviceToHost));
    CUDA_TRY(c, cudaMemset(c->d_err, 0, sizeof(int)));
    if (bad) return fail(c, DSP_ERR_OUT_OF_RANGE, "indices contain ids outside [0, N)");
  }
  if (features) {
    c->dim = dim;
    c->feat_slots = c->n_local;
    c->feat_bytes = (int64_t)region_bytes(c->split_rows, c->n_local, dim);
    CUDA_TRY(c, cudaMalloc(&c->d_feat, (size_t)c->feat_bytes));
    const size_t hb = (size_t)head_bytes_of(c->split_rows, dim), tb = (size_t)tail_bytes_of(c->split_rows, dim), rb = sizeof(float) * dim;
    char *dst = reinterpret_cast<char *>(c->d_feat);
    if (c->n_local > 0 && hb)
      CUDA_TRY(c, cudaMemcpy2D(dst, hb, features, rb, hb, (size_t)c->n_local, cudaMemcpyDefault));
    if (c->n_local > 0 && tb)
      CUDA_TRY(c, cudaMemcpy2D(dst + tail_offset(c->split_rows, c->n_local, dim), tb, reinterpret_cast<const char *>(features) + hb, rb,
                               tb, (size_t)c->n_local, cudaMemcpyDefault));
  }
  c->peer_feat[c->rank] = c->d_feat;
  c->peer_feat_tail[c->rank] =
      c->d_feat ? reinterpret_cast<const float *>(reinterpret_cast<const char *>(c->d_feat) + tail_offset(c->split_rows, c->n_local, dim))
                : nullptr;
  c->loaded = true;
  return DSP_OK;
}

dsp_status dsp_load_features_tiered(dsp_ctx *c, const float *features, int32_t dim, int64_t hot_rows) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition (with features = NULL) first");
  if (c->d_feat || c->tiered) return fail(c, DSP_ERR_STATE, "features already loaded");
  if (c->reserved && c->world > 1) return fail(c, DSP_ERR_STATE, "load features before dsp_reserve");
  if (!features && c->n_local > 0) return fail(c, DSP_ERR_INVALID_ARG, "features is NULL");
  if (dim < 4 || dim > 4096 || dim % 4 != 0)
    return fail(c, DSP_ERR_INVALID_ARG, "dim %d must be a multiple of 4 in [4, 4096]", dim);
  const int64_t n = c->n_local;
  if (hot_rows < 0 || hot_rows > n) hot_rows = n;
  DeviceGuard g(c->device);
  c->dim = dim;
  const size_t row_bytes = sizeof(float) * (size_t)dim, hb = (size_t)head_bytes_of(c->split_rows, dim), tb = (size_t)tail_bytes_of(c->split_rows, dim);
  // hot rows: the hot_rows largest in-degrees (P:L114 default criterion), ties by id
  std::vector<int64_t> ip((size_t)n + 1);
  CUDA_TRY(c, cudaMemcpy(ip.data(), c->d_indptr, sizeof(int64_t) * (size_t)(n + 1), cudaMemcpyDeviceToHost));
  std::vector<int32_t> order((size_t)n);
  for (int64_t v = 0; v < n; ++v) order[(size_t)v] = (int32_t)v;
  std::stable_sort(order.begin(), order.end(), [&](int32_t x, int32_t y) {
    return ip[(size_t)x + 1] - ip[(size_t)x] > ip[(size_t)y + 1] - ip[(size_t)y];
  });
  std::vector<char> hot((size_t)n, 0);
  for (int64_t j = 0; j < hot_rows; ++j) hot[(size_t)order[(size_t)j]] = 1;
  std::vector<int32_t> fpos((size_t)n);
  int64_t nh = 0, nc = 0;
  for (int64_t v = 0; v < n; ++v) fpos[(size_t)v] = hot[(size_t)v] ? (int32_t)nh++ : (int32_t)(-(++nc));
  // host staging of the rows (the input may live on the device)
  std::vector<float> src;
  const float *hsrc = features;
  cudaPointerAttributes at;
  if (n > 0 && cudaPointerGetAttributes(&at, features) == cudaSuccess &&
      (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged)) {
    src.resize((size_t)n * dim);
    CUDA_TRY(c, cudaMemcpy(src.data(), features, row_bytes * (size_t)n, cudaMemcpyDeviceToHost));
    hsrc = src.data();
  }
  cudaGetLastError();
  // a row into slot q of a split region (head array, then the tail array at tail_offset)
  auto put_row = [&](char *region, int64_t slots, int64_t q, const float *row) {
    memcpy(region + (size_t)q * hb, row, hb);
    memcpy(region + tail_offset(c->split_rows, slots, dim) + (size_t)q * tb, reinterpret_cast<const char *>(row) + hb, tb);
  };
  // hot rows -> HBM, cold rows -> pinned host memory (UVA-mapped), both split head / tail
  c->feat_slots = nh;
  c->cold_slots = nc;
  c->feat_bytes = (int64_t)region_bytes(c->split_rows, nh, dim);
  CUDA_TRY(c, cudaMalloc(&c->d_feat, (size_t)c->feat_bytes));
  {
    std::vector<char> stage((size_t)c->feat_bytes, 0);
    for (int64_t v = 0; v < n; ++v)
      if (fpos[(size_t)v] >= 0) put_row(stage.data(), nh, fpos[(size_t)v], hsrc + (size_t)v * dim);
    CUDA_TRY(c, cudaMemcpy(c->d_feat, stage.data(), (size_t)c->feat_bytes, cudaMemcpyHostToDevice));
  }
  c->cold_bytes = (int64_t)region_bytes(c->split_rows, nc, dim);
  if (c->world > 1) {  // cross-process readable: POSIX shm registered with CUDA
    static int counter = 0;
    snprintf(c->cold_shm, sizeof(c->cold_shm), "/dsp_cold_%d_%d_%d", (int)getpid(), c->rank, counter++);
    int fd = shm_open(c->cold_shm, O_CREAT | O_EXCL | O_RDWR, 0600);
    if (fd < 0) return fail(c, DSP_ERR_OOM, "shm_open(%s) failed", c->cold_shm);
    if (ftruncate(fd, (off_t)c->cold_bytes) != 0) {
      close(fd);
      shm_unlink(c->cold_shm);
      return fail(c, DSP_ERR_OOM, "ftruncate of the cold shm failed");
    }
    void *p = mmap(nullptr, (size_t)c->cold_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) {
      shm_unlink(c->cold_shm);
      return fail(c, DSP_ERR_OOM, "mmap of the cold shm failed");
    }
    c->h_cold = static_cast<float *>(p);
    CUDA_TRY(c, cudaHostRegister(c->h_cold, (size_t)c->cold_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
  } else {
    CUDA_TRY(c, cudaHostAlloc((void **)&c->h_cold, (size_t)c->cold_bytes, cudaHostAllocMapped | cudaHostAllocPortable));
  }
  for (int64_t v = 0; v < n; ++v)
    if (fpos[(size_t)v] < 0)
      put_row(reinterpret_cast<char *>(c->h_cold), nc, -fpos[(size_t)v] - 1, hsrc + (size_t)v * dim);
  CUDA_TRY(c, cudaMalloc(&c->d_fpos, sizeof(int32_t) * (size_t)std::max<int64_t>(1, n)));
  if (n > 0) CUDA_TRY(c, cudaMemcpy(c->d_fpos, fpos.data(), sizeof(int32_t) * (size_t)n, cudaMemcpyHostToDevice));
  void *dev_cold = nullptr;
  CUDA_TRY(c, cudaHostGetDevicePointer(&dev_cold, c->h_cold, 0));
  c->tiered = true;
  c->cold_regloads = c->gather_reg;
  c->peer_feat[c->rank] = c->d_feat;
  c->peer_feat_tail[c->rank] = reinterpret_cast<const float *>(reinterpret_cast<const char *>(c->d_feat) + tail_offset(c->split_rows, nh, dim));
  c->peer_fpos[c->rank] = nc > 0 ? c->d_fpos : nullptr;  // all hot: fpos is the identity
  c->peer_cold[c->rank] = static_cast<const float *>(dev_cold);
  c->peer_cold_tail[c->rank] = reinterpret_cast<const float *>(static_cast<const char *>(dev_cold) + tail_offset(c->split_rows, nc, dim));
  return DSP_OK;
}

dsp_status dsp_load_weights(dsp_ctx *c, const float *edge_weights) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  if (c->d_weights) return fail(c, DSP_ERR_STATE, "weights already loaded");
  if (!edge_weights && c->nnz > 0) return fail(c, DSP_ERR_INVALID_ARG, "edge_weights is NULL");
  DeviceGuard g(c->device);
  const size_t n = (size_t)std::max<int64_t>(1, c->nnz);
  // 32 zero words of padding: the biased sampler reads rows as whole aligned
  // 128-byte lines, the last one possibly past the last weight
  CUDA_TRY(c, cudaMalloc(&c->d_weights, sizeof(uint32_t) * (n + 32)));
  CUDA_TRY(c, cudaMemset(c->d_weights, 0, sizeof(uint32_t) * (n + 32)));
  if (c->nnz > 0) {
    float *tmp = nullptr;
    CUDA_TRY(c, cudaMalloc(&tmp, sizeof(float) * n));
    cudaError_t e = cudaMemcpy(tmp, edge_weights, sizeof(float) * (size_t)c->nnz, cudaMemcpyDefault);
    if (e == cudaSuccess) e = cudaMemset(c->d_err, 0, sizeof(int));
    if (e == cudaSuccess) {
      k_weights_fixed<<<c->num_sms * 8, 256>>>(tmp, c->nnz, c->d_weights, c->d_err);
      e = cudaGetLastError();
    }
    int bad = 0;
    if (e == cudaSuccess) e = cudaMemcpy(&bad, c->d_err, sizeof(int), cudaMemcpyDeviceToHost);
    cudaFree(tmp);
    cudaMemset(c->d_err, 0, sizeof(int));
    if (e != cudaSuccess) {
      cudaGetLastError();
      cudaFree(c->d_weights);
      c->d_weights = nullptr;
      return fail(c, DSP_ERR_CUDA, "dsp_load_weights: %s", cudaGetErrorString(e));
    }
    if (bad) {
      cudaFree(c->d_weights);
      c->d_weights = nullptr;
      return fail(c, DSP_ERR_INVALID_ARG,
                  "%d edge weights are neither 0 nor in [2^-16, 65536) (negative, NaN, too large, or a positive "
                  "weight that would quantize to 0 in 16.16 fixed point)", bad);
    }
  }
  return DSP_OK;
}

dsp_status dsp_reserve(dsp_ctx *c, int32_t max_seeds, const int32_t *fanouts, int32_t L) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  if (c->reserved) return fail(c, DSP_ERR_STATE, "already reserved");
  dsp_status st = check_fanouts(c, fanouts, L);
  if (st != DSP_OK) return st;
  if (max_seeds < 0) return fail(c, DSP_ERR_INVALID_ARG, "max_seeds < 0");
  Plan p = make_plan(c->N, max_seeds, fanouts, L, c->relabel_mode);
  for (int l = 0; l < L; ++l)
    if ((uint64_t)p.F[l] + (uint64_t)p.E[l] >= (1ull << 31))
      return fail(c, DSP_ERR_CAPACITY, "layer %d: frontier * (1 + fanout) exceeds 2^31", l);
  c->max_seeds = max_seeds;
  c->L = L;
  c->kmax = 0;
  for (int l = 0; l < L; ++l) {
    c->fanouts[l] = fanouts[l];
    c->kmax = std::max(c->kmax, fanouts[l]);
  }
  if (c->world > 1) {
    DeviceGuard g(c->device);
    c->xl = make_xch_layout(std::max<int64_t>(1, p.max_F), c->kmax);
    c->chan_stride = align_up(c->xl.bytes, 256);
    CUDA_TRY(c, cudaMalloc(&c->d_xch, c->chan_stride * (size_t)c->channels));
    CUDA_TRY(c, cudaMemset(c->d_xch, 0, c->chan_stride * (size_t)c->channels));
    for (int ch = 0; ch < c->channels && c->channels > 1; ++ch)
      CUDA_TRY(c, cudaEventCreateWithFlags(&c->chan_ev[ch], cudaEventDisableTiming));
    CUDA_TRY(c, cudaDeviceSynchronize());
  }
  c->peer_xch[c->rank] = c->d_xch;
  c->reserved = true;
  return DSP_OK;
}

dsp_status dsp_reserve_layerwise(dsp_ctx *c, int32_t max_seeds, const int32_t *sizes, int32_t L) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  if (c->lw_reserved) return fail(c, DSP_ERR_STATE, "layer-wise already reserved");
  if (c->imported) return fail(c, DSP_ERR_STATE, "reserve before dsp_import_handles");
  dsp_status st = check_sizes(c, sizes, L);
  if (st != DSP_OK) return st;
  if (max_seeds < 0) return fail(c, DSP_ERR_INVALID_ARG, "max_seeds < 0");
  Plan p = make_plan_lw(c->N, max_seeds, sizes, L, c->world == 1);
  for (int l = 0; l < L; ++l)
    if ((uint64_t)p.F[l] + (uint64_t)p.E[l] >= (1ull << 31))
      return fail(c, DSP_ERR_CAPACITY, "layer %d: frontier + layer size exceeds 2^31", l);
  DeviceGuard g(c->device);
  c->lxl = make_lw_layout(std::max<int64_t>(1, p.max_F), (int32_t)p.ncap);
  CUDA_TRY(c, cudaMalloc(&c->d_lxch, c->lxl.bytes));
  CUDA_TRY(c, cudaMemset(c->d_lxch, 0, c->lxl.bytes));
  CUDA_TRY(c, cudaDeviceSynchronize());
  c->lw_max_seeds = max_seeds;
  c->lw_L = L;
  for (int l = 0; l < L; ++l) c->lw_sizes[l] = sizes[l];
  c->peer_lxch[c->rank] = c->d_lxch;
  c->peer_indptr[c->rank] = c->d_indptr;
  c->lw_reserved = true;
  return DSP_OK;
}

dsp_status dsp_sample_bounds_layerwise(const dsp_ctx *cc, int32_t num_seeds, const int32_t *sizes, int32_t L,
                                       int64_t *max_src, int64_t *max_edges, size_t *workspace_bytes) {
  dsp_ctx *c = const_cast<dsp_ctx *>(cc);
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  dsp_status st = check_sizes(c, sizes, L);
  if (st != DSP_OK) return st;
  if (num_seeds < 0) return fail(c, DSP_ERR_INVALID_ARG, "num_seeds < 0");
  if (c->lw_reserved && num_seeds > c->lw_max_seeds)
    return fail(c, DSP_ERR_CAPACITY, "num_seeds %d > reserved max_seeds %d", num_seeds, c->lw_max_seeds);
  Plan p = make_plan_lw(c->N, c->lw_reserved ? c->lw_max_seeds : num_seeds, sizes, L, c->world == 1);
  for (int l = 0; l < L; ++l) {
    if (max_src) max_src[l] = p.S[l];
    if (max_edges) max_edges[l] = p.E[l];
  }
  if (workspace_bytes) *workspace_bytes = p.bytes;
  return DSP_OK;
}

dsp_status dsp_export_handle(const dsp_ctx *cc, void *out) {
  dsp_ctx *c = const_cast<dsp_ctx *>(cc);
  if (!c || !out) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded || !(c->reserved || c->lw_reserved || c->walk_reserved))
    return fail(c, DSP_ERR_STATE, "load_partition + reserve first");
  PeerHandle h;
  memset(&h, 0, sizeof(h));
  h.magic = HANDLE_MAGIC;
  h.rank = c->rank;
  h.world = c->world;
  h.device = c->device;
  h.pid = (int64_t)getpid();
  h.boot_id = boot_id();
  h.feat_ptr = (uint64_t)(uintptr_t)c->d_feat;
  h.xch_ptr = (uint64_t)(uintptr_t)c->d_xch;
  h.feat_bytes = c->feat_bytes;
  h.xch_bytes = (int64_t)(c->chan_stride * (size_t)c->channels);
  h.channels = c->channels;
  h.dim = c->dim;
  h.head_bytes = head_bytes_of(c->split_rows, c->dim);
  h.feat_slots = c->feat_slots;
  h.cold_slots = c->cold_slots;
  h.max_seeds = c->max_seeds;
  for (int r = 0; r <= c->world; ++r) h.bounds[r] = c->bounds[r];
  DeviceGuard g(c->device);
  if (c->d_feat && c->world > 1) {
    h.has_feat = 1;
    CUDA_TRY(c, cudaIpcGetMemHandle(&h.feat_ipc, c->d_feat));
  }
  if (c->d_xch) {
    h.has_xch = 1;
    CUDA_TRY(c, cudaIpcGetMemHandle(&h.xch_ipc, c->d_xch));
  }
  h.tiered = c->tiered ? 1 : 0;
  if (c->tiered) {
    h.fpos_ptr = (uint64_t)(uintptr_t)c->peer_fpos[c->rank];
    h.cold_ptr = (uint64_t)(uintptr_t)c->peer_cold[c->rank];
    h.cold_bytes = c->cold_bytes;
    memcpy(h.cold_shm, c->cold_shm, sizeof(h.cold_shm));
    if (c->world > 1 && h.fpos_ptr) CUDA_TRY(c, cudaIpcGetMemHandle(&h.fpos_ipc, c->d_fpos));
  }
  h.lw_max_seeds = c->lw_reserved ? c->lw_max_seeds : -1;
  h.lw_L = c->lw_L;
  for (int l = 0; l < DSP_MAX_LAYERS; ++l) h.lw_sizes[l] = c->lw_sizes[l];
  if (c->lw_reserved) {
    h.has_lxch = 1;
    h.lxch_ptr = (uint64_t)(uintptr_t)c->d_lxch;
    h.indptr_ptr = (uint64_t)(uintptr_t)c->d_indptr;
    if (c->world > 1) {
      CUDA_TRY(c, cudaIpcGetMemHandle(&h.lxch_ipc, c->d_lxch));
      CUDA_TRY(c, cudaIpcGetMemHandle(&h.indptr_ipc, c->d_indptr));
    }
  }
  h.walk_max = c->walk_reserved ? c->walk_max : -1;
  h.walk_len = c->walk_len;
  if (c->walk_reserved) {
    h.has_wxch = 1;
    h.wxch_ptr = (uint64_t)(uintptr_t)c->d_wxch;
    if (c->world > 1) CUDA_TRY(c, cudaIpcGetMemHandle(&h.wxch_ipc, c->d_wxch));
  }
  memset(out, 0, DSP_HANDLE_BYTES);
  memcpy(out, &h, sizeof(h));
  return DSP_OK;
}

dsp_status dsp_import_handles(dsp_ctx *c, const void *all) {
  if (!c || !all) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded || !(c->reserved || c->lw_reserved || c->walk_reserved))
    return fail(c, DSP_ERR_STATE, "load_partition + reserve first");
  if (c->imported) return fail(c, DSP_ERR_STATE, "handles already imported");
  DeviceGuard g(c->device);
  const int64_t my_pid = (int64_t)getpid();
  for (int r = 0; r < c->world; ++r) {
    PeerHandle h;
    memcpy(&h, static_cast<const char *>(all) + (size_t)r * DSP_HANDLE_BYTES, sizeof(h));
    if (h.magic != HANDLE_MAGIC || h.rank != r || h.world != c->world)
      return fail(c, DSP_ERR_INVALID_ARG, "handle %d is not rank %d of this world", r, r);
    for (int q = 0; q <= c->world; ++q)
      if (h.bounds[q] != c->bounds[q]) return fail(c, DSP_ERR_STATE, "rank %d has different bounds", r);
    if (h.dim != c->dim || h.head_bytes != head_bytes_of(c->split_rows, c->dim) || h.max_seeds != c->max_seeds)
      return fail(c, DSP_ERR_STATE, "rank %d has a different dim / max_seeds", r);
    if (h.has_xch && h.channels != c->channels)
      return fail(c, DSP_ERR_STATE, "rank %d reserved %d exchange channels, this rank %d", r, h.channels, c->channels);
    if ((h.tiered != 0) != c->tiered) return fail(c, DSP_ERR_STATE, "all ranks must use the cold tier or none");
    if (h.lw_max_seeds != (c->lw_reserved ? c->lw_max_seeds : -1) || h.lw_L != c->lw_L ||
        memcmp(h.lw_sizes, c->lw_sizes, sizeof(c->lw_sizes)) != 0)
      return fail(c, DSP_ERR_STATE, "rank %d reserved a different layer-wise configuration", r);
    if (h.walk_max != (c->walk_reserved ? c->walk_max : -1) || h.walk_len != c->walk_len)
      return fail(c, DSP_ERR_STATE, "rank %d reserved a different random-walk configuration", r);
    if (r == c->rank) continue;
    const bool same_process = h.pid == my_pid && h.boot_id == boot_id();
    if (same_process) {
      if (h.device != c->device) {
        cudaError_t e = cudaDeviceEnablePeerAccess(h.device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaDeviceEnablePeerAccess(%d -> %d): %s", c->device, h.device,
                      cudaGetErrorString(e));
        }
        cudaGetLastError();
      }
      c->peer_feat[r] = reinterpret_cast<const float *>(h.feat_ptr);
      c->peer_xch[r] = reinterpret_cast<char *>(h.xch_ptr);
      if (h.tiered) {
        c->peer_fpos[r] = reinterpret_cast<const int32_t *>(h.fpos_ptr);
        c->peer_cold[r] = reinterpret_cast<const float *>(h.cold_ptr);
      }
      if (h.has_lxch) {
        c->peer_lxch[r] = reinterpret_cast<char *>(h.lxch_ptr);
        c->peer_indptr[r] = reinterpret_cast<const int64_t *>(h.indptr_ptr);
      }
      if (h.has_wxch) c->peer_wxch[r] = reinterpret_cast<char *>(h.wxch_ptr);
    } else {
      if (h.has_wxch) {
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h.wxch_ipc, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaIpcOpenMemHandle(walk region of rank %d): %s", r, cudaGetErrorString(e));
        }
        c->ipc_opened[5 * DSP_MAX_WORLD + r] = p;
        c->peer_wxch[r] = static_cast<char *>(p);
      }
      if (h.has_lxch) {
        void *p = nullptr, *q = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h.lxch_ipc, cudaIpcMemLazyEnablePeerAccess);
        if (e == cudaSuccess) {
          c->ipc_opened[3 * DSP_MAX_WORLD + r] = p;
          e = cudaIpcOpenMemHandle(&q, h.indptr_ipc, cudaIpcMemLazyEnablePeerAccess);
        }
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaIpcOpenMemHandle(layer-wise region / indptr of rank %d): %s", r,
                      cudaGetErrorString(e));
        }
        c->ipc_opened[4 * DSP_MAX_WORLD + r] = q;
        c->peer_lxch[r] = static_cast<char *>(p);
        c->peer_indptr[r] = static_cast<const int64_t *>(q);
      }
      if (h.tiered && h.fpos_ptr) {
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h.fpos_ipc, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaIpcOpenMemHandle(fpos of rank %d): %s", r, cudaGetErrorString(e));
        }
        c->ipc_opened[2 * DSP_MAX_WORLD + r] = p;
        c->peer_fpos[r] = static_cast<const int32_t *>(p);
        int fd = shm_open(h.cold_shm, O_RDWR, 0);
        if (fd < 0) return fail(c, DSP_ERR_PEER, "shm_open(%s) of rank %d failed", h.cold_shm, r);
        void *m = mmap(nullptr, (size_t)h.cold_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
        close(fd);
        if (m == MAP_FAILED) return fail(c, DSP_ERR_PEER, "mmap of rank %d's cold rows failed", r);
        c->peer_cold_map[r] = m;
        c->peer_cold_bytes[r] = h.cold_bytes;
        e = cudaHostRegister(m, (size_t)h.cold_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
        void *dp = nullptr;
        if (e == cudaSuccess) e = cudaHostGetDevicePointer(&dp, m, 0);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaHostRegister of rank %d's cold rows: %s", r, cudaGetErrorString(e));
        }
        c->peer_cold[r] = static_cast<const float *>(dp);
      }
      if (h.has_feat) {
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h.feat_ipc, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaIpcOpenMemHandle(features of rank %d): %s", r, cudaGetErrorString(e));
        }
        c->ipc_opened[2 * r] = p;
        c->peer_feat[r] = static_cast<const float *>(p);
      }
      if (h.has_xch) {
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h.xch_ipc, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
          cudaGetLastError();
          return fail(c, DSP_ERR_PEER, "cudaIpcOpenMemHandle(exchange of rank %d): %s", r, cudaGetErrorString(e));
        }
        c->ipc_opened[2 * r + 1] = p;
        c->peer_xch[r] = static_cast<char *>(p);
      }
    }
    // the tail arrays of rank r's split feature regions (dsp_kernels.cuh GatherArgs)
    if (c->peer_feat[r])
      c->peer_feat_tail[r] = reinterpret_cast<const float *>(reinterpret_cast<const char *>(c->peer_feat[r]) +
                                                             tail_offset(c->split_rows, h.feat_slots, c->dim));
    if (c->peer_cold[r])
      c->peer_cold_tail[r] = reinterpret_cast<const float *>(reinterpret_cast<const char *>(c->peer_cold[r]) +
                                                             tail_offset(c->split_rows, h.cold_slots, c->dim));
  }
  c->imported = true;
  return DSP_OK;
}

dsp_status dsp_sample_bounds(const dsp_ctx *cc, int32_t num_seeds, const int32_t *fanouts, int32_t L,
                             int64_t *max_src, int64_t *max_edges, size_t *workspace_bytes) {
  dsp_ctx *c = const_cast<dsp_ctx *>(cc);
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  dsp_status st = check_fanouts(c, fanouts, L);
  if (st != DSP_OK) return st;
  if (num_seeds < 0) return fail(c, DSP_ERR_INVALID_ARG, "num_seeds < 0");
  if (c->reserved && num_seeds > c->max_seeds)
    return fail(c, DSP_ERR_CAPACITY, "num_seeds %d > reserved max_seeds %d", num_seeds, c->max_seeds);
  Plan p = make_plan(c->N, c->reserved ? c->max_seeds : num_seeds, fanouts, L, c->relabel_mode);
  for (int l = 0; l < L; ++l) {
    if (max_src) max_src[l] = p.S[l];
    if (max_edges) max_edges[l] = p.E[l];
  }
  if (workspace_bytes) *workspace_bytes = p.bytes;
  return DSP_OK;
}

dsp_status dsp_sample(dsp_ctx *c, const int32_t *seeds, int32_t num_seeds, const int32_t *fanouts,
                      int32_t L, uint64_t rng_seed, dsp_block *blocks, void *workspace,
                      size_t workspace_bytes, uint32_t flags, void *stream) {
  std::vector<Call> calls(1);
  if ((flags & (DSP_ASYNC | DSP_PIPELINED)) != 0)
    return fail(c, DSP_ERR_INVALID_ARG, "dsp_sample takes DSP_BIASED only (async steps: dsp_sample_gather)");
  dsp_status st = prepare_call(calls[0], c, seeds, num_seeds, fanouts, L, rng_seed, blocks, workspace,
                               workspace_bytes, flags, stream);
  if (st != DSP_OK) return st;
  return run_calls(calls);
}

dsp_status dsp_sample_gather(dsp_ctx *c, const int32_t *seeds, int32_t num_seeds, const int32_t *fanouts,
                             int32_t L, uint64_t rng_seed, dsp_block *blocks, float *feat_out,
                             int64_t feat_cap_rows, void *workspace, size_t workspace_bytes,
                             int64_t *sizes_out, uint32_t flags, void *stream) {
  std::vector<Call> calls(1);
  dsp_status st = prepare_call(calls[0], c, seeds, num_seeds, fanouts, L, rng_seed, blocks, workspace,
                               workspace_bytes, flags, stream);
  if (st != DSP_OK) return st;
  if (!feat_out) return fail(c, DSP_ERR_INVALID_ARG, "feat_out is NULL");
  if ((st = check_gather_out(c, feat_out)) != DSP_OK) return st;
  if (c->world > 1 && !c->imported) return fail(c, DSP_ERR_STATE, "dsp_import_handles first");
  if (feat_cap_rows < calls[0].plan.S[L - 1])
    return fail(c, DSP_ERR_CAPACITY, "feat_cap_rows %lld < max_src[L-1] %lld", (long long)feat_cap_rows,
                (long long)calls[0].plan.S[L - 1]);
  if (calls[0].plan.S[L - 1] * (c->dim / 4) >= (1ll << 31))
    return fail(c, DSP_ERR_CAPACITY, "max_src[L-1] * dim / 4 must be < 2^31");
  calls[0].feat_out = feat_out;
  calls[0].sizes_out = sizes_out;
  calls[0].pipelined = (flags & DSP_PIPELINED) != 0;
  calls[0].async = (flags & (DSP_ASYNC | DSP_PIPELINED)) != 0;
  return run_calls(calls);
}

dsp_status dsp_set_persistent_blocks(dsp_ctx *c, int32_t blocks) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  const int maxb = c->num_sms * c->persist_blocks_per_sm;
  if (blocks < 0 || blocks > maxb)
    return fail(c, DSP_ERR_INVALID_ARG, "blocks %d not in [0, %d]", blocks, maxb);
  c->persist_blocks = blocks;
  return DSP_OK;
}

dsp_status dsp_set_option(dsp_ctx *c, int32_t option, int64_t value) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  switch (option) {
    case DSP_OPT_RELABEL_MAP:
      if (value < 0 || value > 3) return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_RELABEL_MAP %lld not in [0, 3]", (long long)value);
      if (c->reserved || c->lw_reserved)
        return fail(c, DSP_ERR_STATE, "DSP_OPT_RELABEL_MAP must be set before dsp_reserve (the workspace plan depends on it)");
      c->relabel_mode = (int)value;
      return DSP_OK;
    case DSP_OPT_LANE_ROUNDS:
      if (value < 1 || value > 1024) return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_LANE_ROUNDS %lld not in [1, 1024]", (long long)value);
      c->lane_rounds = (int)value;
      return DSP_OK;
    case DSP_OPT_LOADER_ROWS:
      if (value < 1 || value > 32) return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_LOADER_ROWS %lld not in [1, 32]", (long long)value);
      c->loader_rows = (int)value;
      return DSP_OK;
    case DSP_OPT_GATHER_REGLOADS:
      if (value != 0 && value != 1) return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_GATHER_REGLOADS must be 0 or 1");
      c->gather_reg = value != 0 || c->tma_unavailable;
      c->cold_regloads = c->gather_reg;
      return DSP_OK;
    case DSP_OPT_SPLIT_ROWS:
      if (value != 0 && value != 1) return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_SPLIT_ROWS must be 0 or 1");
      if (c->loaded) return fail(c, DSP_ERR_STATE, "DSP_OPT_SPLIT_ROWS must be set before dsp_load_partition");
      c->split_rows = value != 0;
      return DSP_OK;
    case DSP_OPT_EXCHANGE_CHANNELS:
      if (value < 1 || value > DSP_MAX_CHANNELS)
        return fail(c, DSP_ERR_INVALID_ARG, "DSP_OPT_EXCHANGE_CHANNELS %lld not in [1, %d]", (long long)value, DSP_MAX_CHANNELS);
      if (c->reserved) return fail(c, DSP_ERR_STATE, "DSP_OPT_EXCHANGE_CHANNELS must be set before dsp_reserve");
      c->channels = (int)value;
      return DSP_OK;
    default:
      return fail(c, DSP_ERR_INVALID_ARG, "unknown option %d", option);
  }
}

dsp_status dsp_pipeline_flush(dsp_ctx *c, void *stream) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  for (auto &p : c->pend)
    if (p.active) {
      dsp_status st = flush_one(c, p, static_cast<cudaStream_t>(stream));
      if (st != DSP_OK) return st;
    }
  return DSP_OK;
}

dsp_status dsp_sample_group(dsp_ctx *const *ctxs, int32_t n, const int32_t *const *seeds,
                            const int32_t *num_seeds, const int32_t *fanouts, int32_t L,
                            uint64_t rng_seed, dsp_block *const *blocks, void *const *workspaces,
                            size_t workspace_bytes, uint32_t flags, void *const *streams) {
  if (!ctxs || n < 1 || !seeds || !num_seeds || !blocks || !workspaces || !streams)
    return DSP_ERR_INVALID_ARG;
  const int world = ctxs[0] ? ctxs[0]->world : 0;
  if (n != world) return fail(ctxs[0], DSP_ERR_INVALID_ARG, "dsp_sample_group needs all %d ranks", world);
  std::vector<int> seen(world, 0);
  for (int i = 0; i < n; ++i) {
    if (!ctxs[i] || ctxs[i]->world != world || seen[ctxs[i]->rank]++)
      return fail(ctxs[0], DSP_ERR_INVALID_ARG, "ctxs must be the distinct ranks of one world");
    for (int j = 0; j < i; ++j)
      if (ctxs[j]->device == ctxs[i]->device && streams[j] != streams[i])
        return fail(ctxs[0], DSP_ERR_INVALID_ARG,
                    "virtual ranks on one device must share a stream (stage-by-stage issue)");
  }
  std::vector<Call> calls(n);
  for (int i = 0; i < n; ++i) {
    if ((flags & DSP_PIPELINED) != 0)
      return fail(ctxs[0], DSP_ERR_INVALID_ARG, "dsp_sample_group takes DSP_BIASED, DSP_LAYERWISE, DSP_ASYNC");
    dsp_status st = prepare_call(calls[i], ctxs[i], seeds[i], num_seeds[i], fanouts, L, rng_seed,
                                 blocks[i], workspaces[i], workspace_bytes, flags & ~DSP_ASYNC, streams[i]);
    if (st != DSP_OK) return st;
    calls[i].async = (flags & DSP_ASYNC) != 0;
  }
  return run_calls(calls);
}

dsp_status dsp_gather_features(dsp_ctx *c, const int32_t *ids, int64_t n, float *out, void *stream) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "no partition loaded");
  if (c->world > 1 && !c->imported) return fail(c, DSP_ERR_STATE, "dsp_import_handles first");
  if (n < 0 || (n > 0 && (!ids || !out))) return fail(c, DSP_ERR_INVALID_ARG, "bad ids / out / n");
  dsp_status st = check_gather_out(c, out);
  if (st != DSP_OK) return st;
  if (n == 0) return DSP_OK;
  DeviceGuard g(c->device);
  GatherArgs a = make_gather(c, ids, n, nullptr, out);
  if (n * a.dim4 >= (1ll << 31)) return fail(c, DSP_ERR_CAPACITY, "n * dim / 4 must be < 2^31 per call");
  return launch_gather(c, a, n, static_cast<cudaStream_t>(stream));
}

dsp_status dsp_random_walk(dsp_ctx *c, const int32_t *starts, int64_t n, int32_t length, uint64_t rng_seed,
                           int32_t *traces, uint32_t flags, void *stream) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if ((flags & ~DSP_WALK_INDEPENDENT) != 0) return fail(c, DSP_ERR_INVALID_ARG, "unknown walk flags 0x%x", flags);
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  dsp_status st = check_walk_call(c, starts, n, length, traces);
  if (st != DSP_OK) return st;
  if (c->world > 1) {  // COLLECTIVE: CSP push without reshuffle
    std::vector<dsp_ctx *> cs{c};
    std::vector<WalkArgs> as{walk_args(c, starts, n, length, rng_seed, traces, flags)};
    std::vector<cudaStream_t> ss{static_cast<cudaStream_t>(stream)};
    return run_walks(cs, as, ss, length);
  }
  if (n == 0) return DSP_OK;
  DeviceGuard g(c->device);
  const int64_t want = (n + NT - 1) / NT;
  k_random_walk<<<(int)std::min<int64_t>(want, grid_for(c, 8)), NT, 0, static_cast<cudaStream_t>(stream)>>>(
      starts, n, length, key_of(rng_seed), c->d_indptr, c->d_indices, c->N, traces, c->d_err,
      (flags & DSP_WALK_INDEPENDENT) ? 1 : 0);
  CUDA_TRY(c, cudaGetLastError());
  return DSP_OK;
}

dsp_status dsp_random_walk_group(dsp_ctx *const *ctxs, int32_t n_ctx, const int32_t *const *starts,
                                 const int64_t *n, int32_t length, uint64_t rng_seed, int32_t *const *traces,
                                 uint32_t flags, void *const *streams) {
  if (!ctxs || n_ctx < 1 || !starts || !n || !traces || !streams) return DSP_ERR_INVALID_ARG;
  if ((flags & ~DSP_WALK_INDEPENDENT) != 0) return fail(ctxs[0], DSP_ERR_INVALID_ARG, "unknown walk flags 0x%x", flags);
  const int world = ctxs[0] ? ctxs[0]->world : 0;
  if (n_ctx != world) return fail(ctxs[0], DSP_ERR_INVALID_ARG, "dsp_random_walk_group needs all %d ranks", world);
  std::vector<int> seen(world, 0);
  std::vector<dsp_ctx *> cs(n_ctx);
  std::vector<WalkArgs> as(n_ctx);
  std::vector<cudaStream_t> ss(n_ctx);
  for (int i = 0; i < n_ctx; ++i) {
    if (!ctxs[i] || ctxs[i]->world != world || seen[ctxs[i]->rank]++)
      return fail(ctxs[0], DSP_ERR_INVALID_ARG, "ctxs must be the distinct ranks of one world");
    for (int j = 0; j < i; ++j)
      if (ctxs[j]->device == ctxs[i]->device && streams[j] != streams[i])
        return fail(ctxs[0], DSP_ERR_INVALID_ARG,
                    "virtual ranks on one device must share a stream (stage-by-stage issue)");
    ctxs[i]->err.clear();
    dsp_status st = check_walk_call(ctxs[i], starts[i], n[i], length, traces[i]);
    if (st != DSP_OK) return st;
    cs[i] = ctxs[i];
    as[i] = walk_args(ctxs[i], starts[i], n[i], length, rng_seed, traces[i], flags);
    ss[i] = static_cast<cudaStream_t>(streams[i]);
  }
  if (world == 1) return dsp_random_walk(ctxs[0], starts[0], n[0], length, rng_seed, traces[0], flags, streams[0]);
  return run_walks(cs, as, ss, length);
}

dsp_status dsp_reserve_walks(dsp_ctx *c, int64_t max_walks, int32_t max_length) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, DSP_ERR_STATE, "dsp_load_partition first");
  if (c->walk_reserved) return fail(c, DSP_ERR_STATE, "walks already reserved");
  if (c->imported) return fail(c, DSP_ERR_STATE, "reserve before dsp_import_handles");
  if (max_walks < 0 || max_walks > WALK_MAX) return fail(c, DSP_ERR_INVALID_ARG, "max_walks must be in [0, 2^27]");
  if (max_length < 1 || max_length > 1024) return fail(c, DSP_ERR_INVALID_ARG, "max_length must be in [1, 1024]");
  DeviceGuard g(c->device);
  c->wl = make_walk_layout(c->world, max_walks, max_length);
  CUDA_TRY(c, cudaMalloc(&c->d_walk_hdr, sizeof(WsHeader)));
  CUDA_TRY(c, cudaMalloc(&c->d_wxch, c->wl.bytes));
  CUDA_TRY(c, cudaMemset(c->d_wxch, 0, c->wl.bytes));
  CUDA_TRY(c, cudaDeviceSynchronize());
  c->walk_max = max_walks;
  c->walk_len = max_length;
  c->peer_wxch[c->rank] = c->d_wxch;
  c->walk_reserved = true;
  return DSP_OK;
}

dsp_status dsp_sync(dsp_ctx *c, void *stream) {
  if (!c) return DSP_ERR_INVALID_ARG;
  c->err.clear();
  DeviceGuard g(c->device);
  CUDA_TRY(c, cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  int e = 0;
  CUDA_TRY(c, cudaMemcpy(&e, c->d_err, sizeof(int), cudaMemcpyDeviceToHost));
  if (e != 0) {
    CUDA_TRY(c, cudaMemset(c->d_err, 0, sizeof(int)));
    if (e == E_STATE && c->world > 1) c->broken = true;
    return fail(c, (dsp_status)e, "device-detected error %d (%s)", e, dsp_status_str(e));
  }
  return DSP_OK;
}

}  // extern "C"
