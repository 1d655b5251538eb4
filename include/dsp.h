/*
 * dsp.h -- C ABI of libdsp.so: DSP's collective sampling primitive (CSP) and
 * feature gather on B200 (sm_100a).  ABI version 1.
 *
 * PAPER.md = "DSP: Efficient GNN Training with Multiple GPUs" (PPoPP'23);
 * "P:L<n>" cites its line n.  DESIGN.md "Readings" R1..R23 fix every point
 * the paper leaves open.
 *
 * Model.  The graph's topology (CSR of in-neighbours, global ids in the rows)
 * and its node features are partitioned over `world_size` GPUs by contiguous
 * ranges of renumbered global ids: rank r owns [bounds[r], bounds[r+1])
 * (P:L112-116 data layout, P:L222 renumbering / range check).  One dsp_ctx
 * per (process, GPU) -- or several ctxs driven by one host thread with
 * dsp_sample_group.  A mini-batch's seeds are sampled layer by layer with CSP
 * (shuffle -> sample -> reshuffle) into per-layer blocks, then
 * the features of the sampled nodes are gathered (P:L126 loader).
 *
 * Conventions (all functions):
 *   * Every function returns a dsp_status; none throws, aborts or prints.
 *     dsp_last_error(ctx) gives a one-line detail of the last failure.
 *   * Pointers documented as DEVICE must be CUDA device pointers on the ctx's
 *     device; HOST pointers are ordinary host memory; "host or device" is
 *     detected with cudaPointerGetAttributes.
 *   * `stream` is a cudaStream_t passed as void* (0 = legacy default stream).
 *   * The caller owns every buffer it passes; the library owns its copies of
 *     the shards and its peer-visible exchange buffers.
 *   * No allocation after dsp_reserve: dsp_sample / dsp_gather_features use
 *     only the caller's workspace and library buffers sized at reserve time
 *     (the paper's deadlock hazard of cudaMalloc against in-flight
 *     communication, does not arise).
 *   * COLLECTIVE calls must be made by every rank in the same order with the
 *     same scalar arguments (the "fixed launch order" that CCC enforces,
 *     P:L210-216, with a trivial leader).  Mismatched fanouts / rng_seed are
 *     detected in the exchange header and reported as DSP_ERR_STATE.
 */
#ifndef DSP_H_
#define DSP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DSP_ABI_VERSION 1
#define DSP_MAX_WORLD 8      /* one NVSwitch node */
#define DSP_MAX_LAYERS 8
#define DSP_MAX_FANOUT 32    /* one lane per sampled slot */
#define DSP_HANDLE_BYTES 1024 /* size of an exported peer handle */
#define DSP_MAX_LAYER_SIZE 8192 /* layer-wise: nodes sampled per layer (Table 7 uses 1000) */
#define DSP_MAX_CHANNELS 8   /* node-wise exchange channels (collective calls in flight per rank) */

typedef enum {
  DSP_OK = 0,
  DSP_ERR_INVALID_ARG = -1,   /* bad scalar / null pointer / bad layout      */
  DSP_ERR_OUT_OF_RANGE = -2,  /* a node id outside [0, N)                    */
  DSP_ERR_DUPLICATE_SEED = -3,/* a seed appears twice in one rank's batch    */
  DSP_ERR_CAPACITY = -4,      /* a buffer or workspace is too small          */
  DSP_ERR_STATE = -5,         /* call out of order / ranks disagree          */
  DSP_ERR_CUDA = -6,          /* a CUDA runtime call failed                  */
  DSP_ERR_PEER = -7,          /* peer mapping (CUDA IPC / P2P) failed        */
  DSP_ERR_OOM = -8            /* device allocation failed                    */
} dsp_status;

typedef struct dsp_ctx dsp_ctx; /* opaque; one host thread at a time */

/* ABI version (DSP_ABI_VERSION). */
int dsp_abi_version(void);
/* Static string for a status code. */
const char *dsp_status_str(int status);
/* Detail of the last failure on ctx (owned by ctx, valid until its next call);
   "" when none.  ctx may be NULL (then: last failure of dsp_create). */
const char *dsp_last_error(const dsp_ctx *ctx);

/* ------------------------------------------------------------ lifecycle */

/* Creates a ctx for `rank` of `world_size` (1..DSP_MAX_WORLD) on CUDA device
   `cuda_device`.  Several ctxs may share a device (virtual ranks driven by
   dsp_sample_group).  *out is set on success. */
dsp_status dsp_create(int32_t rank, int32_t world_size, int32_t cuda_device, dsp_ctx **out);

/* Frees everything the library owns (shards, exchange buffers, peer
   mappings).  COLLECTIVE in effect: peers must have stopped using this ctx's
   memory (barrier first).  NULL is a no-op. */
void dsp_destroy(dsp_ctx *ctx);

/* ------------------------------------------------------------ partition */

/* Loads this rank's partition.  Once per ctx.
   bounds  : HOST int64[world_size + 1]; bounds[0] = 0, non-decreasing,
             bounds[world_size] = N with N < 2^31; identical on all ranks.
   indptr  : host or device int64[n_r + 1], n_r = bounds[rank+1] - bounds[rank],
             indptr[0] = 0, non-decreasing.
   indices : host or device int32[indptr[n_r]]: GLOBAL ids of the
             in-neighbours of local row v (global id bounds[rank] + v), each
             row strictly ascending (R9); an id outside [0, N)
             fails the load with DSP_ERR_OUT_OF_RANGE.
   features: host or device fp32[n_r][dim] row-major, or NULL for none.
   dim     : 4 <= dim <= 4096 and dim % 4 == 0 (16-byte rows); ignored when
             features is NULL.
   The library copies everything into its own device memory (the feature
   shard into peer-mappable memory); the caller may free its buffers on
   return. */
dsp_status dsp_load_partition(dsp_ctx *ctx, const int64_t *bounds, const int64_t *indptr,
                              const int32_t *indices, const float *features, int32_t dim);

/* Feature shard with a cold tier ("we cache as many hot nodes as
   possible in GPU memory and store the other nodes (called cold nodes) in CPU
   memory and access them using the UVA technique.  DSP uses large indegrees to
   select hot nodes by default"; P:L224 feature position list).  Use instead of
   passing features to dsp_load_partition (features = NULL there).
   features: host or device fp32[n_r][dim]; hot_rows: rows kept in HBM (the
   hot_rows largest in-degrees of this rank, ties by id; < 0 or > n_r = all);
   the others go to pinned host memory (POSIX shm when world_size > 1, so that
   peers' GPUs can read them too) and are read over UVA by whichever GPU
   gathers them.  Gather results are bit-identical for any hot_rows.  Once per
   ctx, after dsp_load_partition and before dsp_reserve / handle export; all
   ranks must agree on using the tier. */
dsp_status dsp_load_features_tiered(dsp_ctx *ctx, const float *features, int32_t dim, int64_t hot_rows);

/* Edge weights for biased sampling (Sec. 4.2: "each node u ... is
   associated with a non-negative weight w_u ... DSP stores node weight w_u
   along with edge e_{v,u}").  edge_weights: host or device fp32[nnz_r]
   aligned with this rank's `indices` (the weight of the edge's neighbour);
   each must be 0 or lie in [2^-16, 65536) and is used as the 16.16
   fixed-point integer floor(w * 65536) (R24).  A negative, NaN or
   too large weight, or a positive one below 2^-16 (it would quantize to 0
   and never be drawn), fails the load with DSP_ERR_INVALID_ARG; rescale the
   weights of such a graph first (the draw probabilities depend only on the
   ratios).  Once per ctx,
   after dsp_load_partition.  Copied; the caller may free its buffer. */
dsp_status dsp_load_weights(dsp_ctx *ctx, const float *edge_weights);

/* Sizes the library's peer-visible exchange buffers for batches of up to
   max_seeds seeds per rank and the given fan-outs (fanouts: HOST
   int32[num_layers], 1 <= fanouts[l] <= 32, 1 <= num_layers <= 8).
   COLLECTIVE (identical arguments on every rank).  After dsp_load_partition. */
dsp_status dsp_reserve(dsp_ctx *ctx, int32_t max_seeds, const int32_t *fanouts, int32_t num_layers);

/* Layer-wise counterpart of dsp_reserve: sizes the peer-visible layer-wise
   exchange region for batches of up to max_seeds seeds and layer sizes
   sizes[num_layers] (HOST, each in [1, DSP_MAX_LAYER_SIZE]).  Needed for
   DSP_LAYERWISE at every world size; with or without dsp_reserve; before
   dsp_export_handle.  All ranks must pass the same values (checked at import). */
dsp_status dsp_reserve_layerwise(dsp_ctx *ctx, int32_t max_seeds, const int32_t *sizes, int32_t num_layers);

/* Peer handles (CUDA IPC for other processes, raw pointers within one
   process).  After dsp_reserve, every rank exports DSP_HANDLE_BYTES bytes;
   the caller all-gathers them (e.g. torch.distributed) into `all`
   (HOST, world_size * DSP_HANDLE_BYTES bytes, rank order) and imports them.
   Sampling and gather need the import when world_size > 1. */
dsp_status dsp_export_handle(const dsp_ctx *ctx, void *out);
dsp_status dsp_import_handles(dsp_ctx *ctx, const void *all);

/* ------------------------------------------------------------- sampling */

/* Flags.  DSP_BIASED (dsp_sample, dsp_sample_group, dsp_sample_gather):
   biased node-wise sampling with the weights of dsp_load_weights (
   Table 2 `IsBiased`): k successive draws without replacement, each
   neighbour with probability weight / total weight of the not-yet-drawn ones
   (R24-R26); ranks must agree (checked in the exchange header). */
#define DSP_ASYNC 1u
#define DSP_PIPELINED 2u
#define DSP_BIASED 4u
/* DSP_LAYERWISE (dsp_sample, dsp_sample_group, dsp_sample_gather): `fanouts`
   are LAYER SIZES n_l ("the total number of sampled nodes" per layer).
   Per layer, the requester reads each frontier node's degree W_u from its
   owner's indptr (peer memory), draws n_l times with replacement over its
   frontier with probability W_u / sum W (Eq. 2; Philox counter
   {j, seeds[0], l, "DSPL"}, R28-R30) and pushes (u, c_u) to the
   owner, which samples min(c_u, deg u) neighbours of u without replacement
   (the node-wise draws of layer l with fan-out c_u).  Blocks as node-wise
   (dst first, then new nodes in first-occurrence order); E_l <= n_l.
   Needs dsp_reserve_layerwise; not combinable with DSP_BIASED. */
#define DSP_LAYERWISE 8u

typedef struct {
  /* one sampled layer ("block"); arrays are DEVICE memory owned by the CALLER */
  int32_t *indptr;     int64_t cap_indptr; /* out [num_dst+1]: edge offsets per dst         */
  int32_t *indices;    int64_t cap_edges;  /* out [num_edges]: LOCAL src ids in [0,num_src) */
  int32_t *src_ids;    int64_t cap_src;    /* out [num_src]: global ids; [0,num_dst) = dst  */
  int32_t num_dst;     int32_t num_src;    /* out (host), filled on success                 */
  int64_t num_edges;                       /* out (host)                                    */
} dsp_block;

/* Capacities for a call: with F_0 = num_seeds (per-rank maximum), for each
   layer l: max_edges[l] = F_l * fanouts[l], max_src[l] = min(N, F_l +
   max_edges[l]), F_{l+1} = max_src[l].  *workspace_bytes: the device
   workspace dsp_sample needs.  max_src / max_edges: HOST int64[num_layers]
   (either may be NULL).  num_seeds must not exceed the reserved max_seeds. */
dsp_status dsp_sample_bounds(const dsp_ctx *ctx, int32_t num_seeds, const int32_t *fanouts,
                             int32_t num_layers, int64_t *max_src, int64_t *max_edges,
                             size_t *workspace_bytes);

/* Capacities of a DSP_LAYERWISE call: F_0 = num_seeds, max_edges[l] = n_l,
   max_src[l] = min(N, F_l + n_l), F_{l+1} = max_src[l]; workspace as above. */
dsp_status dsp_sample_bounds_layerwise(const dsp_ctx *ctx, int32_t num_seeds, const int32_t *sizes,
                                       int32_t num_layers, int64_t *max_src, int64_t *max_edges,
                                       size_t *workspace_bytes);

/* CSP node-wise uniform sampling without replacement (DESIGN.md
   R1-R17).  COLLECTIVE: every rank calls with identical fanouts, num_layers
   and rng_seed; seeds differ per rank (0 seeds allowed; the rank still takes
   part in every exchange).
   seeds    : DEVICE int32[num_seeds], unique (else DSP_ERR_DUPLICATE_SEED),
              each in [0, N) (else DSP_ERR_OUT_OF_RANGE); any owner.
   fanouts  : HOST int32[num_layers]; fanouts[l] applies at sampling layer l
              (l = 0 is the seeds' hop, R1).
   blocks   : HOST dsp_block[num_layers] in SAMPLING order; capacities must
              cover dsp_sample_bounds (else DSP_ERR_CAPACITY before any work).
              blocks[l].src_ids is the frontier of layer l+1; the last block's
              src_ids are the unique nodes whose features the loader needs.
   flags    : 0, DSP_BIASED or DSP_LAYERWISE (then fanouts = layer sizes).
   workspace: DEVICE, 256-byte aligned, >= workspace_bytes from
              dsp_sample_bounds, ZERO-FILLED before its first use; afterwards
              it belongs to the library (it carries the relabel map's epoch
              from call to call, so the map is never cleared): pass it back
              unmodified, or zero it again.  One workspace per ctx at a time.
   Stream-ordered on `stream`; returns after one stream synchronisation with
   the host-side sizes filled.  The result is a pure function of (graph,
   seeds, fanouts, rng_seed): bit-identical for any world_size / bounds and
   across runs.  On a device-detected error the call returns it and the
   block contents are unspecified. */
dsp_status dsp_sample(dsp_ctx *ctx, const int32_t *seeds, int32_t num_seeds, const int32_t *fanouts,
                      int32_t num_layers, uint64_t rng_seed, dsp_block *blocks, void *workspace,
                      size_t workspace_bytes, uint32_t flags, void *stream);

/* The same collective for n_ctx ctxs of one world driven by ONE host thread
   (virtual ranks sharing a device, or one process owning several GPUs).
   Array arguments are indexed by position in ctxs (any rank order, all ranks
   of the world present).  Node-wise calls run one persistent kernel per rank
   (the exchanges through peer memory inside it); ranks sharing a device each
   get 1/n of its SMs on the ctx's own stream, forked from and joined to the
   given stream after all ranks were launched (layer-wise calls likewise).
   Virtual ranks sharing a device must pass the same stream.  flags: 0,
   DSP_BIASED or DSP_LAYERWISE, plus DSP_ASYNC: return once every rank's call
   is enqueued (blocks[.][l].num_* not filled, device errors latch until
   dsp_sync); with DSP_OPT_EXCHANGE_CHANNELS = C and 1/(ranks per GPU * C)
   of the SMs per launch (dsp_set_persistent_blocks), C asynchronous group
   calls on C streams run concurrently. */
dsp_status dsp_sample_group(dsp_ctx *const *ctxs, int32_t n_ctx, const int32_t *const *seeds,
                            const int32_t *num_seeds, const int32_t *fanouts, int32_t num_layers,
                            uint64_t rng_seed, dsp_block *const *blocks, void *const *workspaces,
                            size_t workspace_bytes, uint32_t flags, void *const *streams);


/* One whole step of the hot path in ONE stream-ordered call: dsp_sample
   followed by the feature gather of the last block's src_ids (the loader
   right after the sampler), with no host round trip in between.
   The step runs as a single persistent kernel per rank (world_size == 1, or
   > 1 with the shuffle / reshuffle through NVLink peer memory inside it).
   Same arguments, rules and collectiveness as dsp_sample, plus:
   feat_out     : DEVICE fp32 [feat_cap_rows][dim], 16-byte aligned; rows
                  [0, blocks[L-1].num_src) receive the features of
                  blocks[L-1].src_ids, bit-exact.
   feat_cap_rows: >= max_src[L-1] of dsp_sample_bounds (else DSP_ERR_CAPACITY).
   sizes_out    : NULL, or int64[3 * num_layers] (HOST pinned or DEVICE)
                  receiving {num_dst, num_src, num_edges} per layer.
   flags        : 0 = synchronous: returns after one stream synchronisation
                  with blocks[l].num_* (and sizes_out) filled and device
                  errors reported.  DSP_ASYNC = returns once the step is
                  enqueued; blocks[l].num_* are NOT filled, sizes_out is
                  written when the stream reaches the end of the step, and
                  device errors latch until dsp_sync.  Consecutive async
                  steps may reuse the same workspace and outputs in stream
                  order (the producer/consumer pipeline of P:L198-200).
                  DSP_PIPELINED (implies DSP_ASYNC) = the loader of the
                  paper's pipeline runs one step behind the sampler
                  (P:L198-200): this call samples its seeds into `blocks`
                  while, in the same launch, it gathers the features owed by
                  the PREVIOUS pipelined call of this ctx on the same workspace into that call's
                  feat_out; this call's features are written by the next
                  pipelined call or by dsp_pipeline_flush.  The caller keeps
                  the previous call's blocks and feat_out alive until then
                  (e.g. two output sets used alternately, a queue of capacity
                  2).  A non-pipelined call flushes first. */
dsp_status dsp_sample_gather(dsp_ctx *ctx, const int32_t *seeds, int32_t num_seeds, const int32_t *fanouts,
                             int32_t num_layers, uint64_t rng_seed, dsp_block *blocks, float *feat_out,
                             int64_t feat_cap_rows, void *workspace, size_t workspace_bytes,
                             int64_t *sizes_out, uint32_t flags, void *stream);

/* Number of 1024-thread blocks of the world-1 persistent kernel (0 = the
   default, one per SM).  A smaller grid lets several steps run concurrently
   on different streams, each with its own workspace and outputs (e.g. two
   steps on half of the SMs each, so one step's latency-bound sampling phases
   overlap the other's bandwidth-bound gather).  Not collective. */
dsp_status dsp_set_persistent_blocks(dsp_ctx *ctx, int32_t blocks);

/* Performance options of a ctx (not collective).  None of them changes a
   result: blocks and gathered rows are bit-identical for every value (the
   GPU tests run the oracle parity under each).  Returns DSP_ERR_INVALID_ARG
   for an unknown option or a value outside its range.
   DSP_OPT_RELABEL_MAP     layout of the relabel map:
                           0 = by N (default: compact 4-byte direct map for
                           N <= 3M, else a batch-sized hash table), 1 = compact
                           direct map, 2 = hash table, 3 = 8-byte direct map.
                           Only before dsp_reserve / dsp_reserve_layerwise
                           (the workspace plan depends on it; DSP_ERR_STATE
                           afterwards); ranks may differ.
   DSP_OPT_LANE_ROUNDS     node-wise sampling with lane groups (G lanes per
                           node) while frontier * G <= value * sampling threads,
                           else a thread per node; 1..1024, default 8.
   DSP_OPT_LOADER_ROWS     rows per TMA gather chunk, 1..32 (default 32).
   DSP_OPT_GATHER_REGLOADS 0 (default) = standalone gathers and cold-tier rows
                           moved by TMA bulk copies; 1 = 16-byte register
                           loads.
   DSP_OPT_SPLIT_ROWS      feature-row layout in HBM: 0 (default) = rows packed
                           at dim * 4 bytes; 1 = each row split at its last
                           128-byte boundary into a head array of whole L2
                           lines and a small tail array kept L2-resident
                           (fewer DRAM bytes per random row: +3 % for a
                           standalone dsp_gather_features of 400-byte rows,
                           none for the pipelined step).  Before
                           dsp_load_partition; all ranks alike (checked at
                           import).
   DSP_OPT_EXCHANGE_CHANNELS  world_size > 1, node-wise: 1..DSP_MAX_CHANNELS
                           (default 1) exchange regions.  The n-th collective
                           node-wise call of a ctx (dsp_sample, dsp_sample_gather,
                           dsp_sample_group; synchronous or not) uses channel
                           n % channels, so that many calls can be in flight at
                           once on different streams (each with its own
                           workspace), the paper's pipeline with concurrent
                           samplers; calls of one channel run in
                           issue order (the library makes the stream of call n
                           wait for call n - channels).  Every rank issues its
                           calls in the same order (checked: the call count's
                           low byte travels in the exchange header, a mismatch
                           is DSP_ERR_STATE) and reserves the same number of
                           channels (checked at import); set before
                           dsp_reserve.  Concurrent calls must fit on the GPU
                           together: give each at most 1/channels of the SMs
                           with dsp_set_persistent_blocks. */
#define DSP_OPT_RELABEL_MAP 1
#define DSP_OPT_LANE_ROUNDS 2
#define DSP_OPT_LOADER_ROWS 4
#define DSP_OPT_GATHER_REGLOADS 5
#define DSP_OPT_EXCHANGE_CHANNELS 6
#define DSP_OPT_SPLIT_ROWS 7
dsp_status dsp_set_option(dsp_ctx *ctx, int32_t option, int64_t value);

/* Enqueues every gather still owed by this ctx's DSP_PIPELINED calls (one
   per workspace; no-op when none is pending) on `stream`.  A call made on
   another stream is waited for first (an event recorded on its stream), so
   work issued on `stream` afterwards sees every feat_out written, whichever
   stream the pipelined calls ran on. */
dsp_status dsp_pipeline_flush(dsp_ctx *ctx, void *stream);

/* --------------------------------------------------------------- gather */

/* Feature gather for the sampled nodes (P:L126 loader, hot features; P:L132:
   one-sided access over NVLink).  ONE-SIDED (not collective): rows owned by
   peers are read directly from their shards over NVLink, so it cannot
   deadlock against CSP.
   ids: DEVICE int32[n] global ids in [0, N); out: DEVICE fp32[n][dim],
   16-byte aligned, row-major.  out[r][c] = features of ids[r], bit-exact.
   Asynchronous on `stream`; an out-of-range id latches an error that
   dsp_sync reports (its row is left unwritten). */
dsp_status dsp_gather_features(dsp_ctx *ctx, const int32_t *ids, int64_t n, float *out, void *stream);

/* Random walks (Sec. 4.2: "a special case of node-wise sampling,
   whose fan-out is 1 for all layers"; R27).  Walk i starts at
   starts[i]; step l from node v takes the neighbour that fan-out-1 node-wise
   sampling picks for v at layer l with this rng_seed (walks meeting at a node
   at the same step continue together); a node without neighbours ends the
   walk and the remaining entries are -1.  NOTE: the draw is keyed by (node,
   step), not by the walk, so walks with the same start node in one call are
   IDENTICAL; for several independent walks per start node (DeepWalk-style)
   pass flags = DSP_WALK_INDEPENDENT: then step l of walk i draws from
   Philox counter {i, v, l, "DSPW"} (i = the walk's index in `starts`;
   DESIGN.md R35), so walks with the same start are independent.  flags: 0
   or DSP_WALK_INDEPENDENT (else DSP_ERR_INVALID_ARG); at world_size > 1
   all ranks pass the same flags (checked in the exchange header).
   starts: DEVICE int32[n] in [0, N) (any owner; else an error latches for
   dsp_sync and the walk is all -1); traces: DEVICE int32[n][length + 1],
   traces[i][0] = starts[i]; 1 <= length <= 1024.  Asynchronous on `stream`.
   world_size > 1: COLLECTIVE (every rank calls with the same length and
   rng_seed; n may differ, 0 allowed) and needs dsp_reserve_walks.  The walk
   follows CSP with the reshuffle removed: each step the walkers move
   to the owner of their node through its peer-mapped inbox (one exchange
   round: counts + header + flag), the owner takes the step and
   stores the new node straight into the trace row at the walk's origin rank
   over NVLink.  Traces are bit-identical for any world_size / bounds. */
#define DSP_WALK_INDEPENDENT 16u
dsp_status dsp_random_walk(dsp_ctx *ctx, const int32_t *starts, int64_t n, int32_t length, uint64_t rng_seed,
                           int32_t *traces, uint32_t flags, void *stream);

/* Sizes the peer-visible walk region for up to max_walks walks per rank
   (<= 2^27) of up to max_length steps (<= 1024): inboxes of
   world_size * max_walks walkers per (parity, sender) and the trace rows of
   this rank's walks.  All ranks pass the same values (checked at import);
   after dsp_load_partition, before dsp_export_handle.  Needed for
   dsp_random_walk with world_size > 1. */
dsp_status dsp_reserve_walks(dsp_ctx *ctx, int64_t max_walks, int32_t max_length);

/* dsp_random_walk for the n_ctx ranks of one world driven by ONE host thread
   (virtual ranks sharing a device must share a stream): stages are issued
   rank by rank.  Arrays are indexed by position in ctxs. */
dsp_status dsp_random_walk_group(dsp_ctx *const *ctxs, int32_t n_ctx, const int32_t *const *starts,
                                 const int64_t *n, int32_t length, uint64_t rng_seed, int32_t *const *traces,
                                 uint32_t flags, void *const *streams);

/* Synchronises `stream` and reports a latched device error (then clears it). */
dsp_status dsp_sync(dsp_ctx *ctx, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* DSP_H_ */
