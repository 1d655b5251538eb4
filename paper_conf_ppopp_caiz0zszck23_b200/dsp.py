"""Thin Python binding of libdsp.so (include/dsp.h), same names as the C ABI.

Argument marshalling only: every step of sampling and gathering runs in the
CUDA kernels behind the C ABI.  torch is used for device memory (workspace,
blocks, outputs), streams and -- for world_size > 1 across processes -- the
all-gather of the peer handles (torch.distributed plumbing).  There is no CPU
fallback: if libdsp.so is missing or no sm_100 GPU is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os
from typing import Callable, Sequence

import numpy as np

from . import _build

DSP_OK = 0
DSP_ERR_INVALID_ARG = -1
DSP_ERR_OUT_OF_RANGE = -2
DSP_ERR_DUPLICATE_SEED = -3
DSP_ERR_CAPACITY = -4
DSP_ERR_STATE = -5
DSP_ERR_CUDA = -6
DSP_ERR_PEER = -7
DSP_ERR_OOM = -8
DSP_MAX_WORLD = 8
DSP_MAX_LAYERS = 8
DSP_MAX_FANOUT = 32
DSP_HANDLE_BYTES = 1024
DSP_MAX_LAYER_SIZE = 8192

#: every symbol include/dsp.h declares
ABI_SYMBOLS = ("dsp_abi_version", "dsp_status_str", "dsp_last_error", "dsp_create", "dsp_destroy",
               "dsp_load_partition", "dsp_load_features_tiered", "dsp_load_weights", "dsp_reserve", "dsp_reserve_layerwise", "dsp_export_handle", "dsp_import_handles",
               "dsp_sample_bounds", "dsp_sample_bounds_layerwise", "dsp_sample", "dsp_sample_gather", "dsp_sample_group",
               "dsp_pipeline_flush", "dsp_set_persistent_blocks", "dsp_gather_features", "dsp_random_walk",
               "dsp_reserve_walks", "dsp_random_walk_group", "dsp_set_option",
               "dsp_sync")
DSP_ASYNC = 1
DSP_PIPELINED = 2
DSP_BIASED = 4
DSP_LAYERWISE = 8
DSP_WALK_INDEPENDENT = 16
DSP_OPT_RELABEL_MAP = 1
DSP_OPT_LANE_ROUNDS = 2
DSP_OPT_LOADER_ROWS = 4
DSP_OPT_GATHER_REGLOADS = 5
DSP_OPT_EXCHANGE_CHANNELS = 6
DSP_OPT_SPLIT_ROWS = 7
DSP_MAX_CHANNELS = 8
#: DSP_OPT_RELABEL_MAP values
RELABEL_MAPS = {"auto": 0, "direct": 1, "hash": 2, "direct64": 3}


class DSPError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"{_status_name(status)}: {detail}")


class dsp_block(ctypes.Structure):
    _fields_ = [("indptr", ctypes.c_void_p), ("cap_indptr", ctypes.c_int64),
                ("indices", ctypes.c_void_p), ("cap_edges", ctypes.c_int64),
                ("src_ids", ctypes.c_void_p), ("cap_src", ctypes.c_int64),
                ("num_dst", ctypes.c_int32), ("num_src", ctypes.c_int32),
                ("num_edges", ctypes.c_int64)]


_lib = None


def lib(path: str | None = None):
    """Loads libdsp.so from the package directory (never from a JIT cache)."""
    global _lib
    if _lib is None:
        # DSP_LIB: an alternative build of the same sources (tools/variants.py experiments)
        path = path or os.environ.get("DSP_LIB") or _build.LIB
        if not os.path.exists(path):
            raise RuntimeError(f"libdsp.so not built ({path}); run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        P, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        L.dsp_abi_version.restype = ctypes.c_int
        L.dsp_status_str.argtypes = [ctypes.c_int]
        L.dsp_status_str.restype = ctypes.c_char_p
        L.dsp_last_error.argtypes = [P]
        L.dsp_last_error.restype = ctypes.c_char_p
        L.dsp_create.argtypes = [i32, i32, i32, ctypes.POINTER(ctypes.c_void_p)]
        L.dsp_destroy.argtypes = [P]
        L.dsp_destroy.restype = None
        L.dsp_load_partition.argtypes = [P, P, P, P, P, i32]
        L.dsp_reserve.argtypes = [P, i32, P, i32]
        L.dsp_load_weights.argtypes = [P, P]
        L.dsp_load_features_tiered.argtypes = [P, P, i32, i64]
        L.dsp_reserve_layerwise.argtypes = [P, i32, P, i32]
        L.dsp_sample_bounds_layerwise.argtypes = [P, i32, P, i32, P, P, ctypes.POINTER(ctypes.c_size_t)]
        L.dsp_export_handle.argtypes = [P, P]
        L.dsp_import_handles.argtypes = [P, P]
        L.dsp_sample_bounds.argtypes = [P, i32, P, i32, P, P, ctypes.POINTER(ctypes.c_size_t)]
        L.dsp_sample.argtypes = [P, P, i32, P, i32, ctypes.c_uint64, P, P, ctypes.c_size_t, ctypes.c_uint32, P]
        L.dsp_sample_gather.argtypes = [P, P, i32, P, i32, ctypes.c_uint64, P, P, i64, P, ctypes.c_size_t, P,
                                         ctypes.c_uint32, P]
        L.dsp_sample_group.argtypes = [P, i32, P, P, P, i32, ctypes.c_uint64, P, P, ctypes.c_size_t,
                                        ctypes.c_uint32, P]
        L.dsp_gather_features.argtypes = [P, P, i64, P, P]
        L.dsp_pipeline_flush.argtypes = [P, P]
        L.dsp_set_persistent_blocks.argtypes = [P, i32]
        L.dsp_random_walk.argtypes = [P, P, i64, i32, ctypes.c_uint64, P, ctypes.c_uint32, P]
        L.dsp_reserve_walks.argtypes = [P, i64, i32]
        L.dsp_random_walk_group.argtypes = [P, i32, P, P, i32, ctypes.c_uint64, P, ctypes.c_uint32, P]
        L.dsp_sync.argtypes = [P, P]
        L.dsp_set_option.argtypes = [P, i32, i64]
        for name in ("dsp_create", "dsp_load_partition", "dsp_load_features_tiered", "dsp_load_weights", "dsp_reserve",
                     "dsp_reserve_layerwise", "dsp_sample_bounds_layerwise", "dsp_export_handle",
                     "dsp_import_handles", "dsp_sample_bounds", "dsp_sample", "dsp_sample_gather", "dsp_sample_group",
                     "dsp_pipeline_flush", "dsp_random_walk", "dsp_set_persistent_blocks",
                     "dsp_reserve_walks", "dsp_random_walk_group",
                     "dsp_gather_features", "dsp_sync", "dsp_set_option"):
            getattr(L, name).restype = ctypes.c_int
        _lib = L
    return _lib


def _status_name(s: int) -> str:
    try:
        return lib().dsp_status_str(s).decode()
    except Exception:  # library unavailable while formatting an error
        return f"status {s}"


def _check(status: int, ctx=None):
    if status != DSP_OK:
        detail = lib().dsp_last_error(ctx).decode() if True else ""
        raise DSPError(status, detail)


def _p(x) -> ctypes.c_void_p:
    """Raw pointer of a torch tensor, numpy array or int."""
    if x is None:
        return ctypes.c_void_p(0)
    if isinstance(x, int):
        return ctypes.c_void_p(x)
    if isinstance(x, np.ndarray):
        return x.ctypes.data_as(ctypes.c_void_p)
    return ctypes.c_void_p(x.data_ptr())


def _i32_array(xs) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(xs, dtype=np.int32))


# ------------------------------------------------------- C-ABI, same names

def dsp_abi_version() -> int:
    return int(lib().dsp_abi_version())


def dsp_status_str(status: int) -> str:
    return lib().dsp_status_str(status).decode()


def dsp_last_error(ctx) -> str:
    return lib().dsp_last_error(ctx).decode()


def dsp_create(rank: int, world_size: int, cuda_device: int) -> ctypes.c_void_p:
    out = ctypes.c_void_p()
    _check(lib().dsp_create(rank, world_size, cuda_device, ctypes.byref(out)), None)
    return out


def dsp_destroy(ctx) -> None:
    lib().dsp_destroy(ctx)


def dsp_load_partition(ctx, bounds, indptr, indices, features, dim: int) -> None:
    b = np.ascontiguousarray(bounds, dtype=np.int64)
    _check(lib().dsp_load_partition(ctx, _p(b), _p(indptr), _p(indices), _p(features), dim), ctx)


def dsp_load_features_tiered(ctx, features, dim: int, hot_rows: int) -> None:
    _check(lib().dsp_load_features_tiered(ctx, _p(features), dim, hot_rows), ctx)


def dsp_load_weights(ctx, edge_weights) -> None:
    _check(lib().dsp_load_weights(ctx, _p(edge_weights)), ctx)


def dsp_reserve(ctx, max_seeds: int, fanouts) -> None:
    f = _i32_array(fanouts)
    _check(lib().dsp_reserve(ctx, max_seeds, _p(f), len(f)), ctx)


def dsp_reserve_layerwise(ctx, max_seeds: int, sizes) -> None:
    f = _i32_array(sizes)
    _check(lib().dsp_reserve_layerwise(ctx, max_seeds, _p(f), len(f)), ctx)


def dsp_sample_bounds_layerwise(ctx, num_seeds: int, sizes):
    f = _i32_array(sizes)
    ms = np.zeros(len(f), np.int64)
    me = np.zeros(len(f), np.int64)
    ws = ctypes.c_size_t(0)
    _check(lib().dsp_sample_bounds_layerwise(ctx, num_seeds, _p(f), len(f), _p(ms), _p(me), ctypes.byref(ws)), ctx)
    return ms, me, ws.value


def dsp_export_handle(ctx) -> bytes:
    buf = ctypes.create_string_buffer(DSP_HANDLE_BYTES)
    _check(lib().dsp_export_handle(ctx, buf), ctx)
    return buf.raw


def dsp_import_handles(ctx, handles: Sequence[bytes]) -> None:
    blob = b"".join(handles)
    buf = ctypes.create_string_buffer(blob, len(blob))
    _check(lib().dsp_import_handles(ctx, buf), ctx)


def dsp_sample_bounds(ctx, num_seeds: int, fanouts):
    f = _i32_array(fanouts)
    ms = np.zeros(len(f), np.int64)
    me = np.zeros(len(f), np.int64)
    ws = ctypes.c_size_t()
    _check(lib().dsp_sample_bounds(ctx, num_seeds, _p(f), len(f), _p(ms), _p(me), ctypes.byref(ws)), ctx)
    return ms, me, int(ws.value)


def dsp_sample(ctx, seeds, num_seeds: int, fanouts, rng_seed: int, blocks, workspace,
               workspace_bytes: int, flags: int, stream: int) -> None:
    f = _i32_array(fanouts)
    _check(lib().dsp_sample(ctx, _p(seeds), num_seeds, _p(f), len(f), ctypes.c_uint64(rng_seed),
                            blocks, _p(workspace), workspace_bytes, flags, ctypes.c_void_p(stream)), ctx)


def dsp_sample_gather(ctx, seeds, num_seeds: int, fanouts, rng_seed: int, blocks, feat_out, feat_cap_rows: int,
                      workspace, workspace_bytes: int, sizes_out, flags: int, stream: int) -> None:
    f = _i32_array(fanouts)
    _check(lib().dsp_sample_gather(ctx, _p(seeds), num_seeds, _p(f), len(f), ctypes.c_uint64(rng_seed), blocks,
                                   _p(feat_out), feat_cap_rows, _p(workspace), workspace_bytes, _p(sizes_out),
                                   flags, ctypes.c_void_p(stream)), ctx)


def dsp_sample_group(ctxs, seeds, num_seeds, fanouts, rng_seed: int, blocks, workspaces,
                     workspace_bytes: int, flags: int, streams) -> None:
    n = len(ctxs)
    f = _i32_array(fanouts)
    c_ctxs = (ctypes.c_void_p * n)(*[c.value for c in ctxs])
    c_seeds = (ctypes.c_void_p * n)(*[_p(s).value for s in seeds])
    c_ns = (ctypes.c_int32 * n)(*num_seeds)
    c_blocks = (ctypes.c_void_p * n)(*[ctypes.cast(b, ctypes.c_void_p).value for b in blocks])
    c_ws = (ctypes.c_void_p * n)(*[_p(w).value for w in workspaces])
    c_st = (ctypes.c_void_p * n)(*streams)
    _check(lib().dsp_sample_group(c_ctxs, n, c_seeds, c_ns, _p(f), len(f), ctypes.c_uint64(rng_seed),
                                  c_blocks, c_ws, workspace_bytes, flags, c_st), ctxs[0])


def dsp_pipeline_flush(ctx, stream: int) -> None:
    _check(lib().dsp_pipeline_flush(ctx, ctypes.c_void_p(stream)), ctx)


def dsp_gather_features(ctx, ids, n: int, out, stream: int) -> None:
    _check(lib().dsp_gather_features(ctx, _p(ids), n, _p(out), ctypes.c_void_p(stream)), ctx)


def dsp_set_option(ctx, option: int, value: int) -> None:
    _check(lib().dsp_set_option(ctx, option, value), ctx)


def dsp_set_persistent_blocks(ctx, blocks: int) -> None:
    _check(lib().dsp_set_persistent_blocks(ctx, blocks), ctx)


def dsp_random_walk(ctx, starts, n: int, length: int, rng_seed: int, traces, stream: int, flags: int = 0) -> None:
    _check(lib().dsp_random_walk(ctx, _p(starts), n, length, ctypes.c_uint64(rng_seed), _p(traces), flags,
                                 ctypes.c_void_p(stream)), ctx)


def dsp_reserve_walks(ctx, max_walks: int, max_length: int) -> None:
    _check(lib().dsp_reserve_walks(ctx, max_walks, max_length), ctx)


def dsp_random_walk_group(ctxs, starts, n, length: int, rng_seed: int, traces, streams, flags: int = 0) -> None:
    k = len(ctxs)
    c_ctxs = (ctypes.c_void_p * k)(*[c.value if isinstance(c, ctypes.c_void_p) else c for c in ctxs])
    c_starts = (ctypes.c_void_p * k)(*[x.data_ptr() for x in starts])
    c_n = (ctypes.c_int64 * k)(*[int(x) for x in n])
    c_tr = (ctypes.c_void_p * k)(*[x.data_ptr() for x in traces])
    c_st = (ctypes.c_void_p * k)(*streams)
    _check(lib().dsp_random_walk_group(c_ctxs, k, c_starts, c_n, length, ctypes.c_uint64(rng_seed), c_tr, flags,
                                       c_st), ctxs[0])


def dsp_sync(ctx, stream: int) -> None:
    _check(lib().dsp_sync(ctx, ctypes.c_void_p(stream)), ctx)


# ------------------------------------------------------------ conveniences

class Block:
    """One sampled layer: its sizes, and views of the Sampler's device buffers
    (torch.int32 `indptr` [num_dst + 1], `indices` [num_edges] local src ids,
    `src_ids` [num_src] global ids) made on first access, so a caller that only
    needs the sizes pays no tensor slicing per step."""
    __slots__ = ("num_dst", "num_src", "num_edges", "_bufs", "_views")

    def __init__(self, num_dst: int, num_src: int, num_edges: int, bufs):
        self.num_dst, self.num_src, self.num_edges = num_dst, num_src, num_edges
        self._bufs = bufs
        self._views = None

    def _view(self, j):
        if self._views is None:
            ip, ix, sr = self._bufs
            self._views = (ip[: self.num_dst + 1], ix[: self.num_edges], sr[: self.num_src])
        return self._views[j]

    indptr = property(lambda self: self._view(0))
    indices = property(lambda self: self._view(1))
    src_ids = property(lambda self: self._view(2))

    def __repr__(self):
        return f"Block(num_dst={self.num_dst}, num_src={self.num_src}, num_edges={self.num_edges})"


class Sampler:
    """One rank of a CSP world: ctx + partition + caller-owned buffers.

    ``exchange(blob) -> list[bytes]`` all-gathers the peer handles when
    world_size > 1 (see :func:`torch_exchange`)."""

    def __init__(self, bounds, indptr, indices, features, fanouts, max_seeds: int, rank: int = 0,
                 world_size: int = 1, device: int | None = None,
                 exchange: Callable[[bytes], list] | None = None, connect: bool = True, n_slots: int = 1,
                 edge_weights=None, n_workspaces: int = 1, hot_rows: int | None = None, scheme: str = "node",
                 max_walks: int | None = None, max_walk_length: int = 1024, options: dict | None = None):
        """max_walks: reserve the random-walk region (needed for random_walk when
        world_size > 1) for up to max_walks walks per rank of max_walk_length steps.
        options: {DSP_OPT_*: value} applied with dsp_set_option right after
        dsp_create (performance only; results are identical)."""
        import torch
        self.torch = torch
        self.device = torch.cuda.current_device() if device is None else device
        self.rank, self.world = rank, world_size
        assert scheme in ("node", "layer")
        self.scheme = scheme          # "layer": fanouts are layer sizes (DSP_LAYERWISE)
        self._sflag = DSP_LAYERWISE if scheme == "layer" else 0
        self.fanouts = [int(k) for k in fanouts]
        self.max_seeds = int(max_seeds)
        self.dim = 0 if features is None else int(features.shape[1])
        self.ctx = dsp_create(rank, world_size, self.device)
        try:
            for opt, val in (options or {}).items():
                dsp_set_option(self.ctx, int(opt), int(val))
            if hot_rows is None:
                dsp_load_partition(self.ctx, bounds, indptr, indices, features, self.dim)
            else:  # cold-feature tier: hot_rows rows in HBM, the rest in host memory
                dsp_load_partition(self.ctx, bounds, indptr, indices, None, 0)
                dsp_load_features_tiered(self.ctx, features, self.dim, hot_rows)
            if edge_weights is not None:
                dsp_load_weights(self.ctx, np.ascontiguousarray(edge_weights, np.float32)
                                 if isinstance(edge_weights, np.ndarray) else edge_weights)
            if scheme == "layer":
                dsp_reserve_layerwise(self.ctx, self.max_seeds, self.fanouts)
                ms, me, ws = dsp_sample_bounds_layerwise(self.ctx, self.max_seeds, self.fanouts)
            else:
                dsp_reserve(self.ctx, self.max_seeds, self.fanouts)
                ms, me, ws = dsp_sample_bounds(self.ctx, self.max_seeds, self.fanouts)
            if max_walks is not None:
                dsp_reserve_walks(self.ctx, int(max_walks), int(max_walk_length))
        except Exception:
            dsp_destroy(self.ctx)
            self.ctx = None
            raise
        dev = torch.device("cuda", self.device)
        self.workspace_bytes = ws
        # zero-filled before first use; several workspaces let steps run concurrently on several streams
        self.workspaces = [torch.zeros(ws, dtype=torch.uint8, device=dev) for _ in range(max(1, n_workspaces))]
        self.workspace = self.workspaces[0]
        F = [self.max_seeds] + [int(x) for x in ms[:-1]]
        self._sets = []
        for _ in range(max(1, n_slots)):   # output sets (a queue of capacity n_slots)
            bufs = []
            cblocks = (dsp_block * len(self.fanouts))()
            for l in range(len(self.fanouts)):
                ip = torch.empty(F[l] + 1, dtype=torch.int32, device=dev)
                ix = torch.empty(max(1, int(me[l])), dtype=torch.int32, device=dev)
                sr = torch.empty(max(1, int(ms[l])), dtype=torch.int32, device=dev)
                bufs.append((ip, ix, sr))
                b = cblocks[l]
                b.indptr, b.cap_indptr = ip.data_ptr(), ip.numel()
                b.indices, b.cap_edges = ix.data_ptr(), int(me[l])
                b.src_ids, b.cap_src = sr.data_ptr(), int(ms[l])
            self._sets.append([bufs, cblocks, None])
        self._bufs, self._cblocks = self._sets[0][0], self._sets[0][1]
        self.max_src = [int(x) for x in ms]
        self.max_edges = [int(x) for x in me]
        self.connected = False
        if connect and (world_size == 1 or exchange is not None):
            handles = [dsp_export_handle(self.ctx)] if world_size == 1 else exchange(dsp_export_handle(self.ctx))
            if world_size > 1:
                dsp_import_handles(self.ctx, handles)
            self.connected = True

    def stream(self) -> int:
        return self.torch.cuda.current_stream(self.device).cuda_stream

    def sample(self, seeds, rng_seed: int, biased: bool = False) -> list[Block]:
        torch = self.torch
        assert seeds.dtype == torch.int32 and seeds.is_cuda and seeds.is_contiguous()
        dsp_sample(self.ctx, seeds, seeds.numel(), self.fanouts, rng_seed, self._cblocks, self.workspace,
                   self.workspace_bytes, (DSP_BIASED if biased else 0) | self._sflag, self.stream())
        return self.blocks()

    def sample_gather(self, seeds, rng_seed: int, slot: int = 0, sizes_out=None, async_: bool = False,
                      pipelined: bool = False, biased: bool = False, ws: int = 0, stream=None):
        """One whole step (sample + gather) in one call into output set `slot`.
        Synchronous: returns (blocks, features view).  async_: returns None;
        sizes land in sizes_out (pinned host / device int64[3L]) in stream order.
        pipelined: the features of this step are written by the next pipelined
        step (or flush()), which gathers them while it samples."""
        torch = self.torch
        assert seeds.dtype == torch.int32 and seeds.is_cuda and seeds.is_contiguous()
        feat_out = self.feat_buffer(slot)
        flags = ((DSP_PIPELINED if pipelined else (DSP_ASYNC if async_ else 0)) | (DSP_BIASED if biased else 0)
                 | self._sflag)
        dsp_sample_gather(self.ctx, seeds, seeds.numel(), self.fanouts, rng_seed, self._sets[slot][1], feat_out,
                          feat_out.shape[0], self.workspaces[ws], self.workspace_bytes, sizes_out, flags,
                          self.stream() if stream is None else stream.cuda_stream)
        if async_ or pipelined:
            return None
        blocks = self.blocks(slot)
        return blocks, feat_out[: blocks[-1].num_src]

    def feat_buffer(self, slot: int = 0):
        if self._sets[slot][2] is None:
            self._sets[slot][2] = self.torch.empty((self.max_src[-1], self.dim), dtype=self.torch.float32,
                                                   device=self.torch.device("cuda", self.device))
        return self._sets[slot][2]

    def blocks(self, slot: int = 0, sizes=None) -> list[Block]:
        """Views of output set `slot`; sizes from the last synchronous call, or
        from an int64[3L] array filled by an async call."""
        bufs, cblocks, _ = self._sets[slot]
        out = []
        for l, (ip, ix, sr) in enumerate(bufs):
            if sizes is None:
                b = cblocks[l]
                nd, ns, ne = b.num_dst, b.num_src, b.num_edges
            else:
                nd, ns, ne = (int(x) for x in sizes[3 * l: 3 * l + 3])
            out.append(Block(nd, ns, ne, (ip, ix, sr)))
        return out

    def gather(self, ids, out=None):
        torch = self.torch
        n = ids.numel()
        if out is None:
            out = torch.empty((n, self.dim), dtype=torch.float32, device=ids.device)
        dsp_gather_features(self.ctx, ids, n, out, self.stream())
        return out

    def random_walk(self, starts, length: int, rng_seed: int, out=None, independent: bool = False):
        """Walk traces int32[n][length + 1], asynchronous on the stream
        (into `out` when given: a caller-owned int32[n][length + 1] buffer).
        independent: DSP_WALK_INDEPENDENT (walks from one start differ, R35)."""
        torch = self.torch
        assert starts.dtype == torch.int32 and starts.is_cuda and starts.is_contiguous()
        if out is None:
            out = torch.empty((starts.numel(), length + 1), dtype=torch.int32, device=starts.device)
        assert out.dtype == torch.int32 and out.is_cuda and out.is_contiguous() and out.shape == (starts.numel(), length + 1)
        dsp_random_walk(self.ctx, starts, starts.numel(), length, rng_seed, out, self.stream(),
                        DSP_WALK_INDEPENDENT if independent else 0)
        return out

    def sync(self) -> None:
        dsp_sync(self.ctx, self.stream())

    def flush(self) -> None:
        dsp_pipeline_flush(self.ctx, self.stream())

    def close(self) -> None:
        if getattr(self, "ctx", None) is not None:
            dsp_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def torch_exchange(group=None) -> Callable[[bytes], list]:
    """all-gather of the peer handles over torch.distributed (plumbing)."""
    import torch.distributed as dist

    def ex(blob: bytes) -> list:
        out = [None] * dist.get_world_size(group)
        dist.all_gather_object(out, blob, group=group)
        return out
    return ex


class LocalGroup:
    """All ranks of a world in one process, driven by one host thread through
    dsp_sample_group.  Ranks may share a device (virtual ranks: stages are
    issued rank by rank on the device's current stream) or sit on several
    GPUs of this node."""

    def __init__(self, bounds, shards, fanouts, max_seeds: int, devices: Sequence[int], hot_rows=None,
                 scheme: str = "node", max_walks: int | None = None, max_walk_length: int = 1024,
                 options: dict | None = None, n_workspaces: int = 1, n_slots: int = 1):
        """shards[r] = (indptr, indices, features[, edge_weights]) of rank r;
        hot_rows[r] (optional) enables the cold-feature tier; options as Sampler."""
        P = len(shards)
        assert len(devices) == P and len(bounds) == P + 1
        self.samplers = [Sampler(bounds, s[0], s[1], s[2], fanouts, max_seeds, rank=r, world_size=P,
                                 device=devices[r], connect=False, edge_weights=s[3] if len(s) > 3 else None,
                                 hot_rows=None if hot_rows is None else hot_rows[r], scheme=scheme,
                                 max_walks=max_walks, max_walk_length=max_walk_length, options=options,
                                 n_workspaces=n_workspaces, n_slots=n_slots)
                         for r, s in enumerate(shards)]
        handles = [dsp_export_handle(s.ctx) for s in self.samplers]
        for s in self.samplers:
            if P > 1:
                dsp_import_handles(s.ctx, handles)
            s.connected = True
        self.fanouts = list(fanouts)

    def sample(self, seeds_per_rank, rng_seed: int, biased: bool = False, async_: bool = False, ws: int = 0,
               slot: int = 0, stream=None) -> list[list[Block]] | None:
        """One group call (every rank).  async_: enqueue only (DSP_ASYNC) on
        `stream`, with workspace `ws` and output set `slot` of every rank;
        returns None (sizes via a later synchronous call or the blocks' data)."""
        S = self.samplers
        st = [s.stream() for s in S] if stream is None else [stream.cuda_stream] * len(S)
        dsp_sample_group([s.ctx for s in S], seeds_per_rank, [x.numel() for x in seeds_per_rank],
                         self.fanouts, rng_seed, [s._sets[slot][1] for s in S], [s.workspaces[ws] for s in S],
                         S[0].workspace_bytes, (DSP_BIASED if biased else 0) | S[0]._sflag
                         | (DSP_ASYNC if async_ else 0), st)
        return None if async_ else [s.blocks(slot) for s in S]

    def random_walk(self, starts_per_rank, length: int, rng_seed: int, independent: bool = False):
        """Walk traces of every rank, CSP push without reshuffle."""
        torch = self.samplers[0].torch
        S = self.samplers
        outs = [torch.empty((x.numel(), length + 1), dtype=torch.int32, device=x.device) for x in starts_per_rank]
        dsp_random_walk_group([s.ctx for s in S], starts_per_rank, [x.numel() for x in starts_per_rank], length,
                              rng_seed, outs, [s.stream() for s in S], DSP_WALK_INDEPENDENT if independent else 0)
        return outs

    def close(self):
        for s in self.samplers:
            s.close()
