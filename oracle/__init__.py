"""CPU oracle for CSP sampling + feature gather -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_ppopp_caiz0zszck23_b200``) never imports it and shares no code
with it.  This module is argument marshalling over ``liboracle.so`` (built from
``oracle/oracle.c``, whose header cites the PAPER.md passages each function
follows).

Parity status: every function here is pinned by ``tests/test_oracle_*.py``
(Random123 known-answer vectors, exhaustive Floyd enumeration, chi-square
uniformity, invariants, the full-row special case against scipy.sparse, the
paper's Fig. 3 / Fig. 5 worked examples, CSP-replay invariance).  No function
is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK = 0
ERR_INVALID_ARG = -1
ERR_OUT_OF_RANGE = -2
ERR_DUPLICATE_SEED = -3
ERR_OOM = -8


class OracleError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: oracle status {code}")
        self.code = code


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain -O2, single thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-Wall", "-Wextra",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _Block(ctypes.Structure):
    _fields_ = [("num_dst", ctypes.c_int32), ("num_src", ctypes.c_int32),
                ("num_edges", ctypes.c_int64),
                ("indptr", ctypes.POINTER(ctypes.c_int32)),
                ("indices", ctypes.POINTER(ctypes.c_int32)),
                ("src_ids", ctypes.POINTER(ctypes.c_int32))]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P = ctypes.c_void_p
        L.oracle_philox4x32_10.argtypes = [P, P, P]
        L.oracle_draw_word.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_int32]
        L.oracle_draw_word.restype = ctypes.c_uint64
        L.oracle_mulhi_range.argtypes = [ctypes.c_uint64, ctypes.c_uint32]
        L.oracle_mulhi_range.restype = ctypes.c_uint32
        L.oracle_draw.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_int32,
                                  ctypes.c_uint32]
        L.oracle_draw.restype = ctypes.c_uint32
        L.oracle_floyd.argtypes = [ctypes.c_int64, ctypes.c_int32, P, P]
        L.oracle_node_positions.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32,
                                            ctypes.c_int64, ctypes.c_int32, P]
        L.oracle_node_positions.restype = ctypes.c_int32
        L.oracle_sample_rows.argtypes = [ctypes.c_int64, P, P, ctypes.c_int64, P, ctypes.c_int64,
                                         ctypes.c_int32, ctypes.c_int32, ctypes.c_uint64, P, P]
        L.oracle_build_block.argtypes = [ctypes.c_int64, P, ctypes.c_int32, P, P, ctypes.c_int32, P,
                                         ctypes.POINTER(_Block)]
        L.oracle_sample.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, ctypes.c_int32,
                                    ctypes.c_uint64, ctypes.POINTER(_Block)]
        L.oracle_free_block.argtypes = [ctypes.POINTER(_Block)]
        L.oracle_gather.argtypes = [ctypes.c_int64, ctypes.c_int32, P, P, ctypes.c_int64, P]
        L.oracle_weight_fixed.argtypes = [ctypes.c_float]
        L.oracle_weight_fixed.restype = ctypes.c_uint32
        L.oracle_biased_picks.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32, P, ctypes.c_int64,
                                          ctypes.c_int32, P]
        L.oracle_biased_picks.restype = ctypes.c_int32
        L.oracle_node_positions_biased.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32, P,
                                                   ctypes.c_int64, ctypes.c_int32, P]
        L.oracle_node_positions_biased.restype = ctypes.c_int32
        L.oracle_sample_rows_ex.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int64, P, ctypes.c_int64,
                                            ctypes.c_int32, ctypes.c_int32, ctypes.c_uint64, P, P]
        L.oracle_sample_ex.argtypes = [ctypes.c_int64, P, P, P, P, ctypes.c_int32, P, ctypes.c_int32,
                                       ctypes.c_uint64, ctypes.POINTER(_Block)]
        L.oracle_draw_word_tag.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, ctypes.c_int32,
                                           ctypes.c_uint32]
        L.oracle_draw_word_tag.restype = ctypes.c_uint64
        L.oracle_layer_alloc.argtypes = [ctypes.c_uint64, ctypes.c_int32, ctypes.c_int32, P, ctypes.c_int32,
                                         ctypes.c_int32, P]
        L.oracle_sample_layerwise.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int32, P, ctypes.c_int32,
                                              ctypes.c_uint64, ctypes.POINTER(_Block)]
        L.oracle_random_walk.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, P]
        L.oracle_random_walk_independent.argtypes = [ctypes.c_int64, P, P, P, ctypes.c_int64, ctypes.c_int32,
                                                     ctypes.c_uint64, P]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


# ------------------------------------------------------------------ RNG

def philox4x32_10(ctr, key) -> np.ndarray:
    c = _c(ctr, np.uint32)
    k = _c(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().oracle_philox4x32_10(_ptr(c), _ptr(k), _ptr(out))
    return out


def draw_word(rng_seed: int, slot: int, v: int, l: int) -> int:
    return int(lib().oracle_draw_word(rng_seed, slot, v, l))


def mulhi_range(x: int, m: int) -> int:
    return int(lib().oracle_mulhi_range(x, m))


def draw(rng_seed: int, slot: int, v: int, l: int, m: int) -> int:
    return int(lib().oracle_draw(rng_seed, slot, v, l, m))


def floyd(d: int, k: int, draws) -> np.ndarray:
    r = _c(draws, np.uint32)
    assert r.shape == (k,)
    out = np.zeros(k, np.int64)
    lib().oracle_floyd(d, k, _ptr(r), _ptr(out))
    return out


def node_positions(rng_seed: int, v: int, l: int, d: int, k: int) -> np.ndarray:
    out = np.zeros(max(32, k), np.int64)
    c = lib().oracle_node_positions(rng_seed, v, l, d, k, _ptr(out))
    return out[:c].copy()


# ------------------------------------------------------------- sampling

def weight_fixed(w: float) -> int:
    """Fixed-point edge weight floor(w * 2^16) (0xffffffff = invalid)."""
    return int(lib().oracle_weight_fixed(w))


def biased_picks(rng_seed: int, v: int, l: int, a, k: int) -> np.ndarray:
    """Successive weighted picks (draw order) over integer weights ``a``."""
    a = _c(a, np.uint32)
    out = np.zeros(max(32, k), np.int64)
    c = lib().oracle_biased_picks(rng_seed, v, l, _ptr(a), len(a), k, _ptr(out))
    return out[:c].copy()


def node_positions_biased(rng_seed: int, v: int, l: int, a, k: int) -> np.ndarray:
    a = _c(a, np.uint32)
    out = np.zeros(max(32, k), np.int64)
    c = lib().oracle_node_positions_biased(rng_seed, v, l, _ptr(a), len(a), k, _ptr(out))
    return out[:c].copy()


def sample_rows(indptr, indices, ids, k: int, l: int, rng_seed: int, id_offset: int = 0, weights=None):
    """Owner-side sampling stage for global ``ids`` over a CSR (shard);
    ``weights`` = fp32 per edge (biased sampling) or None (uniform)."""
    ip = _c(indptr, np.int64)
    ix = _c(indices, np.int32)
    ids = _c(ids, np.int32)
    w = None if weights is None else _c(weights, np.float32)
    cnt = np.zeros(len(ids), np.int32)
    rows = np.zeros(len(ids) * k, np.int32)
    rc = lib().oracle_sample_rows_ex(len(ip) - 1, _ptr(ip), _ptr(ix), None if w is None else _ptr(w), id_offset,
                                     _ptr(ids), len(ids), k, l, rng_seed, _ptr(cnt), _ptr(rows))
    if rc != OK:
        raise OracleError(rc, "oracle_sample_rows")
    return cnt, rows.reshape(len(ids), k)


def _block_to_numpy(b: _Block) -> dict:
    F, S, E = b.num_dst, b.num_src, b.num_edges
    return {
        "num_dst": F, "num_src": S, "num_edges": E,
        "indptr": np.ctypeslib.as_array(b.indptr, shape=(F + 1,)).copy(),
        "indices": (np.ctypeslib.as_array(b.indices, shape=(E,)).copy() if E else np.zeros(0, np.int32)),
        "src_ids": (np.ctypeslib.as_array(b.src_ids, shape=(S,)).copy() if S else np.zeros(0, np.int32)),
    }


def build_block(N: int, frontier, cnt, rows) -> dict:
    """Requester-side block construction (dedup + relabel) from sampled rows."""
    fr = _c(frontier, np.int32)
    cnt = _c(cnt, np.int32)
    rows = np.ascontiguousarray(rows, dtype=np.int32)
    k = rows.shape[1] if rows.ndim == 2 else 1
    loc = np.full(max(N, 1), -1, np.int32)
    b = _Block()
    rc = lib().oracle_build_block(N, _ptr(fr), len(fr), _ptr(cnt), _ptr(rows), k, _ptr(loc),
                                  ctypes.byref(b))
    if rc != OK:
        raise OracleError(rc, "oracle_build_block")
    out = _block_to_numpy(b)
    lib().oracle_free_block(ctypes.byref(b))
    return out


def sample(indptr, indices, seeds, fanouts, rng_seed: int, weights=None) -> list[dict]:
    """Multi-layer node-wise sampling for one rank's seeds on the whole graph
    (biased when ``weights``, fp32 per edge, is given)."""
    ip = _c(indptr, np.int64)
    ix = _c(indices, np.int32)
    sd = _c(seeds, np.int32)
    fo = _c(fanouts, np.int32)
    w = None if weights is None else _c(weights, np.float32)
    L = len(fo)
    blocks = (_Block * max(L, 1))()
    rc = lib().oracle_sample_ex(len(ip) - 1, _ptr(ip), _ptr(ix), None if w is None else _ptr(w), _ptr(sd),
                                len(sd), _ptr(fo), L, rng_seed, blocks)
    if rc != OK:
        raise OracleError(rc, "oracle_sample")
    out = [_block_to_numpy(blocks[l]) for l in range(L)]
    for l in range(L):
        lib().oracle_free_block(ctypes.byref(blocks[l]))
    return out


def draw_word_tag(rng_seed: int, slot: int, v: int, l: int, tag: int) -> int:
    """x1:x0 of Philox({slot, v, l, tag}, seed)."""
    return int(lib().oracle_draw_word_tag(rng_seed, slot, v, l, tag))


def layer_alloc(rng_seed: int, g0: int, l: int, W, n: int) -> np.ndarray:
    """Eq. 2 allocation: draw counts c[i] of n draws with
    replacement over the frontier with probability W_i / sum W."""
    w = _c(W, np.uint64)
    c = np.zeros(max(1, len(w)), np.int32)
    rc = lib().oracle_layer_alloc(rng_seed, g0, l, _ptr(w), len(w), n, _ptr(c))
    if rc != OK:
        raise OracleError(rc, "oracle_layer_alloc")
    return c[:len(w)].copy()


def sample_layerwise(indptr, indices, seeds, sizes, rng_seed: int) -> list[dict]:
    """Multi-layer layer-wise sampling (Eq. 2 allocation + node-wise sampling
    of c_u neighbours without replacement) for one rank's seeds."""
    ip = _c(indptr, np.int64)
    ix = _c(indices, np.int32)
    sd = _c(seeds, np.int32)
    sz = _c(sizes, np.int32)
    L = len(sz)
    blocks = (_Block * max(L, 1))()
    rc = lib().oracle_sample_layerwise(len(ip) - 1, _ptr(ip), _ptr(ix), _ptr(sd), len(sd), _ptr(sz), L,
                                       rng_seed, blocks)
    if rc != OK:
        raise OracleError(rc, "oracle_sample_layerwise")
    out = [_block_to_numpy(blocks[l]) for l in range(L)]
    for l in range(L):
        lib().oracle_free_block(ctypes.byref(blocks[l]))
    return out


def random_walk(indptr, indices, starts, length: int, rng_seed: int, independent: bool = False) -> np.ndarray:
    """Walk traces int32[n][length + 1] (-1 after a dead end).
    independent: each walk draws with its own index (R35)."""
    ip = _c(indptr, np.int64)
    ix = _c(indices, np.int32)
    st = _c(starts, np.int32)
    out = np.zeros((len(st), length + 1), np.int32)
    fn = lib().oracle_random_walk_independent if independent else lib().oracle_random_walk
    rc = fn(len(ip) - 1, _ptr(ip), _ptr(ix), _ptr(st), len(st), length, rng_seed, _ptr(out))
    if rc != OK:
        raise OracleError(rc, "oracle_random_walk")
    return out


def gather(features, ids) -> np.ndarray:
    """out[r] = features[ids[r]] (fp32 bits copied)."""
    f = np.ascontiguousarray(features, dtype=np.float32)
    N, dim = f.shape
    ids = _c(ids, np.int32)
    out = np.empty((len(ids), dim), np.float32)
    rc = lib().oracle_gather(N, dim, _ptr(f), _ptr(ids), len(ids), _ptr(out))
    if rc != OK:
        raise OracleError(rc, "oracle_gather")
    return out
