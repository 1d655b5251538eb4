"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds none of the sampling method's arithmetic: it only makes the
graph (R-MAT, symmetrised, renumbered by a Feistel bijection), the fp32
feature table, the train-id set and the per-rank seed batches.  See
``datagen.cpp`` for the recipe and DESIGN.md "Input recipe" for the reasoning.
"""
from __future__ import annotations

import ctypes
import dataclasses
import math
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "datagen.cpp")
_LIB = os.path.join(_HERE, "libdatagen.so")

GRAPH_SEED = 1
FEAT_SEED = 2
BASE_SEED = 0x5EED
RMAT_ABC = (0.45, 0.15, 0.15)  # d = 0.25 (SURVEY.md 8(d) calibration)


@dataclasses.dataclass(frozen=True)
class Config:
    """One BASELINE.json configuration (shapes from PAPER.md Table 3)."""
    name: str
    num_nodes: int
    num_undirected_edges: int
    dim: int
    fanouts: tuple
    batch: int              # seeds per GPU per step (read per GPU)
    train_count: int        # size of the train-id set
    rmat: tuple = RMAT_ABC


CONFIGS = {
    # BASELINE.json configs[0]: the small case the oracle finishes in seconds
    "tiny": Config("tiny", 10_000, 100_000, 16, (5, 5), 64, 10_000),
    # configs[1]/[2]: ogbn-products shaped (Table 3: 2.45M nodes,
    # 123M directed edges, dim 100); train split size of ogbn-products
    "products": Config("products", 2_449_029, 61_859_140, 100, (15, 10, 5), 1024, 196_615),
    # configs[3]: ogbn-papers100M shaped (111M nodes, 3.2B directed, dim 128)
    "papers": Config("papers", 111_059_956, 1_615_685_872, 128, (15, 10, 5), 1024, 1_207_179),
    # configs[4]: Friendster shaped (65.6M nodes, 3.6B directed, dim 256); 1% train
    "friendster": Config("friendster", 65_608_366, 1_806_067_135, 256, (15, 10, 5), 1024, 656_084),
}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O3", "-march=x86-64-v3", "-std=c++17", "-fPIC", "-shared",
                               "-fopenmp", "-Wall", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P = ctypes.c_void_p
        L.datagen_rmat_csr.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                       ctypes.c_double, ctypes.c_uint64, ctypes.c_int, P,
                                       ctypes.POINTER(ctypes.c_void_p)]
        L.datagen_rmat_csr.restype = ctypes.c_int64
        L.datagen_free.argtypes = [P]
        L.datagen_features.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64,
                                       ctypes.c_int, P]
        L.datagen_features_of.argtypes = [P, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, P]
        L.datagen_node_weights.argtypes = [ctypes.c_int64, ctypes.c_uint64, P]
        L.datagen_edge_weights.argtypes = [P, ctypes.c_int64, P, P]
        L.datagen_permute.argtypes = [ctypes.c_int64, ctypes.c_uint64, ctypes.c_int64]
        L.datagen_permute.restype = ctypes.c_int64
        L.datagen_permute_many.argtypes = [ctypes.c_int64, ctypes.c_uint64, P, ctypes.c_int64, P]
        _lib = L
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def threads_default() -> int:
    return max(1, len(os.sched_getaffinity(0)))


def rmat_csr(num_nodes: int, num_undirected_edges: int, abc=RMAT_ABC, graph_seed: int = GRAPH_SEED,
             threads: int | None = None):
    """Renumbered symmetric R-MAT CSR: (indptr int64[N+1], indices int32[nnz])."""
    indptr = np.zeros(num_nodes + 1, np.int64)
    raw = ctypes.c_void_p()
    nnz = lib().datagen_rmat_csr(num_nodes, num_undirected_edges, abc[0], abc[1], abc[2], graph_seed,
                                 threads or threads_default(), _ptr(indptr), ctypes.byref(raw))
    if nnz < 0:
        raise MemoryError("datagen_rmat_csr: allocation failed")
    indices = np.empty(nnz, np.int32)
    if nnz:
        ctypes.memmove(indices.ctypes.data, raw.value, nnz * 4)
    lib().datagen_free(raw)
    return indptr, indices


def features(lo: int, hi: int, dim: int, feat_seed: int = FEAT_SEED, threads: int | None = None):
    out = np.empty((hi - lo, dim), np.float32)
    lib().datagen_features(lo, hi, dim, feat_seed, threads or threads_default(), _ptr(out))
    return out


def features_of(ids, dim: int, feat_seed: int = FEAT_SEED):
    ids = np.ascontiguousarray(ids, np.int32)
    out = np.empty((len(ids), dim), np.float32)
    lib().datagen_features_of(_ptr(ids), len(ids), dim, feat_seed, _ptr(out))
    return out


WEIGHT_SEED = 3


def node_weights(n: int, seed: int = WEIGHT_SEED) -> np.ndarray:
    """Biased-sampling node weights w_u: ~1/32 zeros, else k/16 in (0, 256]."""
    out = np.empty(n, np.float32)
    lib().datagen_node_weights(n, seed, _ptr(out))
    return out


def edge_weights(indices: np.ndarray, w: np.ndarray) -> np.ndarray:
    """Weight stored with each edge e_{v,u}: w[u] ("DSP stores node weight w_u along
    with edge e_{v,u}")."""
    ix = np.ascontiguousarray(indices, np.int32)
    w = np.ascontiguousarray(w, np.float32)
    out = np.empty(len(ix), np.float32)
    lib().datagen_edge_weights(_ptr(ix), len(ix), _ptr(w), _ptr(out))
    return out


def permute(n: int, key: int, x) -> np.ndarray:
    x = np.ascontiguousarray(x, np.int64)
    out = np.empty_like(x)
    lib().datagen_permute_many(n, key, _ptr(x), len(x), _ptr(out))
    return out


def bounds(num_nodes: int, world: int) -> np.ndarray:
    """Contiguous ownership ranges: bounds[r] = floor(r N / P) (R21)."""
    return np.array([(r * num_nodes) // world for r in range(world + 1)], np.int64)


def train_ids(num_nodes: int, count: int, graph_seed: int = GRAPH_SEED) -> np.ndarray:
    """The train-id set sigma(0 .. count-1) of a second Feistel bijection."""
    return permute(num_nodes, graph_seed * 0xD1B54A32D192ED03 + 7, np.arange(count, dtype=np.int64))


def rank_seed_batches(train: np.ndarray, bnds: np.ndarray, rank: int, batch: int, epoch: int,
                      base_seed: int = BASE_SEED) -> np.ndarray:
    """Seeds co-partitioned with the topology: this rank's train ids,
    shuffled per epoch, cut into full batches -> int32[steps, batch]."""
    lo, hi = int(bnds[rank]), int(bnds[rank + 1])
    mine = np.sort(train[(train >= lo) & (train < hi)])
    rng = np.random.default_rng([base_seed, epoch, rank])
    mine = mine[rng.permutation(len(mine))]
    steps = len(mine) // batch
    return mine[: steps * batch].astype(np.int32).reshape(steps, batch)


def steps_per_epoch(train: np.ndarray, bnds: np.ndarray, batch: int) -> int:
    """Every rank makes the same number of collective calls: min over ranks."""
    P = len(bnds) - 1
    return min(int(((train >= bnds[r]) & (train < bnds[r + 1])).sum()) // batch for r in range(P))


def shard(indptr: np.ndarray, indices: np.ndarray, lo: int, hi: int):
    """Rows [lo, hi) of a CSR as a local CSR (indptr rebased to 0, global ids kept)."""
    ip = indptr[lo: hi + 1]
    return (ip - ip[0]).astype(np.int64), indices[ip[0]: ip[-1]]


_cache: dict = {}


def make_graph(cfg: Config | str, threads: int | None = None):
    """(indptr, indices) of a named config, cached per process."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    key = (cfg.num_nodes, cfg.num_undirected_edges, cfg.rmat)
    if key not in _cache:
        _cache[key] = rmat_csr(cfg.num_nodes, cfg.num_undirected_edges, cfg.rmat, threads=threads)
    return _cache[key]


def scale_of(n: int) -> int:
    return max(1, math.ceil(math.log2(max(n, 2))))
