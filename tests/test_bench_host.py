"""CPU checks of bench.py's N > 1 host arithmetic (no GPU): the NVLink byte
count of a step from a rank's blocks (per requester, remote
frontier ids sent + count and rows returned, remote feature rows read) on
the oracle's blocks of a 2-way partition, and the host description the CPU
baseline reports."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import bench  # noqa: E402
import datagen  # noqa: E402
import oracle  # noqa: E402


class _B:
    """A block as the binding's Block (tensor views) from an oracle block."""

    def __init__(self, b):
        self.num_dst, self.num_src, self.num_edges = int(b["num_dst"]), int(b["num_src"]), int(b["num_edges"])
        self.indptr = torch.from_numpy(b["indptr"].astype(np.int32))
        self.indices = torch.from_numpy(b["indices"].astype(np.int32))
        self.src_ids = torch.from_numpy(b["src_ids"].astype(np.int32))


def test_remote_bytes_counts_every_cross_rank_transfer(tiny_graph):
    ip, ix = tiny_graph
    bnds = datagen.bounds(10_000, 2)
    seeds = np.arange(int(bnds[0]), int(bnds[1]), 50, dtype=np.int32)
    blocks = oracle.sample(ip, ix, seeds, [5, 5], 7)
    csp, gat, rows = bench.remote_bytes([_B(b) for b in blocks], bnds, 0, 16)
    lo, hi = int(bnds[0]), int(bnds[1])
    exp_csp = 0
    for b in blocks:
        f = b["src_ids"][: b["num_dst"]]
        deg = np.diff(b["indptr"])
        rem = (f < lo) | (f >= hi)
        exp_csp += 4 * rem.sum() + 4 * rem.sum() + 4 * deg[rem].sum()   # id out, count back, rows back
    u = blocks[-1]["src_ids"]
    exp_rows = int(((u < lo) | (u >= hi)).sum())
    assert csp == exp_csp and rows == exp_rows and gat == exp_rows * 16 * 4
    assert rows > 0 and csp > 0                     # a random partition: about half the nodes are remote
    # layer 0 frontier = the rank's own seeds: nothing crosses for it
    first = blocks[0]["src_ids"][: blocks[0]["num_dst"]]
    assert ((first >= lo) & (first < hi)).all()


def test_host_cpu_reports_model_and_cores():
    h = bench.host_cpu()
    assert h["logical_cores"] >= 1 and 1 <= h["cores_available"] <= h["logical_cores"]
    assert h["model"] is None or isinstance(h["model"], str)


def test_default_instances():
    """--instances defaults: 2 streams for uniform node-wise steps at world 1, else 4."""
    assert bench.default_instances("uniform", 1) == 2
    for scheme in ("biased", "layer", "walk"):
        assert bench.default_instances(scheme, 1) == 4
    assert bench.default_instances("uniform", 2) == 4 and bench.default_instances("uniform", 8) == 4


def test_ncu_traffic_keys():
    """The bench-configuration capture keeps the plain kernel name bench.py reads;
    other workloads' captures of the same kernel do not overwrite it."""
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    import ncu_summary
    k = "k_csp_persistent<864, 1, 0, 1024>"
    assert ncu_summary.traffic_key(k, "r02g") == "k_csp_persistent"
    assert ncu_summary.traffic_key(k, "biased_r02g") == "k_csp_persistent@biased"
    assert ncu_summary.traffic_key(k, "single_r02g") == "k_csp_persistent@single"
    assert ncu_summary.traffic_key("k_gather_tma<0>", "gather_r02") == "k_gather_tma@gather"
