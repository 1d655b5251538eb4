"""bench.py -- CSP sampling + feature gather throughput (work in progress)."""
import torch
import torch.distributed as dist


def reduce_max_over_ranks(x: float) -> float:
    """Max of a per-rank device time over all ranks (1 rank: identity)."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(x)
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


if __name__ == "__main__":
    raise SystemExit("bench.py: CUDA path not built yet")
