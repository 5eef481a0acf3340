"""bqr_dist -- host-side multi-GPU plumbing for the bench (no method arithmetic).

The batch shards trivially: independent matrices ("we
distribute independent problems across different multiprocessors", extended
here across GPUs).  Each rank owns a contiguous slice of one seeded stream,
so any world size sees identical matrices; there is no data-path collective.
NCCL (or gloo on CPU) is used only for barriers, the MAX of per-rank device
times and a gather of per-rank checksums.
"""
from __future__ import annotations

import hashlib
import os

import numpy as np


def env_rank():
    """(rank, world_size, local_rank) from the torchrun environment."""
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def rank_slice(rank: int, world: int, per_rank: int, weak: bool = True, total: int | None = None):
    """Matrix index range [lo, hi) of `rank`.

    weak=True: every rank gets `per_rank` matrices of a world*per_rank stream
    (per-GPU work fixed as N grows).  weak=False: `total` matrices split
    floor(r B / P) .. floor((r+1) B / P) (strong scaling)."""
    if weak:
        return rank * per_rank, (rank + 1) * per_rank
    assert total is not None
    return (rank * total) // world, ((rank + 1) * total) // world


def _dev_tensor(torch, dist, values, dtype):
    backend = dist.get_backend() if dist.is_initialized() else "gloo"
    dev = "cuda" if backend == "nccl" else "cpu"
    return torch.tensor(values, dtype=dtype, device=dev)


def max_over_ranks(torch, dist, x: float) -> float:
    """MAX of a per-rank scalar (device time) over the process group."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(x)
    t = _dev_tensor(torch, dist, [float(x)], torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(torch, dist):
    """Device sync + process-group barrier + device sync (bench timing rule)."""
    if torch.cuda.is_available():
        torch.cuda.synchronize()
    if dist is not None and dist.is_initialized() and dist.get_world_size() > 1:
        dist.barrier()
    if torch.cuda.is_available():
        torch.cuda.synchronize()


def checksum(arr: np.ndarray) -> int:
    """64-bit checksum of an array's bytes (bitwise determinism across P)."""
    return int.from_bytes(hashlib.blake2b(np.ascontiguousarray(arr).tobytes(), digest_size=8).digest(), "little")


def gather_ints(torch, dist, values: list[int]) -> list[list[int]]:
    """all_gather of a small list of ints from every rank."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return [list(values)]
    t = _dev_tensor(torch, dist, [v & 0x7FFFFFFFFFFFFFFF for v in values], torch.int64)
    out = [torch.empty_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(out, t)
    return [o.cpu().tolist() for o in out]
