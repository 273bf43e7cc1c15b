"""Multi-GPU plumbing of the hot path (row a9): whole files are sharded across
ranks by contiguous file ranges (no file straddles two GPUs, so chunk ownership is unchanged), each
rank runs its own libgsys instance (own syscall area, service threads and streams), and ONE
all-reduce(SUM) of the int64 vector [64 word counts | per-file grep hits] over the process group
(NCCL over NVLink on the B200 box; gloo in the CPU tests) produces the global answer.  Files are
disjoint across ranks, so the summed hit vector equals the OR."""
from __future__ import annotations

import torch


def shard_range(nfiles: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous file range [lo, hi) of `rank`; sizes differ by at most one file."""
    if world <= 0 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return rank * nfiles // world, (rank + 1) * nfiles // world


def pack_result(hist: torch.Tensor, hits: torch.Tensor | None, lo: int, hi: int, nfiles: int,
                ndict: int = 64) -> torch.Tensor:
    """[ndict counts | nfiles hits] with this rank's hits placed at [ndict+lo, ndict+hi)."""
    v = torch.zeros(ndict + nfiles, dtype=torch.int64, device=hist.device)
    v[:ndict] = hist.to(torch.int64)
    if hits is not None and hi > lo:
        v[ndict + lo: ndict + hi] = hits.to(torch.int64)[: hi - lo]
    return v


def reduce_result(v: torch.Tensor, group=None) -> torch.Tensor:
    """The only collective of the path: all_reduce(SUM) in place (no-op without a process group)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(v, op=dist.ReduceOp.SUM, group=group)
    return v


def unpack_result(v: torch.Tensor, ndict: int = 64):
    return v[:ndict], v[ndict:]
