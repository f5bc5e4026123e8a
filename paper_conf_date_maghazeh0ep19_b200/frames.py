"""Frame-batch sharding across GPUs (BASELINE configs[3]: "batch of 64 8K
frames ... sharded across 1/2/4/8 B200").

Frames are independent (the kernel graph never reads across frames; PAPER.md:189 blocks
are independent, z = frame), so the one batch is split into contiguous frame ranges, one
per rank, with no data-path collective: each rank plans and executes the same graph over
its own frames.  Only timing crosses ranks (a barrier and the max over ranks).
Bookkeeping only — no pixel arithmetic here."""
from __future__ import annotations


def frame_range(total: int, world: int, rank: int) -> tuple[int, int]:
    """(first frame, frame count) of `rank`: contiguous ranges, the first total % world ranks
    take one frame more, so every frame is owned by exactly one rank."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("need 0 <= rank < world")
    if total < world:
        raise ValueError(f"{total} frames cannot be sharded over {world} ranks (one frame per rank at least)")
    q, r = divmod(total, world)
    n = q + (1 if rank < r else 0)
    f0 = rank * q + min(rank, r)
    return f0, n


def max_over_ranks(ms: float, world: int, device=None) -> float:
    """The step time of the whole job: the slowest rank's (all_reduce MAX); identity at
    world == 1."""
    if world <= 1:
        return ms
    import torch
    import torch.distributed as dist
    t = torch.tensor([ms], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def job_mpix_per_s(pixels_per_rank: list, ms: float) -> float:
    """Whole-job throughput: every rank's pixels over the max-over-ranks step time."""
    return sum(pixels_per_rank) / (ms / 1000.0) / 1e6
