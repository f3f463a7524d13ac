"""Row sharding and the one collective of the path.

Rows of the batch are independent (Eq. 1 acts per sample; clustering runs per shard), so each rank
infers a contiguous block of rows with replicated weights.  The only exchange is the final
all-gather of the category ids: counts first, then ids padded to the max count
(torch.distributed: NCCL on GPUs, gloo in the CPU tests).
"""
from __future__ import annotations

from typing import List, Tuple


def shard_rows(batch: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous block [start, end) of rows owned by `rank` (sizes differ by at most 1)."""
    base, rem = divmod(batch, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


def allgather_categories(local_ids, group=None):
    """All-gather variable-length int64 category ids (ascending per rank, ranks own ascending row
    blocks) -> the global ascending category set on every rank."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    dev = local_ids.device
    n = torch.tensor([local_ids.numel()], dtype=torch.int64, device=dev)
    counts: List = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(counts, n, group=group)
    cnt = [int(c.item()) for c in counts]
    m = max(cnt) if cnt else 0
    padded = torch.full((max(m, 1),), -1, dtype=torch.int64, device=dev)
    if local_ids.numel():
        padded[:local_ids.numel()] = local_ids
    parts = [torch.empty_like(padded) for _ in range(world)]
    dist.all_gather(parts, padded, group=group)
    return torch.cat([p[:c] for p, c in zip(parts, cnt)])
