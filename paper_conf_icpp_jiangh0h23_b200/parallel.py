"""Row sharding and the one collective of the path.

Rows of the batch are independent (Eq. 1 acts per sample; clustering runs per shard), so
each rank infers a contiguous block of rows with replicated weights.  The only exchange is the final
all-gather of the category ids (torch.distributed: NCCL over NVLink on GPUs, gloo in the CPU tests).

Two forms:
* ``allgather_categories_padded`` -- the production form: every rank exports [count, ids...] into a
  fixed-size device buffer (``snicit_categories_device``, no host round trip, capacity = the largest
  shard) and ONE all_gather of those buffers leaves the whole category set on every rank.  No host
  synchronisation is needed inside the step; ``assemble_categories`` turns the gathered buffers into the
  ascending global list when the caller wants it.
* ``allgather_categories`` -- variable-length ids (counts first, then ids padded to the max count), for
  callers that already hold a host/device id list.
"""
from __future__ import annotations

from typing import List, Tuple


def shard_rows(batch: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous block [start, end) of rows owned by `rank` (sizes differ by at most 1)."""
    base, rem = divmod(batch, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


def shard_capacity(batch: int, world: int) -> int:
    """Largest shard of `batch` rows over `world` ranks (the padded all-gather's capacity)."""
    return -(-batch // world) if world > 0 else batch


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


def allgather_categories_padded(local_buf, group=None):
    """local_buf: int64 tensor [1 + cap] = [count, ids...] (``SnicitNetwork.categories_device``).
    Returns the gathered [world, 1 + cap] tensor (same device): row r = rank r's [count, ids...].
    One collective, no host synchronisation."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    out = torch.empty((world, local_buf.numel()), dtype=local_buf.dtype, device=local_buf.device)
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(out, local_buf, group=group)
    else:  # gloo (CPU tests, the shared-GPU hook): list form
        dist.all_gather(list(out.unbind(0)), local_buf, group=group)
    return out


def assemble_categories(gathered):
    """[world, 1 + cap] gathered buffers -> ascending global category ids (int64, same device).
    Reads the counts (one small device->host copy)."""
    import torch

    counts = gathered[:, 0].tolist()
    cap = gathered.shape[1] - 1
    if any(c > cap for c in counts):
        raise ValueError("a shard has more categories than the buffer capacity")
    parts = [gathered[r, 1:1 + int(c)] for r, c in enumerate(counts)]
    return torch.cat(parts) if parts else gathered.new_empty(0)
