"""Multi-process (gloo, world_size 2) coverage of the N>1 host path: row sharding and the final
category all-gather (the path's only collective)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_jiangh0h23_b200.parallel import (allgather_categories, allgather_categories_padded,
                                                       assemble_categories, shard_capacity, shard_rows)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, B, cats, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    a, b = shard_rows(B, world, rank)
    local = torch.tensor([c for c in cats if a <= c < b], dtype=torch.int64)
    got = allgather_categories(local)
    # the padded device-export form: [count, ids..., junk] per rank, one collective
    cap = shard_capacity(B, world)
    buf = torch.full((1 + cap,), -5, dtype=torch.int64)
    buf[0] = local.numel()
    buf[1:1 + local.numel()] = local
    gathered = allgather_categories_padded(buf)
    assert tuple(gathered.shape) == (world, 1 + cap)
    got2 = assemble_categories(gathered)
    assert got2.tolist() == got.tolist()
    q.put((rank, got.tolist(), (a, b)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,B,cats", [(2, 11, [0, 3, 4, 9, 10]), (2, 7, [5]), (3, 9, [])])
def test_allgather_categories_gloo(world, B, cats):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, B, cats, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    shards = sorted(r[2] for r in res)
    assert shards[0][0] == 0 and shards[-1][1] == B
    assert all(shards[i][1] == shards[i + 1][0] for i in range(len(shards) - 1))
    for _, got, _ in res:
        assert got == sorted(cats)


def test_shard_rows_cover():
    for B in (0, 1, 7, 60000):
        for w in (1, 2, 4, 8):
            spans = [shard_rows(B, w, r) for r in range(w)]
            assert spans[0][0] == 0 and spans[-1][1] == B
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1
