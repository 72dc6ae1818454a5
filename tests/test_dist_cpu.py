"""Host-side logic of the row-sharded path, world_size 2 over gloo on CPU (no GPU needed):
row partition, seeded shard reproducibility, NCCL-id broadcast, and the bench harness's
max-over-ranks timing reduction."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import dist as rdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        m, n = 2 * gi.ROW_BLOCK * 2, 8
        row0, ml = rdist.shard_rows(m, world, rank)
        shard = gi.gaussian(ml, n, seed=5, dtype="fp16", row0=row0)
        # every rank gathers the shards; concatenation must equal the unsharded matrix
        parts = [None] * world
        dist.all_gather_object(parts, (row0, shard))
        # id broadcast: rank 0's object reaches everyone
        obj = [b"id-from-rank0" if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        # bench-style max over ranks of a per-rank time
        t = torch.tensor([float(rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        out[rank] = (parts, obj[0], float(t.item()))
    finally:
        dist.destroy_process_group()


def test_shard_rows_partition():
    m = 8 * rdist.ROW_ALIGN
    blocks = [rdist.shard_rows(m, 4, r) for r in range(4)]
    assert blocks[0] == (0, 2 * rdist.ROW_ALIGN)
    assert sum(b[1] for b in blocks) == m
    assert all(blocks[i][0] + blocks[i][1] == blocks[i + 1][0] for i in range(3))
    with pytest.raises(ValueError):
        rdist.shard_rows(m + 8, 4, 0)


def test_gloo_world2_host_logic():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    m = 2 * gi.ROW_BLOCK * 2
    full = gi.gaussian(m, 8, seed=5, dtype="fp16")
    for r in range(world):
        parts, uid, tmax = out[r]
        assert uid == b"id-from-rank0"
        assert tmax == float(world)
        stacked = np.concatenate([p[1] for p in sorted(parts, key=lambda x: x[0])], axis=0)
        np.testing.assert_array_equal(stacked, full)
