"""Row-sharded (multi-GPU) plumbing around the C ABI.

One process per GPU.  Each rank owns a contiguous block of rows of A (and Q); every rank
runs the same recursion on its rows.  The library itself exchanges what the method needs:
the R12 partials after each inner product (ncclAllReduce) and the leaf's per-column
reductions (in-kernel red.add into every GPU's exchange words over NVLink).  torch is used
only to broadcast the 128-byte NCCL id and for rank bookkeeping.
"""
from __future__ import annotations

from .rgsqr import Handle, load_library

ROW_ALIGN = 4096          # shards start on rgsqr_inputs.ROW_BLOCK boundaries (reproducible inputs)


def shard_rows(m: int, world: int, rank: int, align: int = ROW_ALIGN) -> tuple[int, int]:
    """(row0, m_local) of `rank`'s contiguous row block.  The library requires the same
    m_local on every rank, so m must split into `world` equal aligned blocks."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank / world")
    if m % (world * align):
        raise ValueError(f"m={m} must be a multiple of world*align={world * align}")
    ml = m // world
    return rank * ml, ml


def broadcast_unique_id(rank: int, pg=None) -> bytes:
    """Rank 0 creates the NCCL id; torch.distributed broadcasts it (any backend)."""
    import torch.distributed as dist
    obj = [Handle.unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=pg)
    return obj[0]


def create_handle(device: int, rank: int, world: int, pg=None) -> Handle:
    """Collective: every rank calls it; returns a distributed library context."""
    load_library()
    uid = broadcast_unique_id(rank, pg)
    return Handle(device, rank=rank, nranks=world, unique_id=uid)
