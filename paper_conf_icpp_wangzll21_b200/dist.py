"""Host-side plumbing for multi-GPU search: one process per GPU.

References shard by global id into contiguous ranges; rank 0 creates the NCCL unique id
(libtid) and broadcasts it through the torch.distributed process group; every rank then
creates its tid.Index with (rank, world_size, id_base) and calls search collectively (the
library all-gathers the per-rank top-k over NCCL and merges on the GPU).
"""
from __future__ import annotations


def shard_plan(R_total: int, world_size: int, rank: int) -> tuple[int, int]:
    """[start, end) of this rank's references: contiguous, sizes differ by at most one."""
    if world_size < 1 or not 0 <= rank < world_size:
        raise ValueError("bad rank/world_size")
    base, rem = divmod(R_total, world_size)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


def exchange_nccl_id(make_id, group=None) -> bytes:
    """Rank 0 calls make_id() (-> 128 bytes); every rank returns the same bytes."""
    import torch.distributed as dist
    obj = [make_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    uid = obj[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise RuntimeError("bad ncclUniqueId")
    return bytes(uid)


def create_sharded_index(R_total: int, ref_kp: int, device: int, **kw):
    """Collective: build this rank's Index for a reference set of R_total ids."""
    import torch.distributed as dist
    from . import Index, nccl_unique_id
    rank, world = dist.get_rank(), dist.get_world_size()
    start, end = shard_plan(R_total, world, rank)
    uid = exchange_nccl_id(nccl_unique_id) if world > 1 else None
    return Index(ref_kp=ref_kp, device=device, id_base=start, rank=rank, world_size=world, nccl_id=uid, **kw), (start, end)
