"""Multi-GPU bootstrap: one process per GPU (torchrun), the NCCL unique id
created by rank 0 through the C ABI and broadcast over the caller's
torch.distributed group, then ratel_init on every rank.

The library's own communicator carries only the two collectives BASELINE.json
allows: the 8-byte grad-norm allreduce (clip mode) and the per-block bf16
P16 all-gather.  Partitioning is ratel_rank_slice (a pure C
function), so every rank derives the same slices without communication.
"""
from __future__ import annotations

from . import ratel as R


def broadcast_unique_id(group=None, getter=None) -> bytes:
    """Rank 0 calls `getter` (default: ratel_get_nccl_unique_id) and the 128
    bytes are broadcast to every rank of `group`."""
    import torch
    import torch.distributed as dist
    getter = getter or R.ratel_get_nccl_unique_id
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    buf = torch.zeros(128, dtype=torch.uint8, device=dev)
    if dist.get_rank(group) == 0:
        uid = getter()
        assert len(uid) == 128
        buf.copy_(torch.frombuffer(bytearray(uid), dtype=torch.uint8))
    dist.broadcast(buf, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    return bytes(buf.cpu().numpy().tobytes())


def init_distributed(device_index: int, cfg=None, group=None) -> tuple[int, int]:
    """ratel_init for this process.  Single process: world 1, no NCCL."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        R.ratel_init(device_index, 0, 1, None, cfg)
        return 0, 1
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = broadcast_unique_id(group)
    R.ratel_init(device_index, rank, world, uid, cfg)
    return rank, world
