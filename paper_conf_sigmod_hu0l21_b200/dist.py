"""Multi-GPU plumbing for a11 (one process per GPU, torch.distributed for rendezvous).

The exchange step of the path is ONE ncclAllReduce of the per-rank uint64 partials, issued
by the library itself inside ``tc_count_dist`` (libnccl.so.2 is dlopen'ed by libtc_b200).
This module only moves the 128-byte NCCL unique id between processes and reduces host
timings; it works with any torch.distributed backend (gloo in the CPU tests, nccl on B200).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def broadcast_bytes(payload: bytes | None, src: int = 0, group=None) -> bytes:
    """Rank `src` provides `payload`; every rank returns it."""
    obj = [payload if dist.get_rank() == src else None]
    dist.broadcast_object_list(obj, src=src, group=group)
    return obj[0]


def init_nccl_comm(rank: int, world: int, device: int, group=None):
    """Create the library's NCCL communicator (rank 0 makes the unique id)."""
    from . import tc_nccl_comm_init, tc_nccl_get_unique_id
    uid = broadcast_bytes(tc_nccl_get_unique_id() if rank == 0 else None, 0, group)
    return tc_nccl_comm_init(uid, rank, world, device)


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank scalar (multi-GPU timings are reported as the max over ranks)."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    dev = device if device is not None else (
        torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl"
        else torch.device("cpu"))
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def sum_over_ranks_u64(value: int, device=None, group=None) -> int:
    """Exact sum of per-rank non-negative integers (< 2^63) — host-side check helper."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return int(value)
    dev = device if device is not None else torch.device("cpu")
    t = torch.tensor([int(value)], dtype=torch.int64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return int(t.item())
