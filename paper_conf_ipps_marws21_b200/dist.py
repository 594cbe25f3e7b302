"""Multi-rank plumbing (one process per GPU, torchrun): process group, NCCL unique-id
exchange for the library's replica-merge communicator, and max/sum reductions used for the
timing rules.  torch.distributed is plumbing only; the merge itself is hb_merge (ncclAllReduce
inside libhogbatch.so)."""
from __future__ import annotations

import ctypes as C
import os

import numpy as np


def env_ranks():
    """(rank, world, local_rank) from the torchrun environment (defaults: single process)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def init(backend: str = "nccl", device=None):
    """Initialise the default process group when WORLD_SIZE > 1; returns (rank, world, local)."""
    import torch.distributed as dist
    rank, world, local = env_ranks()
    if world > 1 and not dist.is_initialized():
        kw = {"device_id": device} if (backend == "nccl" and device is not None) else {}
        dist.init_process_group(backend, **kw)
    return rank, world, local


def share_bytes(payload: bytes | None, src: int = 0) -> bytes:
    """Broadcast a byte string from `src` to every rank (the 128-byte ncclUniqueId)."""
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return payload
    obj = [payload]
    dist.broadcast_object_list(obj, src=src)
    return obj[0]


def reduce_scalar(value: float, op: str, device=None) -> float:
    """max / sum of a scalar over ranks (timing: max over ranks; samples: sum)."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return value
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
    return float(t.item())


def merge_schedule(N: int, merges_per_epoch: int, batches) -> tuple[int, int]:
    """(mid-epoch merges, total merges) of one rank's epoch, from the C++ MergeClock."""
    from . import _check, lib
    arr = np.ascontiguousarray(batches, dtype=np.int32)
    mid, tot = C.c_int32(), C.c_int32()
    _check(lib.hb_merge_schedule(N, merges_per_epoch, arr.ctypes.data_as(C.POINTER(C.c_int32)), arr.size,
                                 C.byref(mid), C.byref(tot)))
    return mid.value, tot.value
