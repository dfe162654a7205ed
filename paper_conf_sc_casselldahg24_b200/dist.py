"""Host-side helpers of the multi-GPU path; torch.distributed is
plumbing only: it carries the NCCL unique id and the max-over-ranks timing.
The exchange itself (the per-step all-gather) runs inside libnbody_b200.so."""
from __future__ import annotations

import ctypes as C

from . import _capi


def owned_range(n: int, rank: int, world: int):
    """[begin, end) of the sorted slots `rank` owns (the library's rule [A21])."""
    b, e = C.c_int64(), C.c_int64()
    st = _capi.load().nbody_partition(int(n), int(rank), int(world), C.byref(b), C.byref(e))
    if st != 0:
        raise _capi.NBodyError(st, "nbody_partition")
    return b.value, e.value


def new_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    st = _capi.load().nbody_nccl_unique_id(buf)
    if st != 0:
        raise _capi.NBodyError(st, "ncclGetUniqueId failed")
    return buf.raw


def broadcast_unique_id(rank: int, group=None) -> bytes:
    """Rank 0 creates an ncclUniqueId; the process group broadcasts it."""
    import torch.distributed as dist
    obj = [new_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def max_over_ranks(value: float, device=None) -> float:
    """All-reduce MAX of a host float (timing is reported as the max over ranks)."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
