"""Multi-process plumbing for the sharded run (one process per GPU, torch.distributed).

torch.distributed only carries the NCCL unique id to every rank and reduces timings; the
per-round exchange (allreduce-MIN of the component minima) happens inside
libmst.so on its own NCCL communicator. Works with the gloo backend (CPU tests) and nccl.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def _device_for(group=None):
    backend = dist.get_backend(group)
    return torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")


def broadcast_bytes(payload: bytes | None, nbytes: int, src: int = 0, group=None) -> bytes:
    """Rank `src` sends `payload` (exactly nbytes); every rank returns it."""
    t = torch.zeros(nbytes, dtype=torch.uint8, device=_device_for(group))
    if dist.get_rank(group) == src:
        assert payload is not None and len(payload) == nbytes
        t.copy_(torch.frombuffer(bytearray(payload), dtype=torch.uint8))
    dist.broadcast(t, src, group=group)
    return bytes(t.cpu().numpy().tobytes())


def share_unique_id(make_id, group=None) -> bytes:
    """Rank 0 creates the 128-byte NCCL unique id (mst_get_unique_id); all ranks get it."""
    payload = make_id() if dist.get_rank(group) == 0 else None
    return broadcast_bytes(payload, 128, 0, group)


def allreduce_min_u64_(words, group=None) -> None:
    """In place: words (numpy uint64) <- their element-wise minimum over all ranks. The
    exchange of mst_create_dist_hostx (test aid) over any backend: uint64 -> int64 by flipping
    the sign bit preserves the order, so the backend's signed MIN is the unsigned MIN."""
    import numpy as np
    flip = np.uint64(1 << 63)
    t = torch.from_numpy((words ^ flip).view(np.int64).copy())
    dev = _device_for(group)
    if dev.type != "cpu":
        t = t.to(dev)
    dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    words[:] = t.cpu().numpy().view(np.uint64) ^ flip


def max_over_ranks(x: float, group=None) -> float:
    """The bench's timing rule: the slowest rank's time."""
    t = torch.tensor([float(x)], dtype=torch.float64, device=_device_for(group))
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
