"""Multi-process wiring over torch.distributed -- control plane only.

One process per GPU (data parallelism).  NCCL (or gloo in CPU tests) carries
only the init-time metadata: the IPC handle of every rank's cache slab (peer-based access
in a unified address space) and a placement digest proving every rank solved
the same policy, plus barriers.  Nothing here runs per batch, and no collective ever
carries embedding rows (the paper's message-based AllToAll, is what UGache
avoids).
"""
from __future__ import annotations

import hashlib
from typing import List, Optional

import numpy as np


def world():
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        return dist.get_rank(), dist.get_world_size()
    return 0, 1


def placement_digest(plan_dict: dict, order: Optional[np.ndarray]) -> str:
    h = hashlib.sha256()
    for k in sorted(plan_dict):
        h.update(f"{k}={plan_dict[k]!r};".encode())
    if order is not None:
        h.update(np.ascontiguousarray(order).tobytes())
    return h.hexdigest()


def exchange_handles(handle: bytes, digest: str, group=None) -> List[bytes]:
    """all_gather of (IPC handle, placement digest); raises if ranks disagree on the
    placement.  Works with any backend that supports all_gather_object."""
    import torch.distributed as dist
    rank, ws = world()
    if ws == 1:
        return [handle]
    got: List = [None] * ws
    dist.all_gather_object(got, (handle, digest), group=group)
    digests = {d for _, d in got}
    if len(digests) != 1:
        raise RuntimeError(f"ranks solved different placements: {sorted(digests)}")
    return [h for h, _ in got]


def barrier(group=None):
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized():
        dist.barrier(group=group)


def _reduce(value: float, op_name: str) -> float:
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    dev = "cpu"
    if dist.get_backend() == "nccl":
        dev = torch.device("cuda", torch.cuda.current_device())
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=getattr(dist.ReduceOp, op_name))
    return float(t.item())


def max_over_ranks(value: float) -> float:
    """Max of a per-rank scalar (batch time = max over GPUs)."""
    return _reduce(value, "MAX")


def sum_over_ranks(value: float) -> float:
    return _reduce(value, "SUM")


def gather_rows(values) -> np.ndarray:
    """All ranks' copies of a per-rank 1-D float vector, as a [world, len] float64 array
    (a SUM all-reduce of a matrix whose row r only rank r fills; gloo or NCCL)."""
    import torch
    import torch.distributed as dist
    v = np.asarray(values, dtype=np.float64).ravel()
    rank, ws = world()
    if ws == 1:
        return v[None, :].copy()
    dev = "cpu"
    if dist.get_backend() == "nccl":
        dev = torch.device("cuda", torch.cuda.current_device())
    m = torch.zeros((ws, len(v)), dtype=torch.float64, device=dev)
    m[rank] = torch.from_numpy(v).to(dev)
    dist.all_reduce(m, op=dist.ReduceOp.SUM)
    return m.cpu().numpy()


def connect(cache, group=None, order: Optional[np.ndarray] = None):
    """Exchange slab IPC handles and map every peer (ugache_open_peers)."""
    _, ws = world()
    if ws == 1:
        return
    digest = placement_digest(cache.plan.as_dict(), order)
    handles = exchange_handles(cache.ipc_handle(), digest, group)
    cache.open_peers(handles)
