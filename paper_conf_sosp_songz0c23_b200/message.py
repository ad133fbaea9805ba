"""Message-based extraction baseline -- NOT the hot path.

"With message-based extraction, a GPU sends keys to the GPU caching them, which then looks
up and sends back the values ... the GPU then has to reorder the values back to the
original key order".  This is what WholeGraph-style peer loads and UGache's
factored extraction replace; it is here so the comparison runs through the same
placement, location tables and kernels (include/ugache.h "message-based baseline").

Per batch and GPU: ``ugache_msg_extract_local`` (locate + bucket + local/host rows) ->
``ugache_msg_requests`` (per-peer slot ids, host sync for the counts) -> all-to-all of
counts and requests -> ``ugache_msg_serve`` on each owner -> all-to-all of rows ->
``ugache_msg_scatter`` into key order.  The exchanges are torch.distributed all-to-alls
(NCCL) in :func:`message_extract`, or device copies between contexts sharing one device
in :func:`message_extract_group` (the single-GPU "fake peer" setting of the tests).
Python does marshalling and the collective calls only; every row moves in libugache's
kernels or in the collective.
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np

from . import _abi
from ._abi import check, lib
from .ugache import UGache, _ptr, _stream_handle


def _key_type(keys):
    import torch
    if keys.dtype == torch.int64:
        return _abi.KEY_I64
    if keys.dtype in (torch.int32, torch.uint32):
        return _abi.KEY_U32
    raise TypeError("keys must be int64 or (u)int32")


def _local(c: UGache, keys, out, stream):
    check(lib().ugache_msg_extract_local(c.ctx, _ptr(keys), _key_type(keys), keys.numel(),
                                         _ptr(out), _stream_handle(stream)),
          "ugache_msg_extract_local", c.ctx)


def _requests(c: UGache, stream):
    """-> (counts[G+1] numpy, req u32 device tensor packed in peer rank order)."""
    import torch
    G = c.num_gpus
    counts = np.zeros(G + 1, dtype=np.uint64)
    # the packed size is only known after the counts; allocate the upper bound (batch size)
    req = torch.empty(max(1, c._msg_n), dtype=torch.int32, device="cuda")
    check(lib().ugache_msg_requests(c.ctx, _ptr(counts), _ptr(req), _stream_handle(stream)),
          "ugache_msg_requests", c.ctx)
    counts = counts.astype(np.int64)
    n_req = int(sum(counts[j] for j in range(G) if j != c.rank))
    return counts, req[:n_req]


def _serve(c: UGache, req_in, send, stream):
    check(lib().ugache_msg_serve(c.ctx, _ptr(req_in), req_in.numel(), _ptr(send),
                                 _stream_handle(stream)), "ugache_msg_serve", c.ctx)


def _scatter(c: UGache, replies, out, stream):
    check(lib().ugache_msg_scatter(c.ctx, _ptr(replies), _ptr(out), _stream_handle(stream)),
          "ugache_msg_scatter", c.ctx)


def message_extract_group(caches: Sequence[UGache], keys_list: Sequence, outs: Sequence = None,
                          stream=None) -> List:
    """One message-based batch for G contexts of ONE process (fake peers on one device, or
    several devices with peer access): the two all-to-alls are device-to-device copies."""
    import torch
    G = len(caches)
    R = caches[0].row_bytes
    if outs is None:
        outs = [torch.empty((k.numel(), R), dtype=torch.uint8, device="cuda") for k in keys_list]
    for c, k, o in zip(caches, keys_list, outs):
        c._msg_n = k.numel()
        _local(c, k, o, stream)
    reqs = []
    for c in caches:
        counts, req = _requests(c, stream)
        # split req by destination peer (rank order, skipping self)
        parts, off = {}, 0
        for j in range(G):
            if j == c.rank:
                continue
            parts[j] = req[off: off + int(counts[j])]
            off += int(counts[j])
        reqs.append(parts)
    # exchange 1 (requests): owner j receives, from every requester i in rank order, parts
    replies = [dict() for _ in range(G)]
    for j, owner in enumerate(caches):
        incoming = [reqs[i][j] for i in range(G) if i != j]
        req_in = torch.cat(incoming) if incoming else torch.empty(0, dtype=torch.int32, device="cuda")
        send = torch.empty((max(1, req_in.numel()), R), dtype=torch.uint8, device="cuda")
        _serve(owner, req_in, send, stream)
        off = 0
        for i in range(G):  # exchange 2 (rows): slice the send buffer back per requester
            if i == j:
                continue
            m = reqs[i][j].numel()
            replies[i][j] = send[off: off + m]
            off += m
    for i, c in enumerate(caches):
        parts = [replies[i][j] for j in range(G) if j != i]
        rep = torch.cat(parts) if parts else torch.empty((0, R), dtype=torch.uint8, device="cuda")
        _scatter(c, rep, outs[i], stream)
    return list(outs)


def message_extract(c: UGache, keys, out=None, group=None, stream=None):
    """One message-based batch on this rank; every rank of ``group`` calls it together.
    Exchanges: all_to_all_single of counts, of slot ids, and of rows -- NCCL on device
    buffers, or staged through host memory when the group's backend is gloo (ranks sharing
    one GPU in tests)."""
    import torch
    import torch.distributed as dist
    G, me, R = c.num_gpus, c.rank, c.row_bytes
    if out is None:
        out = torch.empty((keys.numel(), R), dtype=torch.uint8, device="cuda")
    host_xchg = dist.get_backend(group) == "gloo"

    def a2a(dst, src, out_split=None, in_split=None):
        if host_xchg:
            d = torch.empty(dst.shape, dtype=dst.dtype)
            torch.cuda.synchronize()
            dist.all_to_all_single(d, src.cpu(), output_split_sizes=out_split,
                                   input_split_sizes=in_split, group=group)
            dst.copy_(d)
        else:
            dist.all_to_all_single(dst, src, output_split_sizes=out_split,
                                   input_split_sizes=in_split, group=group)

    c._msg_n = keys.numel()
    _local(c, keys, out, stream)
    counts, req = _requests(c, stream)
    send_counts = [0 if j == me else int(counts[j]) for j in range(G)]
    sc = torch.tensor(send_counts, dtype=torch.int64, device="cuda")
    rc = torch.empty_like(sc)
    a2a(rc, sc)
    recv_counts = rc.cpu().tolist()
    req_in = torch.empty(sum(recv_counts), dtype=torch.int32, device="cuda")
    a2a(req_in, req[: sum(send_counts)], recv_counts, send_counts)
    send = torch.empty((max(1, req_in.numel()), R), dtype=torch.uint8, device="cuda")
    _serve(c, req_in, send, stream)
    rep = torch.empty((sum(send_counts), R), dtype=torch.uint8, device="cuda")
    a2a(rep, send[: req_in.numel()], send_counts, recv_counts)
    _scatter(c, rep, out, stream)
    return out
