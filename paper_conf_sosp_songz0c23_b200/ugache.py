"""Thin Python layer over the C ABI (include/ugache.h): marshalling only.

``UGache`` is the embedding-layer object of P:1572-1580 ("applications ... replacing the
reference of embedding layer with UGache"): construct it once per GPU (solve + place),
connect peers, fill, then call :meth:`UGache.extract` per batch.  Every step of the
extraction runs in libugache's sm_100a kernels; torch is used only for device memory and
streams.
"""
from __future__ import annotations

import ctypes
from typing import List, Optional, Sequence

import numpy as np

from . import _abi
from ._abi import check, lib, ugache_config, ugache_plan


def _ptr(obj) -> int:
    """Address of a host/device buffer: int, numpy array, torch tensor, or obj.ptr."""
    if obj is None:
        return 0
    if isinstance(obj, int):
        return obj
    if hasattr(obj, "data_ptr"):
        return obj.data_ptr()
    if isinstance(obj, np.ndarray):
        return obj.ctypes.data
    if hasattr(obj, "ptr"):
        return int(obj.ptr)
    raise TypeError(f"cannot take the address of {type(obj)}")


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def make_config(num_rows: int, row_bytes: int, capacity_rows: int, num_gpus: int = 1,
                rank: int = 0, device: int = 0, policy: str = "ugache", bw_local: float = 0.0,
                bw_peer: float = 0.0, bw_host: float = 0.0, host_sms: int = 0,
                peer_sms: int = 0, num_sms: int = 0, host_tier: bool = False) -> ugache_config:
    return ugache_config(num_rows=num_rows, row_bytes=row_bytes, reserved0=0,
                         capacity_rows=capacity_rows, num_gpus=num_gpus, rank=rank,
                         device=device, policy=_abi.POLICIES[policy] if isinstance(policy, str) else policy,
                         bw_local=bw_local, bw_peer=bw_peer, bw_host=bw_host,
                         host_sms=host_sms, peer_sms=peer_sms, num_sms=num_sms,
                         flags=_abi.FLAG_HOST_TIER if host_tier else 0)


def model_time(plan: ugache_plan, locs, hotness: Optional[np.ndarray]) -> float:
    """Section 6.2 model value z of a placement (one location table per GPU) under hotness,
    with plan's T / R (ugache_model_time)."""
    arrs = [np.ascontiguousarray(l, dtype=np.uint64) for l in locs]
    ptrs = (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
    h = None if hotness is None else np.ascontiguousarray(hotness, dtype=np.float32)
    z = ctypes.c_double()
    check(lib().ugache_model_time(ctypes.byref(plan), len(arrs), len(arrs[0]), ctypes.cast(ptrs, ctypes.c_void_p),
                                  _ptr(h), ctypes.byref(z)), "ugache_model_time")
    return float(z.value)


def host_tier_rows(plan: ugache_plan, num_rows: int) -> int:
    return int(lib().ugache_host_tier_rows(ctypes.byref(plan), num_rows))


def fill_host_tier(cfg: ugache_config, order: np.ndarray, plan: ugache_plan, table, tier):
    """Host-only: tier[t] = table[order[(band_end + t) mod N]] for t < N (ugache_fill_host_tier)."""
    order = np.ascontiguousarray(order, dtype=np.uint64)
    check(lib().ugache_fill_host_tier(ctypes.byref(cfg), _ptr(order), ctypes.byref(plan),
                                      _ptr(table), _ptr(tier)), "ugache_fill_host_tier")


def solve(cfg: ugache_config, hotness: Optional[np.ndarray], want_order: bool = True):
    """Host-only placement solve (ugache_solve).  Returns (plan, order or None)."""
    plan = ugache_plan()
    order = np.empty(cfg.num_rows, dtype=np.uint64) if want_order else None
    h = None if hotness is None else np.ascontiguousarray(hotness, dtype=np.float32)
    check(lib().ugache_solve(ctypes.byref(cfg), _ptr(h), _ptr(order), ctypes.byref(plan)),
          "ugache_solve")
    return plan, order


def build_placement(cfg: ugache_config, order: np.ndarray, plan: ugache_plan, gpu: int):
    """Host-only: (loc[N] uint64, slot_keys[n_slots] uint64) of GPU ``gpu``."""
    loc = np.empty(cfg.num_rows, dtype=np.uint64)
    slots = np.empty(max(plan.capacity_rows, 1), dtype=np.uint64)
    ns = ctypes.c_uint64()
    order = np.ascontiguousarray(order, dtype=np.uint64)
    check(lib().ugache_build_placement(ctypes.byref(cfg), _ptr(order), ctypes.byref(plan), gpu,
                                       _ptr(loc), _ptr(slots), ctypes.byref(ns)),
          "ugache_build_placement")
    return loc, slots[: ns.value].copy()


class UGache:
    """One GPU's UGache context (one per process per GPU)."""

    def __init__(self, table, num_rows: int, row_bytes: int, capacity_rows: int,
                 hotness: Optional[np.ndarray] = None, num_gpus: int = 1, rank: int = 0,
                 device: int = 0, policy: str = "ugache", plan: Optional[ugache_plan] = None,
                 order: Optional[np.ndarray] = None, host_tier=False, placement=None, **model):
        """host_tier: False; True (the ctx builds its own rank-ordered host tier); or a
        host buffer already filled by :func:`fill_host_tier` (shared by ranks).
        placement: optional (loc[N] uint64, slot_keys uint64) of this GPU computed elsewhere
        (ugache_init_with_placement), e.g. by :mod:`.milp_solver`."""
        self._table = table  # keep the host buffers alive for the ctx's lifetime
        self._tier = host_tier if not isinstance(host_tier, bool) else None
        self.cfg = make_config(num_rows, row_bytes, capacity_rows, num_gpus, rank, device,
                               policy, host_tier=host_tier is not False, **model)
        self.ctx = ctypes.c_void_p()
        if placement is not None:
            loc = np.ascontiguousarray(placement[0], dtype=np.uint64)
            sk = np.ascontiguousarray(placement[1], dtype=np.uint64)
            st = lib().ugache_init_with_placement(ctypes.byref(self.ctx), ctypes.byref(self.cfg),
                                                  _ptr(table), _ptr(loc), _ptr(sk), len(sk))
        elif plan is not None and order is not None:
            order = np.ascontiguousarray(order, dtype=np.uint64)
            st = lib().ugache_init_with_plan(ctypes.byref(self.ctx), ctypes.byref(self.cfg),
                                             _ptr(table), _ptr(order), ctypes.byref(plan),
                                             _ptr(self._tier))
        else:
            h = None if hotness is None else np.ascontiguousarray(hotness, dtype=np.float32)
            st = lib().ugache_init(ctypes.byref(self.ctx), ctypes.byref(self.cfg), _ptr(table),
                                   _ptr(h))
        if st != _abi.UGACHE_OK:
            m = lib().ugache_last_error_message(None)
            raise _abi.UGacheError(st, "ugache_init", m.decode() if m else "")
        self.num_gpus, self.rank = num_gpus, rank
        self.row_bytes = row_bytes
        self.num_rows = num_rows

    # -- setup ------------------------------------------------------------------------
    @property
    def plan(self) -> ugache_plan:
        p = ugache_plan()
        check(lib().ugache_get_plan(self.ctx, ctypes.byref(p)), "ugache_get_plan", self.ctx)
        return p

    def slab(self):
        ptr, nbytes, ns = ctypes.c_void_p(), ctypes.c_uint64(), ctypes.c_uint64()
        check(lib().ugache_slab(self.ctx, ctypes.byref(ptr), ctypes.byref(nbytes), ctypes.byref(ns)),
              "ugache_slab", self.ctx)
        return ptr.value, nbytes.value, ns.value

    def ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(128)
        n = ctypes.c_size_t(128)
        check(lib().ugache_ipc_handle(self.ctx, buf, ctypes.byref(n)), "ugache_ipc_handle", self.ctx)
        return buf.raw[: n.value]

    def open_peers(self, handles: Sequence[bytes]):
        each = max(len(h) for h in handles)
        blob = b"".join(h.ljust(each, b"\0") for h in handles)
        check(lib().ugache_open_peers(self.ctx, blob, each), "ugache_open_peers", self.ctx)

    def set_peer_slabs(self, slabs: Sequence[int]):
        arr = (ctypes.c_void_p * len(slabs))(*[ctypes.c_void_p(s) for s in slabs])
        check(lib().ugache_set_peer_slabs(self.ctx, arr), "ugache_set_peer_slabs", self.ctx)

    def fill(self, stream=None):
        check(lib().ugache_fill(self.ctx, _stream_handle(stream)), "ugache_fill", self.ctx)

    # -- cache refresh (ugache_refresh_*) ------------------------------------
    def refresh_begin(self, loc: np.ndarray, slot_keys: np.ndarray, stream=None):
        loc = np.ascontiguousarray(loc, dtype=np.uint64)
        sk = np.ascontiguousarray(slot_keys, dtype=np.uint64)
        check(lib().ugache_refresh_begin(self.ctx, _ptr(loc), _ptr(sk), len(sk), _stream_handle(stream)),
              "ugache_refresh_begin", self.ctx)

    def refresh_content(self, max_sms: int = 0, max_rows: int = 0, stream=None) -> int:
        """One content step; returns the number of changed slots still to rewrite."""
        rem = ctypes.c_uint64()
        check(lib().ugache_refresh_content(self.ctx, max_sms, max_rows, ctypes.byref(rem),
                                           _stream_handle(stream)), "ugache_refresh_content", self.ctx)
        return int(rem.value)

    def refresh_stage(self, loc: np.ndarray, slot_keys: np.ndarray, stream=None):
        """Chunked refresh: stage the new placement (ugache_refresh_stage)."""
        loc = np.ascontiguousarray(loc, dtype=np.uint64)
        sk = np.ascontiguousarray(slot_keys, dtype=np.uint64)
        check(lib().ugache_refresh_stage(self.ctx, _ptr(loc), _ptr(sk), len(sk), _stream_handle(stream)),
              "ugache_refresh_stage", self.ctx)

    def refresh_chunk(self, step: str, lo: int, hi: int, max_sms: int = 0, stream=None):
        """One step ('evict', 'fill', 'install') of the chunked refresh on slots [lo, hi)."""
        st = {"evict": _abi.REFRESH_EVICT, "fill": _abi.REFRESH_FILL, "install": _abi.REFRESH_INSTALL}[step]
        check(lib().ugache_refresh_chunk(self.ctx, st, lo, hi, max_sms, _stream_handle(stream)),
              "ugache_refresh_chunk", self.ctx)

    def refresh_commit(self, stream=None):
        check(lib().ugache_refresh_commit(self.ctx, _stream_handle(stream)), "ugache_refresh_commit",
              self.ctx)

    def calibrate(self, sample_rows: int = 0) -> dict:
        """A0 calibration through this ctx's sources (ugache_calibrate): bandwidth vs SMs for
        the host and the peers, local gather bandwidth, and the recommended SM counts.  Call
        on every rank at once for the contention of all G readers."""
        c = _abi.ugache_calibration()
        check(lib().ugache_calibrate(self.ctx, sample_rows, ctypes.byref(c)), "ugache_calibrate", self.ctx)
        return {"host_sms": c.host_sms, "peer_sms": c.peer_sms, "bw_local": c.bw_local,
                "bw_peer": c.bw_peer, "bw_host": c.bw_host, "sample_rows": c.sample_rows,
                "host_curve": [(c.host_points_sms[i], c.host_points_bw[i]) for i in range(c.n_host_points)],
                "peer_curve": [(c.peer_points_sms[i], c.peer_points_bw[i]) for i in range(c.n_peer_points)]}

    def set_dedication(self, host_sms: int = 0, peer_sms: int = 0):
        check(lib().ugache_set_dedication(self.ctx, host_sms, peer_sms), "ugache_set_dedication", self.ctx)

    def set_mode(self, mode: str):
        m = {"factored": _abi.MODE_FACTORED, "random": _abi.MODE_RANDOM_DISPATCH}[mode]
        check(lib().ugache_set_mode(self.ctx, m), "ugache_set_mode", self.ctx)

    def set_option(self, option: int, value: int):
        check(lib().ugache_set_option(self.ctx, option, int(value)), "ugache_set_option", self.ctx)

    def set_host_ordering(self, on: bool):
        self.set_option(_abi.OPT_HOST_ORDERING, int(on))

    def set_dedication_mode(self, mode: str, host_warps: int = 0, peer_warps: int = 0):
        """'sms' (whole SMs per source, the paper's) or 'warps' (warps per source on every SM)."""
        self.set_option(_abi.OPT_DEDICATION,
                        {"sms": _abi.DEDICATE_SMS, "warps": _abi.DEDICATE_WARPS}[mode])
        if host_warps:
            self.set_option(_abi.OPT_WARP_HOST, host_warps)
        if peer_warps:
            self.set_option(_abi.OPT_WARP_PEER, peer_warps)

    def set_early_walk(self, on: bool):
        """Fused launch: CTAs without a locate tile walk for host rows before the barrier."""
        self.set_option(_abi.OPT_EARLY_WALK, int(on))

    def set_local_bulk(self, mode):
        """Local rows by TMA bulk copies: False/0 never, True/1 always, 2 auto (default:
        unless the host bucket is dense), 3 on CTAs without a host role."""
        self.set_option(_abi.OPT_LOCAL_BULK, int(mode))

    def set_fused(self, mode):
        """'off' (two launches), 'on' (one cooperative launch) or 'auto'."""
        self.set_option(_abi.OPT_FUSED, {"off": 0, "on": 1, "auto": 2}[mode])

    def set_stream(self, mode):
        """Single-pass extraction: 'off', 'on' or 'auto' (default: unless the previous
        batch's host bucket was dense)."""
        self.set_option(_abi.OPT_STREAM, {"off": 0, "on": 1, "auto": 2}[mode])

    def set_inline(self, host: bool = True, peers: bool = False):
        """Single pass: which non-local sources the locating warps copy themselves."""
        self.set_option(_abi.OPT_INLINE, (_abi.INLINE_HOST if host else 0) |
                        (_abi.INLINE_PEERS if peers else 0))

    def set_host_walk(self, on: bool):
        self.set_option(_abi.OPT_HOST_WALK, int(on))

    def set_preorder(self, on: bool = True):
        """UGACHE_OPT_PREORDER: host range histogram built while locating, host bucket ordered
        by every CTA (default on)."""
        self.set_option(_abi.OPT_PREORDER, int(on))

    def set_stage_host_io(self, on: bool):
        self.set_option(_abi.OPT_STAGE_HOST_IO, int(on))

    def enable_timing(self, on: bool = True):
        check(lib().ugache_enable_timing(self.ctx, int(on)), "ugache_enable_timing", self.ctx)

    # -- hot path ---------------------------------------------------------------------
    def extract(self, keys, out=None, stream=None):
        """out[i] = table[keys[i]] (ugache_extract).  ``keys``: torch int64/int32 tensor
        (device or host) or numpy array; ``out``: tensor/array of n*R bytes or None (a
        uint8 device tensor [n, R] is allocated on the current device)."""
        import torch
        if isinstance(keys, np.ndarray):
            kt = _abi.KEY_U32 if keys.dtype == np.uint32 else _abi.KEY_I64
            if kt == _abi.KEY_I64 and keys.dtype != np.int64:
                raise TypeError("keys must be int64 or uint32")
            n = len(keys)
        else:
            if keys.dtype == torch.int64:
                kt = _abi.KEY_I64
            elif keys.dtype in (torch.int32, torch.uint32):
                kt = _abi.KEY_U32
            else:
                raise TypeError("keys must be int64 or (u)int32")
            if not keys.is_contiguous():
                raise ValueError("keys must be contiguous")
            n = keys.numel()
        if out is None:
            out = torch.empty((n, self.row_bytes), dtype=torch.uint8,
                              device=keys.device if hasattr(keys, "device") and keys.is_cuda else "cuda")
        nbytes = out.nbytes if isinstance(out, np.ndarray) else out.numel() * out.element_size()
        if nbytes < n * self.row_bytes:
            raise ValueError(f"out holds {nbytes} bytes < n * row_bytes = {n * self.row_bytes}")
        check(lib().ugache_extract(self.ctx, _ptr(keys), kt, n, _ptr(out), _stream_handle(stream)),
              "ugache_extract", self.ctx)
        return out

    # -- introspection ----------------------------------------------------------------
    def last_batch_stats(self):
        per = np.zeros(self.num_gpus + 1, dtype=np.uint64)
        bad = ctypes.c_uint64()
        check(lib().ugache_last_batch_stats(self.ctx, _ptr(per), ctypes.byref(bad)),
              "ugache_last_batch_stats", self.ctx)
        return per.astype(np.int64), int(bad.value)

    def last_batch_timing(self):
        a, b = ctypes.c_float(), ctypes.c_float()
        check(lib().ugache_last_batch_timing(self.ctx, ctypes.byref(a), ctypes.byref(b)),
              "ugache_last_batch_timing", self.ctx)
        return a.value, b.value

    def last_launch_count(self) -> int:
        n = ctypes.c_int32()
        check(lib().ugache_last_launch_count(self.ctx, ctypes.byref(n)), "ugache_last_launch_count",
              self.ctx)
        return n.value

    def last_batch_phases(self):
        """(locate done, host ordered, host copies done, last CTA located, launch end) in ms
        from the fused kernel's start (ugache_last_batch_phases)."""
        ms = (ctypes.c_float * 5)()
        check(lib().ugache_last_batch_phases(self.ctx, ms), "ugache_last_batch_phases", self.ctx)
        return tuple(float(x) for x in ms)

    def last_batch_timeline(self):
        """Per-CTA role timeline of the last fused launch (ugache_last_batch_timeline): an
        (SM count, 5) float array of [role source, CTA start, gather start, role done, CTA
        done], ms from the kernel's start.  Needs enable_timing(True)."""
        buf = (ctypes.c_float * (5 * 256))()
        n = ctypes.c_int32()
        check(lib().ugache_last_batch_timeline(self.ctx, buf, ctypes.byref(n)), "ugache_last_batch_timeline",
              self.ctx)
        return np.frombuffer(buf, dtype=np.float32, count=5 * n.value).reshape(n.value, 5).copy()

    def last_extract_path(self) -> str:
        """'split', 'fused', 'single_pass', 'random' or 'none' (ugache_last_extract_path)."""
        p = ctypes.c_int32()
        check(lib().ugache_last_extract_path(self.ctx, ctypes.byref(p)), "ugache_last_extract_path",
              self.ctx)
        return _abi.PATHS[p.value]

    def export_placement(self):
        loc = np.empty(self.num_rows, dtype=np.uint64)
        slots = np.empty(max(self.plan.capacity_rows, 1), dtype=np.uint64)
        ns = ctypes.c_uint64()
        check(lib().ugache_export_placement(self.ctx, _ptr(loc), _ptr(slots), ctypes.byref(ns)),
              "ugache_export_placement", self.ctx)
        return loc, slots[: ns.value].copy()

    def read_slab(self, first: int, count: int) -> np.ndarray:
        dst = np.empty((count, self.row_bytes), dtype=np.uint8)
        check(lib().ugache_read_slab(self.ctx, first, count, _ptr(dst)), "ugache_read_slab", self.ctx)
        return dst

    def close(self):
        if self.ctx:
            lib().ugache_destroy(self.ctx)
            self.ctx = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def connect_in_process(group: List[UGache]):
    """Fake-peer / single-process multi-GPU wiring: every ctx maps the others' slabs
    directly (same device, or peer access between devices)."""
    slabs = [g.slab()[0] for g in group]
    for g in group:
        if len(group) > 1:
            g.set_peer_slabs(slabs)
