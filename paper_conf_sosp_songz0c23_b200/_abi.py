"""ctypes binding of libugache.so -- argument marshalling only (include/ugache.h).

Every name below is the C entry point of the same name; no step of the extraction path
runs in Python.  Loading fails loudly when the in-tree library is missing: there is no
CPU fallback for the product path.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libugache.so")

UGACHE_MAX_GPUS = 16
UGACHE_LOC_SRC_SHIFT = 56
UGACHE_LOC_ROW_MASK = (1 << 56) - 1

UGACHE_OK, UGACHE_EINVAL, UGACHE_ECUDA, UGACHE_ENOMEM, UGACHE_ESTATE, UGACHE_EPEER, UGACHE_EKEY = range(7)
STATUS_NAMES = {0: "UGACHE_OK", 1: "UGACHE_EINVAL", 2: "UGACHE_ECUDA", 3: "UGACHE_ENOMEM",
                4: "UGACHE_ESTATE", 5: "UGACHE_EPEER", 6: "UGACHE_EKEY"}
POLICY_UGACHE, POLICY_REPLICATION, POLICY_PARTITION = 0, 1, 2
POLICIES = {"ugache": POLICY_UGACHE, "replication": POLICY_REPLICATION,
            "partition": POLICY_PARTITION}
KEY_I64, KEY_U32 = 0, 1
MODE_FACTORED, MODE_RANDOM_DISPATCH = 0, 1
OPT_HOST_ORDERING, OPT_STAGE_HOST_IO, OPT_HOST_WARPS = 0, 1, 2
OPT_DEDICATION, OPT_WARP_HOST, OPT_WARP_PEER, OPT_HOST_WALK, OPT_FUSED = 3, 4, 5, 6, 7
OPT_LOCAL_BULK, OPT_EARLY_WALK, OPT_STREAM, OPT_INLINE, OPT_PREORDER = 8, 9, 10, 11, 12
INLINE_HOST, INLINE_PEERS = 1, 2
REFRESH_EVICT, REFRESH_FILL, REFRESH_INSTALL = 0, 1, 2
PATHS = {0: "none", 1: "split", 2: "fused", 3: "single_pass", 4: "random"}
DEDICATE_SMS, DEDICATE_WARPS = 0, 1
FLAG_HOST_TIER = 1


class ugache_config(ctypes.Structure):
    _fields_ = [("num_rows", ctypes.c_uint64), ("row_bytes", ctypes.c_uint32),
                ("reserved0", ctypes.c_uint32), ("capacity_rows", ctypes.c_uint64),
                ("num_gpus", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("device", ctypes.c_int32), ("policy", ctypes.c_int32),
                ("bw_local", ctypes.c_double), ("bw_peer", ctypes.c_double),
                ("bw_host", ctypes.c_double), ("host_sms", ctypes.c_int32),
                ("peer_sms", ctypes.c_int32), ("num_sms", ctypes.c_int32),
                ("flags", ctypes.c_int32)]


class ugache_plan(ctypes.Structure):
    _fields_ = [("policy", ctypes.c_int32), ("num_gpus", ctypes.c_int32),
                ("capacity_rows", ctypes.c_uint64), ("k", ctypes.c_uint64),
                ("band_end", ctypes.c_uint64), ("z", ctypes.c_double),
                ("z_replication", ctypes.c_double), ("z_partition", ctypes.c_double),
                ("T_local", ctypes.c_double), ("T_peer", ctypes.c_double),
                ("T_host", ctypes.c_double), ("R_local", ctypes.c_double),
                ("R_peer", ctypes.c_double), ("R_host", ctypes.c_double),
                ("host_sms", ctypes.c_int32), ("peer_sms", ctypes.c_int32),
                ("num_sms", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("host_mass_frac", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_ if f != "reserved"}


CALIB_MAX_POINTS = 24


class ugache_calibration(ctypes.Structure):
    _fields_ = [("host_sms", ctypes.c_int32), ("peer_sms", ctypes.c_int32),
                ("bw_local", ctypes.c_double), ("bw_peer", ctypes.c_double),
                ("bw_host", ctypes.c_double), ("n_host_points", ctypes.c_int32),
                ("n_peer_points", ctypes.c_int32),
                ("host_points_sms", ctypes.c_int32 * CALIB_MAX_POINTS),
                ("host_points_bw", ctypes.c_double * CALIB_MAX_POINTS),
                ("peer_points_sms", ctypes.c_int32 * CALIB_MAX_POINTS),
                ("peer_points_bw", ctypes.c_double * CALIB_MAX_POINTS),
                ("sample_rows", ctypes.c_uint32), ("reserved", ctypes.c_int32)]


_c = ctypes
_P = ctypes.c_void_p
_ST = ctypes.c_int
# name -> (restype, argtypes); exactly the declarations of include/ugache.h
SIGNATURES = {
    "ugache_solve": (_ST, [ctypes.POINTER(ugache_config), _P, _P, ctypes.POINTER(ugache_plan)]),
    "ugache_build_placement": (_ST, [ctypes.POINTER(ugache_config), _P, ctypes.POINTER(ugache_plan),
                                     _c.c_int32, _P, _P, ctypes.POINTER(_c.c_uint64)]),
    "ugache_init": (_ST, [ctypes.POINTER(_P), ctypes.POINTER(ugache_config), _P, _P]),
    "ugache_init_with_plan": (_ST, [ctypes.POINTER(_P), ctypes.POINTER(ugache_config), _P, _P,
                                    ctypes.POINTER(ugache_plan), _P]),
    "ugache_init_with_placement": (_ST, [ctypes.POINTER(_P), ctypes.POINTER(ugache_config), _P, _P,
                                         _P, _c.c_uint64]),
    "ugache_host_tier_rows":(_c.c_uint64, [ctypes.POINTER(ugache_plan), _c.c_uint64]),
    "ugache_fill_host_tier": (_ST, [ctypes.POINTER(ugache_config), _P, ctypes.POINTER(ugache_plan),
                                    _P, _P]),
    "ugache_get_plan": (_ST, [_P, ctypes.POINTER(ugache_plan)]),
    "ugache_slab": (_ST, [_P, ctypes.POINTER(_P), ctypes.POINTER(_c.c_uint64),
                          ctypes.POINTER(_c.c_uint64)]),
    "ugache_ipc_handle": (_ST, [_P, _P, ctypes.POINTER(_c.c_size_t)]),
    "ugache_open_peers": (_ST, [_P, _P, _c.c_size_t]),
    "ugache_set_peer_slabs": (_ST, [_P, ctypes.POINTER(_P)]),
    "ugache_fill": (_ST, [_P, _P]),
    "ugache_extract": (_ST, [_P, _P, _c.c_int32, _c.c_uint64, _P, _P]),
    "ugache_msg_extract_local": (_ST, [_P, _P, _c.c_int32, _c.c_uint64, _P, _P]),
    "ugache_msg_requests": (_ST, [_P, _P, _P, _P]),
    "ugache_msg_serve": (_ST, [_P, _P, _c.c_uint64, _P, _P]),
    "ugache_msg_scatter": (_ST, [_P, _P, _P, _P]),
    "ugache_refresh_begin": (_ST, [_P, _P, _P, _c.c_uint64, _P]),
    "ugache_refresh_content": (_ST, [_P, _c.c_int32, _c.c_uint64, ctypes.POINTER(_c.c_uint64), _P]),
    "ugache_refresh_commit": (_ST, [_P, _P]),
    "ugache_calibrate": (_ST, [_P, _c.c_uint32, ctypes.POINTER(ugache_calibration)]),
    "ugache_refresh_stage": (_ST, [_P, _P, _P, _c.c_uint64, _P]),
    "ugache_refresh_chunk": (_ST, [_P, _c.c_int32, _c.c_uint64, _c.c_uint64, _c.c_int32, _P]),
    "ugache_model_time": (_ST, [ctypes.POINTER(ugache_plan), _c.c_int32, _c.c_uint64, _P, _P,
                                ctypes.POINTER(_c.c_double)]),
    "ugache_set_dedication": (_ST, [_P, _c.c_int32, _c.c_int32]),
    "ugache_set_mode": (_ST, [_P, _c.c_int32]),
    "ugache_set_option": (_ST, [_P, _c.c_int32, _c.c_int64]),
    "ugache_last_batch_stats": (_ST, [_P, _P, ctypes.POINTER(_c.c_uint64)]),
    "ugache_enable_timing": (_ST, [_P, _c.c_int32]),
    "ugache_last_batch_timing": (_ST, [_P, ctypes.POINTER(_c.c_float), ctypes.POINTER(_c.c_float)]),
    "ugache_last_launch_count": (_ST, [_P, ctypes.POINTER(_c.c_int32)]),
    "ugache_last_extract_path": (_ST, [_P, ctypes.POINTER(_c.c_int32)]),
    "ugache_last_batch_phases": (_ST, [_P, ctypes.POINTER(_c.c_float)]),
    "ugache_last_batch_timeline": (_ST, [_P, ctypes.POINTER(_c.c_float), ctypes.POINTER(_c.c_int32)]),
    "ugache_export_placement": (_ST, [_P, _P, _P, ctypes.POINTER(_c.c_uint64)]),
    "ugache_read_slab": (_ST, [_P, _c.c_uint64, _c.c_uint64, _P]),
    "ugache_destroy": (_ST, [_P]),
    "ugache_error_string": (_c.c_char_p, [_ST]),
    "ugache_last_error_message": (_c.c_char_p, [_P]),
    "ugache_version": (_c.c_int32, []),
}

_lib = None


class UGacheError(RuntimeError):
    def __init__(self, status: int, what: str, detail: str = ""):
        self.status = status
        super().__init__(f"{what} -> {STATUS_NAMES.get(status, status)}"
                         + (f": {detail}" if detail else ""))


def lib():
    """Load the in-tree libugache.so (built by __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; "
                              f"g.build()'` (there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def check(status: int, what: str, ctx=None):
    if status != UGACHE_OK:
        detail = ""
        if ctx is not None:
            m = lib().ugache_last_error_message(ctx)
            detail = m.decode() if m else ""
        raise UGacheError(status, what, detail)


def __getattr__(name):  # ugache_* names resolve to the raw C functions
    if name in SIGNATURES:
        return getattr(lib(), name)
    raise AttributeError(name)
