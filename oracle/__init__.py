"""oracle -- plain, slow, obviously-correct CPU implementation of UGache's extraction path.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import, call, link or execute anything
under ``oracle/``.  It shares no code with the CUDA path (``paper_conf_sosp_songz0c23_b200``)
and neither imports the other; both draw inputs from ``synth/`` only.

Contents (each function cites the PAPER.md passage it follows; ``P:n`` = line n):

* ``gather.c`` / :func:`gather`     -- out[i] = table[keys[i]]
* ``placement.py``                  -- rank order, replication / partition / hot-replicate
  warm-partition placements, the section 6.2 extraction-time model
   evaluated literally in fp64, the brute-force sweep over the replicated
  prefix, and the placement checker (resolution, capacity, local preference).
* ``milp.py``                       -- the section 6.2 MILP verbatim (scipy/HiGHS), used only on
  tiny instances as an exact reference and to pin the reading of every term through the
  paper's size formula.

Pins (tests/test_oracle_*.py): generator re-derivation of every gathered row, numpy fancy
indexing, brute force over all storage choices on tiny instances, the MILP optimum, the
MILP size formula, closed-form Zipf coverage.  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib_path() -> str:
    return os.path.join(_HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile oracle/gather.c -> oracle/liboracle.so (plain gcc -O2, OpenMP)."""
    src = os.path.join(_HERE, "gather.c")
    out = lib_path()
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", out, src])
    return out


def _lib():
    global _LIB
    if _LIB is None:
        build()
        L = ctypes.CDLL(lib_path())
        for name in ("oracle_gather_i64", "oracle_gather_u32"):
            f = getattr(L, name)
            f.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p,
                          ctypes.c_uint64, ctypes.c_void_p]
            f.restype = ctypes.c_int64
        _LIB = L
    return _LIB


def gather(table_ptr: int, num_rows: int, row_bytes: int, keys: np.ndarray,
           out: np.ndarray | None = None):
    """CPU oracle of ugache_extract: returns (out[n, R] uint8, number of out-of-range keys).

    ``table_ptr`` is the address of the N x R host table (the same buffer the GPU path
    reads).  P:266-269 / P:597-615 / P:626-627."""
    if keys.dtype == np.uint32:
        fn = _lib().oracle_gather_u32
    else:
        keys = np.ascontiguousarray(keys, dtype=np.int64)
        fn = _lib().oracle_gather_i64
    keys = np.ascontiguousarray(keys)
    n = len(keys)
    if out is None:
        out = np.empty((n, row_bytes), dtype=np.uint8)
    bad = fn(table_ptr, num_rows, row_bytes, keys.ctypes.data, n, out.ctypes.data) if n else 0
    return out, int(bad)
