"""synth -- seeded synthetic workload generators (INPUTS only; none of the method's arithmetic).

This is the one module both sides share: the CPU oracle under
``oracle/`` and the product path (``bench.py``, GPU tests) draw the same tables, key batches
and hotness from here.  It never locates, buckets, places or gathers anything.

Recipe (PAPER.md lines cited as P:n):

* Table: N x R bytes, row-major, self-describing words (``synth/table_gen.c``):
  ``word(k, w) = lo32(splitmix64(seed ^ (k*R/4 + w)))``.
* Skew: bounded Zipf(alpha) over ranks 1..N_t, ``P(r) ~ r^-alpha`` -- "Zipfian-generated
  (alpha = 1.2)", SYN-A/B "power-law ... alpha=1.2 and 1.4".
* Rank -> key bijection per table t: ``key = off_t + ((a_t*(r-1) + b_t) mod N_t)`` with
  ``a_t`` the first odd number >= 0x9E3779B1 coprime to N_t and ``b_t = t*0x632BE5AB mod N_t``,
  so hot rows are scattered over the key space.
* Batches (data parallel: each GPU draws its own batch):
  - ``iid``   : n i.i.d. Zipf keys with duplicates (tiny config);
  - ``unique``: i.i.d. draws until ``n_unique`` distinct keys, then shuffled (GNN: sampled
    k-hop neighbourhoods are unique vertex sets);
  - ``dlr``   : ``samples`` requests, one Zipf key per table each, laid out sample-major
    ``keys[s*T + t]`` ("Each request contains a single key for each table").
* Hotness (application-provided access frequency, global over GPUs):
  expected accesses per GPU per batch -- ``n*p(r)`` for iid/dlr, ``1-(1-p(r))^m`` for
  unique batches (m = draws needed, i.e. the probability an entry is in a batch).
"""
from __future__ import annotations

import ctypes
import math
import mmap
import os
import zlib
from dataclasses import dataclass, field, replace
from typing import List, Optional, Tuple

import numpy as np

TABLE_SEED = 0x55474143  # "UGAC"
_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib_path() -> str:
    return os.path.join(_HERE, "libsynth.so")


def build(force: bool = False) -> str:
    """Compile synth/table_gen.c -> synth/libsynth.so (gcc, OpenMP)."""
    src = os.path.join(_HERE, "table_gen.c")
    out = lib_path()
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(src):
        import subprocess
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", out, src])
    return out


def _lib():
    global _LIB
    if _LIB is None:
        build()
        L = ctypes.CDLL(lib_path())
        L.synth_fill_table.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                                       ctypes.c_uint32, ctypes.c_uint64]
        L.synth_fill_table.restype = None
        L.synth_rows_for_keys.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                          ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64]
        L.synth_rows_for_keys.restype = None
        _LIB = L
    return _LIB


# ----------------------------------------------------------------------------- workloads
@dataclass(frozen=True)
class Workload:
    """One synthetic workload shape (BASELINE.json ``configs``)."""
    name: str
    table_rows: Tuple[int, ...]      # rows per embedding table (N = sum)
    row_bytes: int                   # R
    alpha: float                     # Zipf exponent
    batch_kind: str                  # "iid" | "unique" | "dlr"
    batch_n: int                     # iid: keys; unique: distinct keys; dlr: samples
    num_gpus: int = 1
    cache_ratio: float = 0.10        # per-GPU capacity C = cache_ratio * N
    dtype: str = "f32"               # element type of the table (only names the row layout)
    note: str = ""

    @property
    def num_rows(self) -> int:
        return int(sum(self.table_rows))

    @property
    def num_tables(self) -> int:
        return len(self.table_rows)

    @property
    def capacity_rows(self) -> int:
        return int(round(self.cache_ratio * self.num_rows))

    @property
    def keys_per_batch(self) -> int:
        if self.batch_kind == "dlr":
            return self.batch_n * self.num_tables
        return self.batch_n

    @property
    def table_bytes(self) -> int:
        return self.num_rows * self.row_bytes

    def scaled(self, rows_scale: float) -> "Workload":
        rows = tuple(max(1, int(r * rows_scale)) for r in self.table_rows)
        if self.batch_kind == "unique":
            n = min(self.batch_n, max(1, sum(rows) // 20))
        else:
            n = self.batch_n
        return replace(self, table_rows=rows, batch_n=n,
                       name=f"{self.name}@{rows_scale:g}",
                       note=(self.note + f" rows scaled x{rows_scale:g}").strip())


WORKLOADS = {
    # BASELINE.json configs[0]: 100K x 128 fp32, Zipf(1.2), 8K batch, 2 GPUs, 10 % cache.
    "tiny": Workload("tiny", (100_000,), 512, 1.2, "iid", 8192, num_gpus=2, cache_ratio=0.10),
    # configs[1]: Papers100M-shaped 111M x 128 fp32, ~500K unique keys per batch.
    "gnn_pa": Workload("gnn_pa", (111_000_000,), 512, 1.2, "unique", 500_000, num_gpus=8,
                       cache_ratio=0.10),
    # configs[2]: Criteo-TB-shaped, 26 tables x 30,769,231 rows x 128 fp32, 8192 x 26 keys.
    "dlr_criteo": Workload("dlr_criteo", (30_769_231,) * 26, 512, 1.2, "dlr", 8192, num_gpus=8,
                           cache_ratio=0.10),
    # configs[3]: MAG240M-shaped 244M x 768 fp16 (1536 B rows), ~500K unique keys.
    "gnn_mag": Workload("gnn_mag", (244_000_000,), 1536, 1.2, "unique", 500_000, num_gpus=8,
                        cache_ratio=0.10, dtype="f16"),
}


def get_workload(name: str) -> Workload:
    """``name`` or ``name@scale`` (rows scaled, e.g. ``dlr_criteo@0.15``)."""
    if "@" in name:
        base, s = name.split("@", 1)
        return WORKLOADS[base].scaled(float(s))
    return WORKLOADS[name]


# ----------------------------------------------------------------------------- skew
def zipf_pmf(num: int, alpha: float) -> np.ndarray:
    """P(r) for r = 1..num of the bounded Zipf(alpha), float64."""
    w = np.arange(1, num + 1, dtype=np.float64) ** (-alpha)
    return w / w.sum()


_CDF_CACHE: dict = {}


def zipf_cdf(num: int, alpha: float) -> np.ndarray:
    key = (num, alpha)
    if key not in _CDF_CACHE:
        if len(_CDF_CACHE) > 2:
            _CDF_CACHE.clear()
        c = np.cumsum(zipf_pmf(num, alpha))
        c[-1] = 1.0
        _CDF_CACHE[key] = c
    return _CDF_CACHE[key]


def sample_ranks(rng: np.random.Generator, num: int, alpha: float, m: int) -> np.ndarray:
    """m i.i.d. Zipf ranks (0-based: rank r-1) by inverse CDF.  Queries are sorted before
    the binary search for cache locality and the original draw order restored."""
    cdf = zipf_cdf(num, alpha)
    u = rng.random(m)
    order = np.argsort(u, kind="stable")
    r = np.empty(m, dtype=np.int64)
    r[order] = np.searchsorted(cdf, u[order], side="right")
    np.minimum(r, num - 1, out=r)
    return r


def bijection_params(num: int, table_idx: int) -> Tuple[int, int]:
    a = 0x9E3779B1
    if a % 2 == 0:
        a += 1
    while math.gcd(a, num) != 1:
        a += 2
    b = (table_idx * 0x632BE5AB) % num
    return a, b


def rank_to_key(ranks0: np.ndarray, num: int, table_idx: int = 0, offset: int = 0) -> np.ndarray:
    """0-based ranks -> keys for table ``table_idx`` with ``num`` rows at ``offset``."""
    a, b = bijection_params(num, table_idx)
    r = ranks0.astype(np.uint64)
    k = (np.uint64(a % num) * (r % np.uint64(num)) + np.uint64(b)) % np.uint64(num)
    return (k + np.uint64(offset)).astype(np.int64)


def key_to_rank(keys: np.ndarray, num: int, table_idx: int = 0, offset: int = 0) -> np.ndarray:
    """Inverse of :func:`rank_to_key` (0-based ranks)."""
    a, b = bijection_params(num, table_idx)
    ainv = pow(a % num, -1, num) if num > 1 else 0
    k = (keys.astype(np.int64) - offset).astype(np.uint64)
    d = (k + np.uint64(num) - np.uint64(b)) % np.uint64(num)
    # (d * ainv) mod num without overflow: split ainv
    lo = np.uint64(ainv & 0xFFFF)
    hi = np.uint64(ainv >> 16)
    n = np.uint64(num)
    r = ((d * hi) % n * np.uint64(1 << 16) % n + d * lo % n) % n
    return r.astype(np.int64)


def table_offsets(wl: Workload) -> np.ndarray:
    return np.concatenate([[0], np.cumsum(wl.table_rows)[:-1]]).astype(np.int64)


def batch_seed(wl: Workload, rank: int, batch_idx: int) -> np.random.SeedSequence:
    return np.random.SeedSequence([zlib.crc32(wl.name.encode()), int(rank), int(batch_idx)])


def make_batch(wl: Workload, rank: int, batch_idx: int, return_draws: bool = False):
    """The int64 key batch GPU ``rank`` extracts at step ``batch_idx``."""
    rng = np.random.Generator(np.random.PCG64(batch_seed(wl, rank, batch_idx)))
    offs = table_offsets(wl)
    if wl.batch_kind == "iid":
        ranks = sample_ranks(rng, wl.table_rows[0], wl.alpha, wl.batch_n)
        keys = rank_to_key(ranks, wl.table_rows[0])
        return (keys, wl.batch_n) if return_draws else keys
    if wl.batch_kind == "dlr":
        T = wl.num_tables
        keys = np.empty((wl.batch_n, T), dtype=np.int64)
        for t in range(T):
            ranks = sample_ranks(rng, wl.table_rows[t], wl.alpha, wl.batch_n)
            keys[:, t] = rank_to_key(ranks, wl.table_rows[t], t, int(offs[t]))
        keys = keys.reshape(-1)
        return (keys, wl.batch_n) if return_draws else keys
    if wl.batch_kind == "unique":
        N = wl.table_rows[0]
        target = wl.batch_n
        seen = np.zeros(N, dtype=bool)
        picked: List[np.ndarray] = []
        have = 0
        draws = 0
        chunk = max(4096, target)
        while have < target:
            r = sample_ranks(rng, N, wl.alpha, chunk)
            # first occurrences (in draw order) of ranks not seen before
            uniq, first = np.unique(r, return_index=True)
            fresh = ~seen[uniq]
            uniq, first = uniq[fresh], first[fresh]
            order = np.argsort(first, kind="stable")
            uniq, first = uniq[order], first[order]
            need = target - have
            if len(uniq) >= need:
                uniq = uniq[:need]
                draws += int(first[need - 1]) + 1
            else:
                draws += chunk
            seen[uniq] = True
            picked.append(uniq)
            have += len(uniq)
        ranks = np.concatenate(picked)
        rng.shuffle(ranks)
        keys = rank_to_key(ranks, N)
        return (keys, draws) if return_draws else keys
    raise ValueError(wl.batch_kind)


def expected_draws_unique(num: int, alpha: float, target: int) -> float:
    """m such that sum_r 1-(1-p(r))^m = target.  f(m) is increasing and concave, so
    Newton's method started at m = target approaches the root monotonically from below."""
    if target >= num:
        raise ValueError("target unique count must be < number of rows")
    lp = np.log1p(-zipf_pmf(num, alpha))
    m = float(target)
    for _ in range(100):
        e = np.exp(m * lp)
        f = float(np.sum(1.0 - e)) - target
        df = float(-np.dot(lp, e))
        step = -f / df
        m += step
        if abs(step) <= 1e-9 * m:
            break
    return m


def hotness(wl: Workload, m_unique: Optional[float] = None) -> np.ndarray:
    """float32 hotness h[key] (expected accesses of the entry per GPU per batch)."""
    N = wl.num_rows
    h = np.empty(N, dtype=np.float32)
    offs = table_offsets(wl)
    for t, Nt in enumerate(wl.table_rows):
        p = zipf_pmf(Nt, wl.alpha)
        if wl.batch_kind == "unique":
            m = m_unique if m_unique is not None else expected_draws_unique(Nt, wl.alpha, wl.batch_n)
            hr = -np.expm1(m * np.log1p(-p))
        else:
            hr = wl.batch_n * p
        keys = rank_to_key(np.arange(Nt, dtype=np.int64), Nt, t, int(offs[t]))
        h[keys] = hr.astype(np.float32)
    return h


# ----------------------------------------------------------------------------- tables
class HostTable:
    """A host-resident N x R table (anonymous mmap, or a /dev/shm file shared by ranks).

    The library pins it with ``cudaHostRegister`` inside ``ugache_init``; this class only
    owns the mapping.  (torch's pinned allocator rounds sizes to powers of two, so it is
    not used for the table -- SURVEY.md section 7.3.)"""

    def __init__(self, num_rows: int, row_bytes: int, shm_path: Optional[str] = None,
                 create: bool = True):
        self.num_rows = int(num_rows)
        self.row_bytes = int(row_bytes)
        self.nbytes = self.num_rows * self.row_bytes
        self.shm_path = shm_path
        self._fd = None
        size = max(self.nbytes, 1)
        if shm_path is None:
            self._mm = mmap.mmap(-1, size, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
        else:
            flags = os.O_RDWR | (os.O_CREAT if create else 0)
            self._fd = os.open(shm_path, flags, 0o600)
            if create:
                os.ftruncate(self._fd, size)
            self._mm = mmap.mmap(self._fd, size, flags=mmap.MAP_SHARED)
        try:
            self._mm.madvise(mmap.MADV_HUGEPAGE)
        except Exception:
            pass
        self.array = np.frombuffer(self._mm, dtype=np.uint8, count=self.nbytes).reshape(
            self.num_rows, self.row_bytes)

    @property
    def ptr(self) -> int:
        return self.array.ctypes.data if self.nbytes else 0

    def fill(self, row_begin: int = 0, row_end: Optional[int] = None, seed: int = TABLE_SEED):
        row_end = self.num_rows if row_end is None else row_end
        if row_end <= row_begin:
            return
        _lib().synth_fill_table(ctypes.c_void_p(self.ptr + row_begin * self.row_bytes),
                                row_begin, row_end, self.row_bytes // 4, seed)

    def close(self):
        self.array = None
        try:
            self._mm.close()
        except BufferError:
            pass
        if self._fd is not None:
            os.close(self._fd)
            self._fd = None


class AliasedHostTable:
    """An N-row table whose virtual span is full size but whose physical memory is only the
    first ``phys_rows`` rows: one memfd of phys_rows * R bytes mapped repeatedly at adjacent
    addresses (MAP_FIXED inside one reserved range), so row k holds the generator's row
    ``k mod phys_rows``.  Used to run full-size DLR / MAG key spaces (375-410 GB) on a box
    with less RAM: the device sees the full host address span (translation footprint), and
    the oracle reads the same buffer, so parity is unaffected.  Same interface as HostTable
    (``ptr``, ``array`` over the whole span, ``fill``, ``close``)."""

    def __init__(self, num_rows: int, row_bytes: int, phys_rows: int):
        libc = ctypes.CDLL(None, use_errno=True)
        libc.mmap.restype = ctypes.c_void_p
        libc.mmap.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_int,
                              ctypes.c_int, ctypes.c_long]
        libc.munmap.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
        self._libc = libc
        self.num_rows, self.row_bytes = int(num_rows), int(row_bytes)
        gran = 4096  # rows: phys_rows * R stays a multiple of 2 MB for 512-B multiples
        self.phys_rows = max(gran, min(self.num_rows, (int(phys_rows) // gran) * gran))
        self.nbytes = self.num_rows * self.row_bytes
        self.phys_bytes = self.phys_rows * self.row_bytes
        self.copies = -(-self.num_rows // self.phys_rows)
        self.shm_path = None
        self._fd = os.memfd_create("ugache_aliased_table")
        os.ftruncate(self._fd, self.phys_bytes)
        PROT_NONE, PROT_RW = 0, 3
        MAP_SHARED, MAP_PRIVATE, MAP_FIXED, MAP_ANON, MAP_NORESERVE = 0x01, 0x02, 0x10, 0x20, 0x4000
        total = self.copies * self.phys_bytes
        base = libc.mmap(None, total, PROT_NONE, MAP_PRIVATE | MAP_ANON | MAP_NORESERVE, -1, 0)
        if base in (None, ctypes.c_void_p(-1).value):
            raise OSError(ctypes.get_errno(), "reserving the aliased table span failed")
        self._base, self._total = base, total
        for i in range(self.copies):
            at = libc.mmap(base + i * self.phys_bytes, self.phys_bytes, PROT_RW,
                           MAP_SHARED | MAP_FIXED, self._fd, 0)
            if at != base + i * self.phys_bytes:
                raise OSError(ctypes.get_errno(), f"mapping alias copy {i} failed")
        buf = (ctypes.c_uint8 * self.nbytes).from_address(base)
        self.array = np.frombuffer(buf, dtype=np.uint8, count=self.nbytes).reshape(self.num_rows, self.row_bytes)

    @property
    def ptr(self) -> int:
        return int(self._base)

    def fill(self, seed: int = TABLE_SEED):
        """Generator rows 0..phys_rows-1 (every alias copy sees them)."""
        _lib().synth_fill_table(ctypes.c_void_p(self._base), 0, self.phys_rows, self.row_bytes // 4, seed)

    def close(self):
        self.array = None
        if self._base:
            self._libc.munmap(ctypes.c_void_p(self._base), self._total)
            self._base = 0
        if self._fd is not None:
            os.close(self._fd)
            self._fd = None


def make_table(num_rows: int, row_bytes: int, seed: int = TABLE_SEED) -> HostTable:
    t = HostTable(num_rows, row_bytes)
    t.fill(seed=seed)
    return t


def rows_for_keys(keys: np.ndarray, num_rows: int, row_bytes: int,
                  seed: int = TABLE_SEED) -> np.ndarray:
    """Re-derive table[keys] (zero rows for out-of-range keys) from the generator alone."""
    keys = np.ascontiguousarray(keys, dtype=np.int64)
    out = np.empty((len(keys), row_bytes), dtype=np.uint8)
    if len(keys):
        _lib().synth_rows_for_keys(out.ctypes.data, keys.ctypes.data, len(keys), num_rows,
                                   row_bytes // 4, seed)
    return out


def rows_for_keys_numpy(keys: np.ndarray, num_rows: int, row_bytes: int,
                        seed: int = TABLE_SEED) -> np.ndarray:
    """Pure-numpy second implementation of the generator (tests cross-check the C one)."""
    W = row_bytes // 4
    keys = np.asarray(keys, dtype=np.int64)
    valid = (keys >= 0) & (keys < num_rows)
    k = np.where(valid, keys, 0).astype(np.uint64)
    x = np.uint64(seed) ^ (k[:, None] * np.uint64(W) + np.arange(W, dtype=np.uint64)[None, :])
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    w = (z & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    w[~valid] = 0
    return w.view(np.uint8).reshape(len(keys), row_bytes)
