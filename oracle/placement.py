"""oracle.placement -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Plain fp64 numpy restatement of UGache's cache policy family and of its extraction-time
model, written to be checked against PAPER.md by eye (P:n = PAPER.md line n).

Location-table encoding (the ABI convention of include/ugache.h, restated here):
``loc = (src << 56) | row`` with ``src = j`` for GPU j (j == own rank: local) and
``src = G`` for host DRAM, where ``row = key`` (the host holds every entry).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Tuple

import numpy as np

SRC_SHIFT = np.uint64(56)
ROW_MASK = np.uint64((1 << 56) - 1)


def enc(src, row):
    return (np.uint64(src) << SRC_SHIFT) | np.asarray(row, dtype=np.uint64)


def dec(loc):
    loc = np.asarray(loc, dtype=np.uint64)
    return (loc >> SRC_SHIFT).astype(np.int64), (loc & ROW_MASK).astype(np.int64)


# ----------------------------------------------------------------------------- platform
@dataclass
class Platform:
    """Profiled platform parameters of Table 2, B200 reading (R11).

    T_{i<-j}: "time of reading one embedding from source j to GPU i", "the reciprocal of
    bandwidth".  R_{i<-j}: "ratio of GPU_i's core to extract from j"
    (P:1393-1394).  Local: T = R/BW_L, ratio 1 (local padding may use every core,
    P:1096-1103).  Peer: each remote GPU gets 1/(G-1) of the NVLink bandwidth
    (P:1227-1230), ratio peer_sms/S.  Host: T = R/BW_H, ratio host_sms/S."""
    G: int
    row_bytes: int
    bw_local: float
    bw_peer: float
    bw_host: float
    host_sms: int
    peer_sms: int
    num_sms: int = 148

    def T(self) -> Tuple[float, float, float]:
        tl = self.row_bytes / self.bw_local
        tp = self.row_bytes / (self.bw_peer / max(self.G - 1, 1))
        th = self.row_bytes / self.bw_host
        return tl, tp, th

    def ratios(self) -> Tuple[float, float, float]:
        return 1.0, self.peer_sms / self.num_sms, self.host_sms / self.num_sms

    def T_row(self, i: int) -> np.ndarray:
        """T_{i<-j} for j = 0..G (j == G is host)."""
        tl, tp, th = self.T()
        t = np.full(self.G + 1, tp)
        t[i] = tl
        t[self.G] = th
        return t

    def R_row(self, i: int) -> np.ndarray:
        rl, rp, rh = self.ratios()
        r = np.full(self.G + 1, rp)
        r[i] = rl
        r[self.G] = rh
        return r


# ----------------------------------------------------------------------------- order
def rank_order(h: Optional[np.ndarray], N: int) -> np.ndarray:
    """Entries sorted by decreasing hotness, ties by increasing key (R7).
    Hotness is the application-provided access frequency; values <= 0
    (including -0.0) count as 0.  Returns order[rank] = key."""
    keys = np.arange(N, dtype=np.int64)
    if h is None:
        return keys
    hh = np.maximum(np.asarray(h, dtype=np.float64), 0.0)
    return np.lexsort((keys, -hh)).astype(np.int64)


# ----------------------------------------------------------------------------- policies
def policy_placement(order: np.ndarray, N: int, C: int, G: int, k: int, host_tier: bool = False):
    """Hot-replicate / warm-partition placement with replicated prefix length k.

    * ranks [0, k): on every GPU ("every GPU caches the hottest entries", replication,
      P:385-394), slot = rank;
    * ranks [k, band_end): "evenly partition the hottest entries among each GPU"
       -- round-robin by rank: owner (r-k) mod G, slot k + (r-k) div G;
    * the rest: host DRAM (fallback location).
    k = C is replication, k = 0 is partition, 0 < k < C is the hot-replicate /
    warm-partition family of ref [39].

    host_tier (R24): the host rows live in a copy ordered by hotness rank, so a
    host entry's row is its tier slot ``rank - band_end`` instead of its key.

    Returns (loc[G, N] uint64, slot_keys: list of G uint64 arrays)."""
    C = min(C, N)
    assert 0 <= k <= C
    order = np.asarray(order, dtype=np.int64)
    band_end = min(N, k + G * (C - k))
    band = np.arange(k, band_end, dtype=np.int64)
    owner = (band - k) % G
    slot = k + (band - k) // G
    loc = np.empty((G, N), dtype=np.uint64)
    slot_keys: List[np.ndarray] = []
    for g in range(G):
        lg = enc(G, np.arange(N))                       # default: host, row = key
        if host_tier:                                   # host row = tier slot
            lg[order[band_end:]] = enc(G, np.arange(N - band_end))
        lg[order[:k]] = enc(g, np.arange(k))            # replicated prefix, slot = rank
        lg[order[band]] = (owner.astype(np.uint64) << SRC_SHIFT) | slot.astype(np.uint64)
        loc[g] = lg
        mine = order[band][owner == g]                  # slots k, k+1, ... in rank order
        slot_keys.append(np.concatenate([order[:k], mine]).astype(np.uint64))
    return loc, slot_keys


# ----------------------------------------------------------------------------- model
def model_times(h: np.ndarray, loc: np.ndarray, plat: Platform):
    """Section 6.2 extraction-time model, literally, in fp64.

    The access arrangement a^e_{i<-j} is the location table: a^e_{i<-j} = 1 iff
    LT_i[e].src == j (each GPU reads each entry from exactly one source).
      t^j_i = sum_e T_{i<-j} * h_e * a^e_{i<-j}
      t_i  >= t^j_i  for all j in M;   t_i >= sum_j t^j_i * R_{i<-j}
      z    >= t_i
    Returns (z, t[G], tj[G, G+1])."""
    G = loc.shape[0]
    hh = np.maximum(np.asarray(h, dtype=np.float64), 0.0)
    tj = np.zeros((G, G + 1))
    t = np.zeros(G)
    for i in range(G):
        src, _ = dec(loc[i])
        Ti = plat.T_row(i)
        Ri = plat.R_row(i)
        for j in range(G + 1):
            tj[i, j] = Ti[j] * float(np.sum(hh[src == j]))
        t[i] = max(float(np.max(tj[i])), float(np.sum(tj[i] * Ri)))
    return float(np.max(t)), t, tj


def sweep_z(h: np.ndarray, order: np.ndarray, N: int, C: int, plat: Platform, k: int) -> float:
    loc, _ = policy_placement(order, N, C, plat.G, k)
    return model_times(h, loc, plat)[0]


def solve_sweep(h: np.ndarray, N: int, C: int, plat: Platform):
    """Brute force: evaluate the model for every k in [0, min(C, N)] and return the k of
    minimal z (ties -> larger k, i.e. more local hits; R21).  For G = 1 every k
    gives the same placement; k = C is returned."""
    order = rank_order(h, N)
    Cc = min(C, N)
    if plat.G == 1:
        return Cc, sweep_z(h, order, N, C, plat, Cc)
    best_k, best_z = None, None
    for k in range(Cc, -1, -1):
        z = sweep_z(h, order, N, C, plat, k)
        if best_z is None or z < best_z * (1 - 1e-12):
            best_k, best_z = k, z
    return best_k, best_z


# ----------------------------------------------------------------------------- checker
def check_placement(loc: np.ndarray, slot_keys: List[np.ndarray], N: int, C: int,
                    tier_keys: Optional[np.ndarray] = None, local_preference: bool = True):
    """Placement invariants (SURVEY.md section 8(c) checker items 1-4); raises AssertionError.

    1. resolution: LT_g[k] = (host, k) [or (host, t) with tier_keys[t] == k for a host
       tier] or (GPU j, slot) with slot < n_slots_j and
       slot_keys_j[slot] == k  ("Each cached embedding entry is associated with its source
       location in the format of <GPU_i, Offset>");
    2. capacity: n_slots_j <= C  (sum_e s^e_j <= Cap_j);
    3. storage covers access (s^e_j >= a^e_{i<-j}) -- implied by 1;
    4. local preference: an entry stored on g is read locally by g (the replicate/partition
       family's arrangement; the section 6.2 MILP may choose otherwise, so callers checking
       a MILP placement pass local_preference=False), and no GPU stores an entry twice."""
    G = loc.shape[0]
    for j in range(G):
        assert len(slot_keys[j]) <= C, f"GPU {j}: {len(slot_keys[j])} slots > capacity {C}"
        sk = np.asarray(slot_keys[j], dtype=np.int64)
        assert np.all((sk >= 0) & (sk < N)), f"GPU {j}: slot key out of range"
        assert len(np.unique(sk)) == len(sk), f"GPU {j}: entry stored twice"
    for g in range(G):
        src, row = dec(loc[g])
        keys = np.arange(N)
        assert np.all((src >= 0) & (src <= G)), f"GPU {g}: bad source id"
        host = src == G
        if tier_keys is None:
            assert np.all(row[host] == keys[host]), f"GPU {g}: host row != key"
        else:  # host tier: tier slot row holds the key
            tk = np.asarray(tier_keys, dtype=np.int64)
            assert np.all(row[host] < len(tk)), f"GPU {g}: host tier slot out of range"
            assert np.all(tk[row[host]] == keys[host]), f"GPU {g}: host tier slot holds another key"
        for j in range(G):
            m = src == j
            sk = np.asarray(slot_keys[j], dtype=np.int64)
            assert np.all(row[m] < len(sk)), f"GPU {g}: slot beyond GPU {j}'s filled slots"
            assert np.all(sk[row[m]] == keys[m]), f"GPU {g}: GPU {j} slot holds another key"
        if local_preference:
            own = np.asarray(slot_keys[g], dtype=np.int64)
            assert np.all(src[own] == g), f"GPU {g}: locally stored entry not read locally"
            assert np.all(row[own] == np.arange(len(own))), f"GPU {g}: local slot mismatch"


def source_counts(loc_g: np.ndarray, keys: np.ndarray, N: int, G: int) -> Tuple[np.ndarray, int]:
    """Per-source key counts of one batch on one GPU (per-source rates of Fig. 14,
    P:2744-2748): counts[j] for GPU j (own rank = local), counts[G] = host; plus the
    number of out-of-range keys."""
    keys = np.asarray(keys, dtype=np.int64)
    valid = (keys >= 0) & (keys < N)
    src, _ = dec(loc_g[keys[valid]])
    return np.bincount(src, minlength=G + 1).astype(np.int64), int(np.sum(~valid))
