"""Paper-faithful block-level cache-policy solver (section 6.3) -- host side.

UGache batches entries of similar hotness into blocks and solves the section 6.2 MILP at
block granularity (the paper uses Gurobi; here scipy's HiGHS):

* hotness levels on a log scale: level(e) = floor(log2 h_e);
* block size: at most 0.5 % of all entries, and every level is split into at least G
  blocks -- reading R25: block size = max(1, min(floor(level_size / G),
  ceil(0.005 * E)));
* per block b (size n_b, hotness mass H_b): binary storage s^b_j (j in GPUs) and access
  a^b_{i<-j} (j in GPUs + host); capacity sum_b n_b s^b_j <= Cap_j (footnote 2: "the
  size each block needs to be added"); t^j_i = T_{i<-j} sum_b H_b a^b_{i<-j};
  t_i >= t^j_i, t_i >= sum_j R_{i<-j} t^j_i; minimise z >= t_i.

Unlike the hot-replicate / warm-partition family that ugache_init searches, the block
solution may replicate a block on any subset of GPUs.  The result is turned into per-GPU
location tables and slot lists for ``ugache_init_with_placement``.  Platform parameters
(T, R) are taken from a ``ugache_plan`` so both solvers use the same model.
"""
from __future__ import annotations

import math
from typing import List, Tuple

import numpy as np

SRC_SHIFT = 56


def make_blocks(h_sorted: np.ndarray, G: int, max_frac: float = 0.005) -> List[Tuple[int, int]]:
    """Rank ranges [start, end) of the blocks over hotness sorted in decreasing order."""
    E = len(h_sorted)
    hs = np.maximum(np.asarray(h_sorted, dtype=np.float64), 0.0)
    with np.errstate(divide="ignore"):
        lvl = np.where(hs > 0, np.floor(np.log2(np.where(hs > 0, hs, 1.0))), -np.inf)
    cap = max(1, int(math.ceil(max_frac * E)))
    blocks = []
    start = 0
    while start < E:
        end = start
        while end < E and lvl[end] == lvl[start]:
            end += 1
        size = end - start
        bsz = max(1, min(size // G, cap))  # >= G blocks per level, <= 0.5 % of E each
        for b0 in range(start, end, bsz):
            blocks.append((b0, min(end, b0 + bsz)))
        start = end
    return blocks


def solve_blocks(h_sorted: np.ndarray, blocks, C: int, G: int, T, Rr, time_limit: float = 60.0):
    """Block MILP.  T = (T_local, T_peer, T_host), Rr = (R_local, R_peer, R_host).
    Returns (s[G, B] bool, a[G, G+1, B] bool, z seconds, status message)."""
    import scipy.sparse as sp
    from scipy.optimize import Bounds, LinearConstraint, milp

    B = len(blocks)
    M = G + 1
    hs = np.maximum(np.asarray(h_sorted, dtype=np.float64), 0.0)
    mass = np.array([hs[a:b].sum() for a, b in blocks])
    size = np.array([b - a for a, b in blocks], dtype=np.float64)
    scale = T[0] if T[0] > 0 else 1.0

    def Trow(i):
        t = np.full(M, T[1]) / scale
        t[i] = T[0] / scale
        t[G] = T[2] / scale
        return t

    def Rrow(i):
        r = np.full(M, Rr[1])
        r[i] = Rr[0]
        r[G] = Rr[2]
        return r

    ia = lambda i, j, b: (i * M + j) * B + b
    na = G * M * B
    is_ = lambda j, b: na + j * B + b
    ns = G * B
    itj = lambda i, j: na + ns + i * M + j
    it = lambda i: na + ns + G * M + i
    iz = na + ns + G * M + G
    nv = iz + 1
    rows, cols, vals, lo, hi = [], [], [], [], []
    r = [0]

    def add(ent, l, u):
        for c, v in ent:
            rows.append(r[0])
            cols.append(c)
            vals.append(v)
        lo.append(l)
        hi.append(u)
        r[0] += 1

    for i in range(G):
        for b in range(B):
            add([(ia(i, j, b), 1.0) for j in range(M)], 1.0, 1.0)
    for i in range(G):
        for j in range(G):
            for b in range(B):
                add([(is_(j, b), 1.0), (ia(i, j, b), -1.0)], 0.0, np.inf)
    for j in range(G):
        add([(is_(j, b), size[b]) for b in range(B)], -np.inf, float(C))
    for i in range(G):
        Ti = Trow(i)
        for j in range(M):
            add([(itj(i, j), 1.0)] + [(ia(i, j, b), -Ti[j] * mass[b]) for b in range(B)], 0.0, 0.0)
    for i in range(G):
        for j in range(M):
            add([(it(i), 1.0), (itj(i, j), -1.0)], 0.0, np.inf)
        Ri = Rrow(i)
        add([(it(i), 1.0)] + [(itj(i, j), -Ri[j]) for j in range(M)], 0.0, np.inf)
        add([(iz, 1.0), (it(i), -1.0)], 0.0, np.inf)
    A = sp.csr_array((vals, (rows, cols)), shape=(r[0], nv))
    c = np.zeros(nv)
    c[iz] = 1.0
    integ = np.zeros(nv)
    integ[: na + ns] = 1
    ub = np.full(nv, np.inf)
    ub[: na + ns] = 1.0
    res = milp(c, integrality=integ, bounds=Bounds(np.zeros(nv), ub),
               constraints=LinearConstraint(A, lo, hi),
               options=dict(time_limit=time_limit, disp=False, mip_rel_gap=1e-6))
    if res.x is None:
        raise RuntimeError(f"block MILP failed: {res.message}")
    x = res.x
    s = np.array([[x[is_(j, b)] > 0.5 for b in range(B)] for j in range(G)])
    a = np.array([[[x[ia(i, j, b)] > 0.5 for b in range(B)] for j in range(M)] for i in range(G)])
    return s, a, float(x[iz]) * scale, res.message


def placement_from_blocks(order: np.ndarray, blocks, s: np.ndarray, a: np.ndarray, N: int, G: int):
    """Per-GPU (loc[N] uint64, slot_keys) from a block solution.  Blocks stored on GPU j
    occupy consecutive slots in block order; GPU i reads block b from exactly the source the
    MILP's access arrangement a^b_{i<-j} chose."""
    order = np.asarray(order, dtype=np.int64)
    slot_keys, slot_of = [], []
    for j in range(G):
        keys, offs, pos = [], {}, 0
        for b, (b0, b1) in enumerate(blocks):
            if s[j, b]:
                offs[b] = pos
                keys.append(order[b0:b1])
                pos += b1 - b0
        slot_keys.append(np.concatenate(keys).astype(np.uint64) if keys else np.zeros(0, np.uint64))
        slot_of.append(offs)
    locs = []
    host = np.uint64(G) << np.uint64(SRC_SHIFT)
    for i in range(G):
        loc = host | np.arange(N, dtype=np.uint64)
        for b, (b0, b1) in enumerate(blocks):
            keys = order[b0:b1]
            chosen = [j for j in range(G + 1) if a[i, j, b]]
            src = chosen[0] if chosen else G
            if src < G and not s[src, b]:
                raise ValueError("access arrangement reads a block its source does not store")
            if src < G:
                rows = slot_of[src][b] + np.arange(b1 - b0, dtype=np.uint64)
                loc[keys] = (np.uint64(src) << np.uint64(SRC_SHIFT)) | rows.astype(np.uint64)
        locs.append(loc)
    return locs, slot_keys
