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
    Returns (s[G, B] bool, a[G, G+1, B] bool, z seconds, status message).

    The model is assembled block-major with numpy index arrays: every constraint family is
    one vectorised batch of rows of a COO matrix.  Column layout, with M = G + 1 sources
    (source G = host) and times in units of T_local for conditioning:

      s[b, j]      B*G    binary   block b stored on GPU j
      a[b, i, j]   B*G*M  binary   GPU i reads block b from source j
      u[i, j]      G*M    >= 0     t^j_i, modeled time of GPU i's reads from j
      t[i]         G      >= 0     t_i
      z            1      >= 0     objective
    """
    import scipy.sparse as sp
    from scipy.optimize import Bounds, LinearConstraint, milp

    B, M = len(blocks), G + 1
    hs = np.maximum(np.asarray(h_sorted, dtype=np.float64), 0.0)
    cum = np.concatenate([[0.0], np.cumsum(hs)])
    lo_r = np.array([a for a, _ in blocks], dtype=np.int64)
    hi_r = np.array([b for _, b in blocks], dtype=np.int64)
    mass = cum[hi_r] - cum[lo_r]                       # H_b: hotness mass of block b
    size = (hi_r - lo_r).astype(np.float64)            # n_b: entries of block b
    unit = T[0] if T[0] > 0 else 1.0
    # T[i, j] and R[i, j]: peer everywhere, local on the diagonal, host in the last column
    Tm = np.full((G, M), T[1] / unit)
    Rm = np.full((G, M), float(Rr[1]))
    Tm[np.arange(G), np.arange(G)] = T[0] / unit
    Rm[np.arange(G), np.arange(G)] = Rr[0]
    Tm[:, G] = T[2] / unit
    Rm[:, G] = Rr[2]

    n_s, n_a, n_u = B * G, B * G * M, G * M
    S = np.arange(n_s).reshape(B, G)
    A = n_s + np.arange(n_a).reshape(B, G, M)
    U = n_s + n_a + np.arange(n_u).reshape(G, M)
    Tt = n_s + n_a + n_u + np.arange(G)
    Z = n_s + n_a + n_u + G
    nv = Z + 1

    rows, cols, vals, lo, hi = [], [], [], [], []
    nrow = 0

    def family(r_idx, c_idx, v, l, u, count):
        """count constraint rows; entry k sits in row r_idx[k] (relative) at column c_idx[k]."""
        nonlocal nrow
        rows.append(np.asarray(r_idx, dtype=np.int64).ravel() + nrow)
        cols.append(np.asarray(c_idx, dtype=np.int64).ravel())
        vals.append(np.broadcast_to(np.asarray(v, dtype=np.float64), np.shape(c_idx)).ravel())
        lo.append(np.broadcast_to(np.float64(l), (count,)))
        hi.append(np.broadcast_to(np.float64(u), (count,)))
        nrow += count

    # every GPU reads every block from exactly one source:  sum_j a[b,i,j] = 1
    r = np.broadcast_to(np.arange(B * G).reshape(B, G, 1), (B, G, M))
    family(r, A, 1.0, 1.0, 1.0, B * G)
    # a GPU source must store what is read from it:  s[b,j] - a[b,i,j] >= 0  (j < G)
    r = np.arange(B * G * G).reshape(B, G, G)
    family(np.stack([r, r], -1), np.stack([np.broadcast_to(S[:, None, :], (B, G, G)), A[:, :, :G]], -1),
           np.array([1.0, -1.0]), 0.0, np.inf, B * G * G)
    # capacity, counted in entries (block sizes):  sum_b n_b s[b,j] <= C
    family(np.broadcast_to(np.arange(G), (B, G)), S, np.broadcast_to(size[:, None], (B, G)),
           -np.inf, float(C), G)
    # u[i,j] = T[i,j] * sum_b H_b a[b,i,j]
    r_u = np.arange(G * M).reshape(G, M)
    family(np.concatenate([r_u.ravel(), np.broadcast_to(r_u, (B, G, M)).ravel()]),
           np.concatenate([U.ravel(), A.ravel()]),
           np.concatenate([np.ones(G * M), (-Tm[None, :, :] * mass[:, None, None]).ravel()]),
           0.0, 0.0, G * M)
    # t_i >= u[i,j]
    family(np.stack([r_u, r_u], -1), np.stack([np.broadcast_to(Tt[:, None], (G, M)), U], -1),
           np.array([1.0, -1.0]), 0.0, np.inf, G * M)
    # t_i >= sum_j R[i,j] u[i,j]
    family(np.concatenate([np.arange(G), np.repeat(np.arange(G), M)]),
           np.concatenate([Tt, U.ravel()]), np.concatenate([np.ones(G), -Rm.ravel()]),
           0.0, np.inf, G)
    # z >= t_i
    family(np.stack([np.arange(G)] * 2, -1), np.stack([np.full(G, Z), Tt], -1),
           np.array([1.0, -1.0]), 0.0, np.inf, G)

    Am = sp.coo_array((np.concatenate(vals), (np.concatenate(rows), np.concatenate(cols))),
                      shape=(nrow, nv)).tocsr()
    c = np.zeros(nv)
    c[Z] = 1.0
    binary = np.zeros(nv)
    binary[: n_s + n_a] = 1
    ub = np.full(nv, np.inf)
    ub[: n_s + n_a] = 1.0
    res = milp(c, integrality=binary, bounds=Bounds(np.zeros(nv), ub),
               constraints=LinearConstraint(Am, np.concatenate(lo), np.concatenate(hi)),
               options=dict(time_limit=time_limit, disp=False, mip_rel_gap=1e-6))
    if res.x is None:
        raise RuntimeError(f"block MILP failed: {res.message}")
    x = res.x
    s_out = (x[S] > 0.5).T                              # [G, B]
    a_out = np.transpose(x[A] > 0.5, (1, 2, 0))         # [G, M, B]
    return s_out, a_out, float(x[Z]) * unit, res.message


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
