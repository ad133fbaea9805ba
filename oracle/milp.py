"""oracle.milp -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The section 6.2 MILP of PAPER.md written out verbatim and solved with scipy's HiGHS on
tiny instances.  It is the exact reference against which the library's placement search
is compared (the paper solves it with Gurobi; Gurobi is not available).

Variables (Table 2), with M = GPUs + host:
  a^e_{i<-j}  binary,  i in G, j in M, e in E
  s^e_j       binary,  j in G (the host stores every entry; no s for host, R10)
  t^j_i       continuous, i in G, j in M
  t_i         continuous, i in G
  z           continuous
Constraints:
  sum_j a^e_{i<-j} = 1                      for all i, e
  s^e_j >= a^e_{i<-j}                       for all i, j in G, e
  sum_e s^e_j <= Cap_j                      for all j in G
  t^j_i = sum_e T_{i<-j} h_e a^e_{i<-j}     for all i, j in M
  t_i >= t^j_i                              for all i, j in M
  t_i >= sum_j t^j_i R_{i<-j}               for all i
  minimize z, z >= t_i                      for all i
Counts: E G^2 + 2EG + G^2 + 2G + 1 variables, E G^2 + EG + 2G^2 + 5G constraints
 -- asserted by tests/test_oracle_placement.py.
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp
from scipy.optimize import Bounds, LinearConstraint, milp

from .placement import Platform


def build(h: np.ndarray, cap: int, plat: Platform):
    """Returns (c, integrality, bounds, constraints, index helpers, scale)."""
    E = len(h)
    G = plat.G
    M = G + 1
    h = np.maximum(np.asarray(h, dtype=np.float64), 0.0)
    scale = plat.T()[0]  # express times in units of T_local for conditioning

    ia = lambda i, j, e: (i * M + j) * E + e
    na = G * M * E
    is_ = lambda j, e: na + j * E + e
    ns = G * E
    itj = lambda i, j: na + ns + i * M + j
    ntj = G * M
    it = lambda i: na + ns + ntj + i
    iz = na + ns + ntj + G
    nvar = iz + 1

    rows, cols, vals, lo, hi = [], [], [], [], []
    r = 0

    def add(entries, l, u):
        nonlocal r
        for c_, v in entries:
            rows.append(r)
            cols.append(c_)
            vals.append(v)
        lo.append(l)
        hi.append(u)
        r += 1

    for i in range(G):                       # sum_j a = 1
        for e in range(E):
            add([(ia(i, j, e), 1.0) for j in range(M)], 1.0, 1.0)
    for i in range(G):                       # s >= a  (GPU sources only)
        for j in range(G):
            for e in range(E):
                add([(is_(j, e), 1.0), (ia(i, j, e), -1.0)], 0.0, np.inf)
    for j in range(G):                       # capacity
        add([(is_(j, e), 1.0) for e in range(E)], -np.inf, float(cap))
    for i in range(G):                       # t^j_i definition
        Ti = plat.T_row(i) / scale
        for j in range(M):
            add([(itj(i, j), 1.0)] + [(ia(i, j, e), -Ti[j] * h[e]) for e in range(E)], 0.0, 0.0)
    for i in range(G):                       # t_i >= t^j_i
        for j in range(M):
            add([(it(i), 1.0), (itj(i, j), -1.0)], 0.0, np.inf)
    for i in range(G):                       # t_i >= sum_j R t^j_i
        Ri = plat.R_row(i)
        add([(it(i), 1.0)] + [(itj(i, j), -Ri[j]) for j in range(M)], 0.0, np.inf)
    for i in range(G):                       # z >= t_i
        add([(iz, 1.0), (it(i), -1.0)], 0.0, np.inf)

    A = sp.csr_array((vals, (rows, cols)), shape=(r, nvar))
    c = np.zeros(nvar)
    c[iz] = 1.0
    integrality = np.zeros(nvar)
    integrality[: na + ns] = 1
    lb = np.zeros(nvar)
    ub = np.full(nvar, np.inf)
    ub[: na + ns] = 1.0
    idx = dict(ia=ia, is_=is_, itj=itj, it=it, iz=iz, E=E, G=G, M=M)
    return c, integrality, Bounds(lb, ub), LinearConstraint(A, lo, hi), idx, scale


def size(E: int, G: int, cap: int = 1):
    """(number of variables, number of constraints) of the model as built."""
    plat = Platform(G=G, row_bytes=512, bw_local=1.0, bw_peer=1.0, bw_host=1.0,
                    host_sms=1, peer_sms=1, num_sms=4)
    c, _, _, cons, _, _ = build(np.ones(E), cap, plat)
    return len(c), cons.A.shape[0]


def solve(h: np.ndarray, cap: int, plat: Platform, time_limit: float = 60.0):
    """Exact (or time-limited incumbent) optimum of the section 6.2 MILP.

    Returns dict(z=seconds, status, s[G,E] bool, a[G,M,E] bool, mip_gap)."""
    c, integ, bounds, cons, idx, scale = build(h, cap, plat)
    res = milp(c, integrality=integ, bounds=bounds, constraints=cons,
               options=dict(time_limit=time_limit, disp=False, mip_rel_gap=1e-9))
    if res.x is None:
        raise RuntimeError(f"MILP failed: {res.message}")
    E, G, M = idx["E"], idx["G"], idx["M"]
    x = res.x
    s = np.array([[x[idx["is_"](j, e)] > 0.5 for e in range(E)] for j in range(G)])
    a = np.array([[[x[idx["ia"](i, j, e)] > 0.5 for e in range(E)] for j in range(M)]
                  for i in range(G)])
    return dict(z=float(x[idx["iz"]]) * scale, status=res.status, s=s, a=a,
                mip_gap=getattr(res, "mip_gap", None), message=res.message)
