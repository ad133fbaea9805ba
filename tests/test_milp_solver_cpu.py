"""CPU tests of the block-level MILP solver (paper_conf_sosp_songz0c23_b200/milp_solver.py,
section 6.3): block construction rules; the solver's optimum against an independent
brute-force enumeration of block placements (multi-entry blocks, size-weighted capacity);
agreement with the entry-level MILP oracle when blocks are single entries; and consistency
of the produced placement with the oracle's section 6.2 model and placement checker."""
import itertools
import math

import numpy as np
import pytest

import synth
from oracle import milp
from oracle.placement import Platform, check_placement, model_times, rank_order, sweep_z
from paper_conf_sosp_songz0c23_b200 import make_config, solve
from paper_conf_sosp_songz0c23_b200.milp_solver import make_blocks, placement_from_blocks, solve_blocks

B200 = dict(bw_local=6457.7e9, bw_peer=770e9, bw_host=34.4e9)


def _plat(G, host_sms=8):
    """The platform of make_config(..., host_sms=host_sms) with the library's default SMs per
    peer (R14), so oracle and product evaluate the same model."""
    plan, _ = solve(make_config(1000, 512, 100, num_gpus=G, host_sms=host_sms, bw_host=34.4e9), None,
                    want_order=False)
    return Platform(G=G, row_bytes=512, host_sms=host_sms, peer_sms=int(plan.peer_sms), **B200)


@pytest.mark.parametrize("E,G", [(1000, 4), (20_000, 8), (50, 2)])
def test_block_rules(E, G):
    h = np.sort((synth.zipf_pmf(E, 1.2) * 1e5).astype(np.float32))[::-1]
    blocks = make_blocks(h, G)
    assert blocks[0][0] == 0 and blocks[-1][1] == E
    assert all(a[1] == b[0] for a, b in zip(blocks, blocks[1:]))
    lvl = np.floor(np.log2(h.astype(np.float64)))
    cap = max(1, math.ceil(0.005 * E))
    per_level = {}
    for b0, b1 in blocks:
        assert len(set(lvl[b0:b1])) == 1                  # one hotness level per block
        assert b1 - b0 <= cap                             # <= 0.5 % of entries
        per_level.setdefault(lvl[b0], []).append(b1 - b0)
    for L, sizes in per_level.items():
        if sum(sizes) >= G:
            assert len(sizes) >= G                        # each level split into >= G blocks


def _T_R(cfg):
    plan, _ = solve(cfg, None)
    return (plan.T_local, plan.T_peer, plan.T_host), (plan.R_local, plan.R_peer, plan.R_host)


def test_single_entry_blocks_equal_entry_milp():
    """With E small every block is one entry, so the block MILP is the section 6.2 MILP."""
    G, E, C = 2, 12, 3
    h = np.sort((synth.zipf_pmf(E, 1.2) * 1000).astype(np.float32))[::-1].copy()
    blocks = make_blocks(h, G)
    assert all(b1 - b0 == 1 for b0, b1 in blocks)
    cfg = make_config(E, 512, C, num_gpus=G, host_sms=8, bw_host=34.4e9)
    T, Rr = _T_R(cfg)
    s, a, z, _ = solve_blocks(h, blocks, C, G, T, Rr)
    ref = milp.solve(h, C, _plat(G))
    assert abs(z - ref["z"]) <= 1e-6 * ref["z"]


@pytest.mark.parametrize("G,E,C", [(2, 400, 40), (4, 1500, 60), (4, 3000, 400)])
def test_block_placement_is_valid_and_matches_model(G, E, C):
    rng = np.random.default_rng(E)
    h = (synth.zipf_pmf(E, 1.2) * 5e4).astype(np.float32)[rng.permutation(E)]
    cfg = make_config(E, 512, C, num_gpus=G, host_sms=8, bw_host=34.4e9)
    T, Rr = _T_R(cfg)
    order = rank_order(h, E)
    hs = h[order]
    blocks = make_blocks(hs, G)
    s, a, z, msg = solve_blocks(hs, blocks, C, G, T, Rr, time_limit=60)
    locs, sks = placement_from_blocks(order, blocks, s, a, E, G)
    check_placement(np.stack(locs), sks, E, C, local_preference=False)
    zm, _, _ = model_times(h, np.stack(locs), _plat(G))
    assert abs(zm - z) <= 1e-6 * z                         # MILP objective = model of placement
    z_rep = sweep_z(h, order, E, C, _plat(G), min(C, E))
    z_part = sweep_z(h, order, E, C, _plat(G), 0)
    # block granularity can cost a little against entry-level policies (paper: < 2 %)
    assert z <= min(z_rep, z_part) * 1.02


def _block_brute_force(mass, size, C, G, T, Rr):
    """Exact optimum of the block model by enumeration, independent of any MILP: every
    storage choice (a subset of blocks per GPU, sum of its block sizes <= C), and for each
    GPU every access arrangement over the sources that hold the block (or the host).  Per
    block b and GPU i the sources are 0..G-1 (GPU j; j == i local) and G (host); a GPU's time
    is max(max_j t^j_i, sum_j R_{i<-j} t^j_i) with t^j_i = T_{i<-j} * (mass read from j)
    (P:1359-1385), and z = max over GPUs.  Returns (z, storage masks)."""
    B = len(mass)
    srcs = G + 1
    acc = np.array(list(itertools.product(range(srcs), repeat=B)), dtype=np.int64)  # [K, B]
    bits = 1 << np.arange(B)
    need = np.stack([((acc == j) * bits).sum(axis=1) for j in range(G)], axis=1)    # [K, G]
    t_gpu = []
    for i in range(G):
        Ti = np.array([T[0] if j == i else (T[2] if j == G else T[1]) for j in range(srcs)])
        Ri = np.array([Rr[0] if j == i else (Rr[2] if j == G else Rr[1]) for j in range(srcs)])
        per_src = np.stack([((acc == j) * mass).sum(axis=1) * Ti[j] for j in range(srcs)], axis=1)
        t_gpu.append(np.maximum(per_src.max(axis=1), per_src @ Ri))                # [K]
    sizes = np.array([sum(size[b] for b in range(B) if m >> b & 1) for m in range(1 << B)])
    fits = [m for m in range(1 << B) if sizes[m] <= C]
    best, arg = np.inf, None
    for stores in itertools.product(fits, repeat=G):
        st = np.array(stores)
        ok = (need & ~st[None, :]) == 0                                            # [K, G]
        feasible = ok.all(axis=1)
        z = max(t_gpu[i][feasible].min() for i in range(G))
        if z < best:
            best, arg = z, stores
    return best, arg


@pytest.mark.parametrize("G,sizes,C,seed", [
    (2, [3, 1, 2, 4, 2, 5], 6, 0),     # multi-entry blocks, capacity binds mid-block
    (2, [2, 2, 2, 2, 2, 2], 5, 1),
    (2, [1, 4, 1, 3, 2], 4, 2),
    (3, [2, 3, 1, 2], 4, 3),
])
def test_block_milp_equals_brute_force(G, sizes, C, seed):
    """Independent pin of solve_blocks (not derived from oracle/milp.py): on multi-entry blocks
    its objective equals the exact optimum found by enumerating every block storage (size-
    weighted capacity) and access arrangement, and its own storage/access realise that value
    under the oracle's entry-level model (oracle.placement.model_times)."""
    rng = np.random.default_rng(seed)
    E = int(sum(sizes))
    blocks, b0 = [], 0
    for sz in sizes:
        blocks.append((b0, b0 + sz))
        b0 += sz
    h = np.sort(rng.pareto(1.2, E).astype(np.float32) + 0.05)[::-1].copy()   # sorted hotness
    plat = Platform(G=G, row_bytes=512, host_sms=8, peer_sms=(148 - 8) // (G - 1), **B200)
    T, Rr = plat.T(), plat.ratios()
    mass = np.array([h[a:b].astype(np.float64).sum() for a, b in blocks])
    z_bf, _ = _block_brute_force(mass, np.array(sizes), C, G, T, Rr)
    s, a, z, _ = solve_blocks(h, blocks, C, G, T, Rr)
    assert abs(z - z_bf) <= 1e-6 * z_bf, (z, z_bf)
    assert all(sum(sizes[b] for b in range(len(sizes)) if s[j, b]) <= C for j in range(G))
    order = np.arange(E)                                # h is already in rank order
    locs, sks = placement_from_blocks(order, blocks, s, a, E, G)
    check_placement(np.stack(locs), sks, E, C, local_preference=False)
    zm, _, _ = model_times(h, np.stack(locs), plat)
    assert abs(zm - z) <= 1e-6 * z
