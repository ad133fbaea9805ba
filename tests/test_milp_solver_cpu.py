"""CPU tests of the block-level MILP solver (paper_conf_sosp_songz0c23_b200/milp_solver.py,
section 6.3): block construction rules, agreement with the entry-level MILP oracle when
blocks are single entries, and consistency of the produced placement with the oracle's
section 6.2 model and placement checker."""
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
    peer = (148 - host_sms) // max(G - 1, 1) if G > 1 else 0
    return Platform(G=G, row_bytes=512, host_sms=host_sms, peer_sms=peer, **B200)


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
