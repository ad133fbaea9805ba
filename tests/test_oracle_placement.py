"""Pins for the placement / cost-model oracle (oracle/placement.py, oracle/milp.py).

Pinned against: a hand-derived worked example (tests/golden/tiny_policy_example.txt),
hand-computed model values, brute force over every storage choice, the exact MILP, the
paper's MILP size formula, and invariants that any valid placement meets.
"""
import itertools
import os

import numpy as np
import pytest

from oracle import milp
from oracle.placement import (Platform, check_placement, dec, enc, model_times,
                              policy_placement, rank_order, solve_sweep, source_counts,
                              sweep_z)
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
B200 = dict(bw_local=6457.7e9, bw_peer=770e9, bw_host=55.6e9)


def _golden_example():
    stored, locs = {}, []
    with open(os.path.join(GOLDEN, "tiny_policy_example.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            p = line.split()
            if p[0] == "loc":
                locs.append((p[1], int(p[2]), int(p[3]), int(p[4]), int(p[5]), int(p[6])))
            else:
                stored[(p[0], int(p[1]), int(p[2]))] = [int(x) for x in p[3:]]
    return stored, locs


def test_worked_example_policies():
    N, G, C = 6, 2, 2
    h = np.array([6, 5, 4, 3, 2, 1], dtype=np.float32)
    order = rank_order(h, N)
    assert list(order) == [0, 1, 2, 3, 4, 5]
    stored, locs = _golden_example()
    for (pol, k, g), keys in stored.items():
        loc, sk = policy_placement(order, N, C, G, k)
        assert list(sk[g]) == keys, (pol, k, g)
        check_placement(loc, sk, N, C)
    for pol, k, g, key, src, row in locs:
        loc, _ = policy_placement(order, N, C, G, k)
        s, r = dec(loc[g][key])
        assert (int(s), int(r)) == (src, row), (pol, k, g, key)


def test_rank_order_ties_and_negative_zero():
    h = np.array([1.0, 3.0, 1.0, -0.0, 0.0, 3.0, -2.0], dtype=np.float32)
    assert list(rank_order(h, 7)) == [1, 5, 0, 2, 3, 4, 6]
    assert list(rank_order(None, 4)) == [0, 1, 2, 3]


def test_model_hand_computed_single_gpu():
    # T_L = 1, T_H = 10, R_H = 1/4.  C=2: local mass 11, host mass 10 -> t = max(11,100,36)
    plat = Platform(G=1, row_bytes=1, bw_local=1.0, bw_peer=1.0, bw_host=0.1, host_sms=1,
                    peer_sms=0, num_sms=4)
    h = np.array([6, 5, 4, 3, 2, 1], dtype=np.float32)
    loc, _ = policy_placement(rank_order(h, 6), 6, 2, 1, 2)
    z, t, tj = model_times(h, loc, plat)
    assert tj[0].tolist() == [11.0, 100.0] and z == 100.0
    loc, _ = policy_placement(rank_order(h, 6), 6, 4, 1, 4)
    z, t, tj = model_times(h, loc, plat)
    assert tj[0].tolist() == [18.0, 30.0] and z == 30.0       # area 18 + 7.5 < 30


def test_model_hand_computed_two_gpus():
    # sweep k=1 of the worked example; T_L=1, T_P=2, T_H=2, R_P=3/4, R_H=1/4.
    # GPU0: local {0,1}=11, peer {2}=4*2=8, host {3,4,5}=6*2=12; area 11+6+3=20  -> 20
    # GPU1: local {0,2}=10, peer {1}=5*2=10, host 12;           area 10+7.5+3=20.5 -> 20.5
    plat = Platform(G=2, row_bytes=1, bw_local=1.0, bw_peer=0.5, bw_host=0.5, host_sms=1,
                    peer_sms=3, num_sms=4)
    h = np.array([6, 5, 4, 3, 2, 1], dtype=np.float32)
    loc, _ = policy_placement(rank_order(h, 6), 6, 2, 2, 1)
    z, t, tj = model_times(h, loc, plat)
    assert tj.tolist() == [[11.0, 8.0, 12.0], [10.0, 10.0, 12.0]]
    assert t.tolist() == [20.0, 20.5] and z == 20.5


@pytest.mark.parametrize("E,G,cons_expected,vars_expected",
                         [(10, 2, 78, 89), (7, 4, 192, 193), (100, 8, 7368, 8081)])
def test_milp_size_formula(E, G, cons_expected, vars_expected):
    nv, nc = milp.size(E, G)
    assert nv == E * G * G + 2 * E * G + G * G + 2 * G + 1 == vars_expected
    assert nc == E * G * G + E * G + 2 * G * G + 5 * G == cons_expected


def _brute_force_optimum(h, C, plat):
    """min z over every storage choice (|s_j| <= C) and every access arrangement."""
    E, G = len(h), plat.G
    subsets = [frozenset(c) for r in range(C + 1) for c in itertools.combinations(range(E), r)]
    hh = h.astype(np.float64)
    best = np.inf
    for stores in itertools.product(subsets, repeat=G):
        zi = []
        for i in range(G):
            Ti, Ri = plat.T_row(i), plat.R_row(i)
            opts = [[j for j in range(G) if e in stores[j]] + [G] for e in range(E)]
            ti_best = np.inf
            for a in itertools.product(*opts):
                tj = np.zeros(G + 1)
                for e, j in enumerate(a):
                    tj[j] += Ti[j] * hh[e]
                ti_best = min(ti_best, max(tj.max(), float(np.dot(tj, Ri))))
            zi.append(ti_best)
        best = min(best, max(zi))
    return best


def test_brute_force_equals_milp_and_bounds_sweep():
    plat = Platform(G=2, row_bytes=512, host_sms=8, peer_sms=70, **B200)
    h = np.array([9.0, 5.0, 3.0, 2.0, 1.5], dtype=np.float32)
    C = 2
    bf = _brute_force_optimum(h, C, plat)
    m = milp.solve(h, C, plat)
    assert abs(m["z"] - bf) <= 1e-9 * bf
    k, zs = solve_sweep(h, 5, C, plat)
    assert zs >= bf * (1 - 1e-12)
    # the MILP's own storage/access is a valid placement with the optimum value
    assert m["s"].sum(axis=1).max() <= C


@pytest.mark.parametrize("G,E,C,alpha", [(2, 24, 4, 1.2), (4, 24, 3, 1.2), (4, 40, 6, 1.4)])
def test_sweep_vs_milp_gap(G, E, C, alpha):
    plat = Platform(G=G, row_bytes=512, host_sms=8, peer_sms=(148 - 8) // (G - 1), **B200)
    h = (synth.zipf_pmf(E, alpha) * 1000).astype(np.float32)
    k, zs = solve_sweep(h, E, C, plat)
    m = milp.solve(h, C, plat, time_limit=30)
    gap = zs / m["z"] - 1
    assert gap >= -1e-9
    assert gap < 0.05, gap     # the paper's block method: < 2 % on average


def test_sweep_no_worse_than_rep_and_part():
    G, N, C = 4, 3000, 150
    plat = Platform(G=G, row_bytes=512, host_sms=8, peer_sms=46, **B200)
    h = (synth.zipf_pmf(N, 1.2) * 5e4).astype(np.float32)[np.random.default_rng(0).permutation(N)]
    k, z = solve_sweep(h, N, C, plat)
    order = rank_order(h, N)
    assert z <= sweep_z(h, order, N, C, plat, C) * (1 + 1e-12)
    assert z <= sweep_z(h, order, N, C, plat, 0) * (1 + 1e-12)


def test_checker_accepts_all_k_and_rejects_corruptions():
    N, G, C = 500, 4, 40
    h = np.random.default_rng(3).random(N).astype(np.float32)
    order = rank_order(h, N)
    for k in range(0, C + 1, 7):
        loc, sk = policy_placement(order, N, C, G, k)
        check_placement(loc, sk, N, C)
    loc, sk = policy_placement(order, N, C, G, 10)
    bad = loc.copy()
    s, r = dec(bad[1][order[0]])
    bad[1][order[0]] = enc(G, order[1])                   # host row != key
    with pytest.raises(AssertionError):
        check_placement(bad, sk, N, C)
    bad = loc.copy()
    bad[0][order[20]] = enc(2, 0)                         # slot holds another key
    with pytest.raises(AssertionError):
        check_placement(bad, sk, N, C)
    bad = loc.copy()
    bad[0][order[3]] = enc(G, order[3])                   # local entry not read locally
    with pytest.raises(AssertionError):
        check_placement(bad, sk, N, C)
    sk2 = [s.copy() for s in sk]
    sk2[0] = np.concatenate([sk2[0], sk2[0][:1]])         # stored twice / over capacity
    with pytest.raises(AssertionError):
        check_placement(loc, sk2, N, C)


def test_source_counts_replication_partition_closed_form():
    """Expected per-source shares of the tiny config (SURVEY.md 8(c) "source-mix sanity"):
    replication local = sum_{r<C} p(r); partition local = global/G."""
    wl = synth.get_workload("tiny")
    N, C, G = wl.num_rows, wl.capacity_rows, 2
    h = synth.hotness(wl)
    order = rank_order(h, N)
    p = synth.zipf_pmf(N, wl.alpha)
    keys = np.concatenate([synth.make_batch(wl, r, b) for r in range(2) for b in range(8)])
    loc, _ = policy_placement(order, N, C, G, C)
    cnt, bad = source_counts(loc[0], keys, N, G)
    assert bad == 0
    assert abs(cnt[0] / len(keys) - p[:C].sum()) < 0.01
    loc, _ = policy_placement(order, N, C, G, 0)
    glob = p[:G * C].sum()
    local = [source_counts(loc[g], keys, N, G)[0][g] / len(keys) for g in range(G)]
    assert abs(np.mean(local) - glob / G) < 0.01       # averaged over GPUs
    cnt, _ = source_counts(loc[0], keys, N, G)
    assert abs(cnt[G] / len(keys) - (1 - glob)) < 0.01


def test_paper_policy_claims_model_level():
    """Qualitative claims of section 8.5 reproduced by the model on Zipf(1.2):
    at a small cache ratio the hotness-aware sweep stays close to partition
    (P:2517-2520); at a larger one it replicates a hot prefix, raising the local hit rate
    far above partition's while the global hit rate drops only slightly."""
    G, N = 8, 20_000
    plat = Platform(G=G, row_bytes=512, host_sms=8, peer_sms=17, **B200)
    h = (synth.zipf_pmf(N, 1.2) * 5e4).astype(np.float32)
    order = rank_order(h, N)
    p = h.astype(np.float64) / h.sum()

    def hits(k, C):
        loc, _ = policy_placement(order, N, C, G, k)
        src, _ = dec(loc[0])
        return p[src == 0].sum(), p[src < G].sum()

    C_small = int(0.02 * N)
    k_small, _ = solve_sweep(h, N, C_small, plat)
    C_big = int(0.08 * N)
    k_big, _ = solve_sweep(h, N, C_big, plat)
    assert k_small / C_small <= k_big / C_big
    loc_u, glob_u = hits(k_big, C_big)
    loc_p, glob_p = hits(0, C_big)
    assert loc_u > 2 * loc_p
    assert glob_p - glob_u < 0.05


def test_host_tier_worked_example():
    """Host tier (R24) on the worked example: sweep k=1, C=2, G=2 gives
    band_end = 1 + 2*(2-1) = 3, so ranks 3,4,5 (keys 3,4,5) sit in tier slots 0,1,2."""
    N, G, C = 6, 2, 2
    h = np.array([6, 5, 4, 3, 2, 1], dtype=np.float32)
    order = rank_order(h, N)
    loc, sk = policy_placement(order, N, C, G, 1, host_tier=True)
    for g in range(G):
        for key, slot in ((3, 0), (4, 1), (5, 2)):
            s, r = dec(loc[g][key])
            assert (int(s), int(r)) == (G, slot)
    s, r = dec(loc[0][2])
    assert (int(s), int(r)) == (1, 1)            # GPU entries unchanged
    tier = order[3:]
    check_placement(loc, sk, N, C, tier_keys=tier)
    with pytest.raises(AssertionError):
        check_placement(loc, sk, N, C, tier_keys=tier[::-1])
    with pytest.raises(AssertionError):
        check_placement(loc, sk, N, C)           # host rows are not keys any more


def test_tiny_source_mix_matches_closed_form_coverage():
    """SURVEY.md 8(c) source-mix sanity: batch means of the per-source key shares on tiny
    (N = 100K, C = 10K per GPU, Zipf(1.2), 8,192 i.i.d. keys) match the closed-form Zipf
    coverage: replication local 94.26 % / host 5.74 %; partition over G = 2 local 48.1 %,
    peer 48.1 %, host 3.73 % (the mean over both GPUs).  Sampled through synth's batches and
    the oracle's placement + source counts, so a wrong rank->key map, placement or count fails."""
    wl = synth.get_workload("tiny")
    N, C, G = wl.num_rows, wl.capacity_rows, 2
    order = rank_order(synth.hotness(wl), N)
    shares = {}
    for name, k in (("replication", C), ("partition", 0)):
        loc, _ = policy_placement(order, N, C, G, k)
        tot = np.zeros(3)
        for g in range(G):
            for b in range(10):
                keys = synth.make_batch(wl, g, b)
                cnt, _ = source_counts(loc[g], keys, N, G)
                tot += [cnt[g], cnt[1 - g], cnt[G]]
        shares[name] = tot / tot.sum()
    rep, part = shares["replication"], shares["partition"]
    assert abs(rep[0] - 0.9426) < 0.004 and rep[1] == 0 and abs(rep[2] - 0.0574) < 0.004
    assert abs(part[0] - 0.481) < 0.006 and abs(part[1] - 0.481) < 0.006
    assert abs(part[2] - 0.0373) < 0.004
