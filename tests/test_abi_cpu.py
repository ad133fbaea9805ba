"""CPU tests of the C ABI: the library loads, exports every symbol include/ugache.h
declares, validates configs, and its host-only placement solver matches the oracle
(bit-exact integer placements; model value within fp rounding)."""
import ctypes
import os
import re

import numpy as np
import pytest

import synth
from oracle.placement import (Platform, check_placement, model_times, policy_placement,
                              rank_order, solve_sweep, sweep_z)
from paper_conf_sosp_songz0c23_b200 import _abi, build_placement, make_config, solve

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "ugache.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ugache_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = ctypes.CDLL(_abi.LIB_PATH)
    names = _declared_symbols()
    assert len(names) >= 20
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(_abi.SIGNATURES), set(names) ^ set(_abi.SIGNATURES)
    assert _abi.lib().ugache_version() == 1
    assert _abi.lib().ugache_error_string(1) == b"invalid argument"


def test_struct_layouts_match_header():
    # sizes follow from the header's field list (no implicit padding surprises)
    assert ctypes.sizeof(_abi.ugache_config) == 8 + 4 + 4 + 8 + 4 * 4 + 8 * 3 + 4 * 4
    assert ctypes.sizeof(_abi.ugache_plan) == 4 + 4 + 8 * 3 + 8 * 9 + 4 * 4 + 8


@pytest.mark.parametrize("field,value", [
    ("num_rows", 0), ("num_rows", 1 << 32), ("row_bytes", 0), ("row_bytes", 24),
    ("num_gpus", 0), ("num_gpus", 17), ("policy", 3), ("flags", 2), ("reserved0", 2),
    ("host_sms", 148), ("host_sms", -1), ("bw_host", -1.0)])
def test_solve_rejects_bad_config(field, value):
    cfg = make_config(1000, 512, 100, num_gpus=2)
    setattr(cfg, field, value)
    st = _abi.lib().ugache_solve(ctypes.byref(cfg), None, None, ctypes.byref(_abi.ugache_plan()))
    assert st == _abi.UGACHE_EINVAL


def test_solve_rejects_nan_hotness_and_oversubscribed_sms():
    cfg = make_config(10, 512, 2, num_gpus=2)
    h = np.ones(10, dtype=np.float32)
    h[3] = np.nan
    st = _abi.lib().ugache_solve(ctypes.byref(cfg), h.ctypes.data, None,
                                 ctypes.byref(_abi.ugache_plan()))
    assert st == _abi.UGACHE_EINVAL
    cfg = make_config(10, 512, 2, num_gpus=4, host_sms=10, peer_sms=50)
    st = _abi.lib().ugache_solve(ctypes.byref(cfg), None, None, ctypes.byref(_abi.ugache_plan()))
    assert st == _abi.UGACHE_EINVAL


def _platform(cfg, plan):
    return Platform(G=cfg.num_gpus, row_bytes=cfg.row_bytes,
                    bw_local=cfg.bw_local or 6457.7e9, bw_peer=cfg.bw_peer or 770e9,
                    bw_host=cfg.bw_host or 34.4e9, host_sms=plan.host_sms,
                    peer_sms=plan.peer_sms, num_sms=plan.num_sms)


CASES = [
    # (N, C, G, alpha, hotness perturbation)
    (6, 2, 2, None, "golden"),
    (997, 50, 2, 1.2, "zipf"),
    (2000, 150, 4, 1.2, "zipf"),
    (3000, 90, 8, 1.4, "zipf"),
    (1500, 400, 4, 0.8, "zipf"),
    (500, 500, 3, 1.2, "zipf"),      # C = N
    (400, 1000, 2, 1.2, "zipf"),     # C > N
    (800, 0, 4, 1.2, "zipf"),        # no cache
    (1200, 100, 4, None, "ties"),    # many equal hotness values
    (1000, 60, 1, 1.2, "zipf"),
]


def _hot(N, alpha, kind):
    if kind == "golden":
        return np.array([6, 5, 4, 3, 2, 1], dtype=np.float32)
    if kind == "ties":
        return np.random.default_rng(N).integers(0, 5, size=N).astype(np.float32)
    h = (synth.zipf_pmf(N, alpha) * 1e4).astype(np.float32)
    return h[np.random.default_rng(N).permutation(N)]


@pytest.mark.parametrize("N,C,G,alpha,kind", CASES)
@pytest.mark.parametrize("policy", ["ugache", "replication", "partition"])
def test_solver_matches_oracle(N, C, G, alpha, kind, policy):
    h = _hot(N, alpha, kind)
    cfg = make_config(N, 512, C, num_gpus=G, policy=policy, host_sms=8)
    plan, order = solve(cfg, h)
    assert np.array_equal(order.astype(np.int64), rank_order(h, N))
    plat = _platform(cfg, plan)
    Cc = min(C, N)
    assert plan.capacity_rows == Cc
    if policy == "replication" or G == 1:
        k_ref = Cc
    elif policy == "partition":
        k_ref = 0
    else:
        k_ref, z_ref = solve_sweep(h, N, C, plat)
        z_lib_at_oracle_metric = sweep_z(h, rank_order(h, N), N, C, plat, int(plan.k))
        # the library's k is optimal under the oracle's model (ties may pick another k)
        assert z_lib_at_oracle_metric <= z_ref * (1 + 1e-9)
    if policy != "ugache" or G == 1:
        assert plan.k == k_ref
    z_o = sweep_z(h, rank_order(h, N), N, C, plat, int(plan.k))
    assert abs(plan.z - z_o) <= 1e-9 * max(z_o, 1e-30)
    assert abs(plan.z_replication - sweep_z(h, rank_order(h, N), N, C, plat, Cc)) <= 1e-9 * plan.z_replication
    loc_ref, sk_ref = policy_placement(rank_order(h, N), N, C, G, int(plan.k))
    locs, sks = [], []
    for g in range(G):
        loc, sk = build_placement(cfg, order, plan, g)
        assert np.array_equal(loc, loc_ref[g]), g
        assert np.array_equal(sk, sk_ref[g]), g
        locs.append(loc)
        sks.append(sk)
    check_placement(np.stack(locs), sks, N, Cc)
    if G > 1 and policy == "ugache":
        assert plan.z <= plan.z_replication * (1 + 1e-12)
        assert plan.z <= plan.z_partition * (1 + 1e-12)


def test_solver_uniform_hotness_is_key_order():
    cfg = make_config(100, 512, 10, num_gpus=2)
    plan, order = solve(cfg, None)
    assert np.array_equal(order, np.arange(100, dtype=np.uint64))


def test_solver_negative_zero_hotness():
    h = np.array([1.0, -0.0, 0.0, 2.0, -5.0, 0.0], dtype=np.float32)
    cfg = make_config(6, 512, 2, num_gpus=1)
    _, order = solve(cfg, h)
    assert list(order) == list(rank_order(h, 6)) == [3, 0, 1, 2, 4, 5]


@pytest.mark.slow
def test_solver_scale_pa_shaped():
    """PA-shaped N = 111M is handled by the host solver in seconds (radix sort + O(C*G))."""
    import time
    N = 20_000_000
    h = np.random.default_rng(0).random(N, dtype=np.float32)
    cfg = make_config(N, 512, N // 10, num_gpus=8)
    t = time.time()
    plan, order = solve(cfg, h)
    assert time.time() - t < 60
    assert np.all(np.diff(h[order.astype(np.int64)[:100000]]) <= 0)



@pytest.mark.parametrize("N,C,G,alpha,kind", CASES[:6])
def test_solver_host_tier_matches_oracle(N, C, G, alpha, kind):
    h = _hot(N, alpha, kind)
    cfg = make_config(N, 512, C, num_gpus=G, host_sms=8, host_tier=True)
    plan, order = solve(cfg, h)
    loc_ref, sk_ref = policy_placement(rank_order(h, N), N, C, G, int(plan.k), host_tier=True)
    locs, sks = [], []
    for g in range(G):
        loc, sk = build_placement(cfg, order, plan, g)
        assert np.array_equal(loc, loc_ref[g]) and np.array_equal(sk, sk_ref[g])
        locs.append(loc)
        sks.append(sk)
    check_placement(np.stack(locs), sks, N, min(C, N),
                    tier_keys=rank_order(h, N)[int(plan.band_end):])


def test_fill_host_tier_matches_generator():
    from paper_conf_sosp_songz0c23_b200 import fill_host_tier, host_tier_rows
    N, R = 5000, 512
    h = _hot(N, 1.2, "zipf")
    cfg = make_config(N, R, 300, num_gpus=4, host_sms=8, host_tier=True)
    plan, order = solve(cfg, h)
    t = synth.make_table(N, R)
    rows = host_tier_rows(plan, N)
    assert rows == N                       # every row: host-resident ranks first, then cached
    tier = np.empty((rows, R), dtype=np.uint8)
    fill_host_tier(cfg, order, plan, t, tier)
    keys = np.roll(order.astype(np.int64), -int(plan.band_end))     # slot t: rank (be + t) mod N
    assert np.array_equal(tier, synth.rows_for_keys(keys, N, R))
    t.close()


@pytest.mark.parametrize("G,k_frac,alpha", [(1, 1.0, 1.2), (2, 0.5, 1.2), (4, 0.0, 0.9), (8, 0.3, 1.4)])
def test_model_time_matches_oracle_model(G, k_frac, alpha):
    """ugache_model_time (the Refresher's trigger model behind the ABI) equals the oracle's
    section 6.2 model (oracle.placement.model_times) on family placements and on a shuffled
    (arbitrary) placement, with the plan's T / R."""
    from oracle.placement import Platform, model_times
    from paper_conf_sosp_songz0c23_b200 import model_time
    N, C = 4000, 300
    h = _hot(N, alpha, "zipf")
    cfg = make_config(N, 512, C, num_gpus=G, host_sms=8, bw_local=6457.7e9, bw_peer=770e9, bw_host=34.4e9)
    plan, order = solve(cfg, h)
    plat = Platform(G=G, row_bytes=512, bw_local=6457.7e9, bw_peer=770e9, bw_host=34.4e9, host_sms=8,
                    peer_sms=int(plan.peer_sms), num_sms=int(plan.num_sms))
    loc, _ = policy_placement(rank_order(h, N), N, C, G, int(k_frac * C))
    z_ref, _, _ = model_times(h, loc, plat)
    assert abs(model_time(plan, list(loc), h) - z_ref) <= 1e-9 * z_ref
    rng = np.random.default_rng(G)
    shuffled = np.stack([l[rng.permutation(N)] for l in loc])       # any table: only src counts
    z_ref2, _, _ = model_times(h, shuffled, plat)
    assert abs(model_time(plan, list(shuffled), h) - z_ref2) <= 1e-9 * z_ref2
