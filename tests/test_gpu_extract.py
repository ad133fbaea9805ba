"""GPU parity tests: ugache_extract (through the C ABI) vs the CPU oracle, byte for byte.

Multi-GPU placements are exercised on one device by "fake peers": G contexts in one
process, each with its own cache slab, wired to each other's slabs as peers
(ugache_set_peer_slabs), so bucketing, peer roles and local padding run for G = 2..8.
"""
import numpy as np
import pytest

import oracle
import synth
from oracle.placement import check_placement, source_counts

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    return torch


_TABLES = {}


def table_for(N, R):
    if (N, R) not in _TABLES:
        _TABLES[(N, R)] = synth.make_table(N, R)
    return _TABLES[(N, R)]


def make_group(torch, N, R, C, G, h, policy="ugache", **kw):
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process
    t = table_for(N, R)
    group = [UGache(t, N, R, C, hotness=h, num_gpus=G, rank=g, device=0, policy=policy, **kw)
             for g in range(G)]
    connect_in_process(group)
    for c in group:
        c.fill()
    torch.cuda.synchronize()
    return t, group


def check_batch(torch, cache, table, keys_np, N, R, G, key_dtype=np.int64):
    keys = torch.from_numpy(keys_np.astype(key_dtype)).cuda()
    out = cache.extract(keys)
    torch.cuda.synchronize()
    ref, bad = oracle.gather(table.ptr, N, R, keys_np.astype(np.int64))
    got = out.cpu().numpy()
    assert got.shape == ref.shape
    if not np.array_equal(got, ref):
        rows = np.nonzero((got != ref).any(axis=1))[0]
        raise AssertionError(f"{len(rows)} rows differ, first {rows[:5]} keys {keys_np[rows[:5]]}")
    per, nbad = cache.last_batch_stats()
    loc, _ = cache.export_placement()
    ref_cnt, ref_bad = source_counts(loc, keys_np.astype(np.int64), N, G)
    assert nbad == ref_bad == bad
    assert np.array_equal(per, ref_cnt)
    return per


def test_single_gpu_tiny_parity(torch_cuda):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, (c,) = make_group(torch_cuda, wl.num_rows, wl.row_bytes, wl.capacity_rows, 1, h)
    for b in range(4):
        per = check_batch(torch_cuda, c, t, synth.make_batch(wl, 0, b), wl.num_rows, wl.row_bytes, 1)
        assert per[0] > 0 and per[1] > 0
        assert c.last_launch_count() == 1      # UGACHE_OPT_FUSED auto: one launch per batch
    c.close()


@pytest.mark.parametrize("G", [2, 3, 4, 8])
@pytest.mark.parametrize("policy", ["ugache", "replication", "partition"])
def test_fake_peer_parity(torch_cuda, G, policy):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    N, R = wl.num_rows, wl.row_bytes
    C = 5000
    t, group = make_group(torch_cuda, N, R, C, G, h, policy=policy)
    locs, sks = [], []
    for g, c in enumerate(group):
        loc, sk = c.export_placement()
        locs.append(loc)
        sks.append(sk)
        per = check_batch(torch_cuda, c, t, synth.make_batch(wl, g, 1), N, R, G)
        if policy != "replication":
            assert per[[j for j in range(G) if j != g]].sum() > 0     # peer roles exercised
        # slab content equals the table rows of its slot keys (Filler)
        if len(sk):
            idx = np.linspace(0, len(sk) - 1, 257).astype(np.int64)
            slab = c.read_slab(0, len(sk))
            assert np.array_equal(slab[idx], t.array[sk[idx].astype(np.int64)])
    check_placement(np.stack(locs), sks, N, C)
    for c in group:
        c.close()


@pytest.mark.parametrize("n", [1, 31, 2047, 2048, 2049, 10_001])
def test_ragged_batch_sizes(torch_cuda, n):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, group = make_group(torch_cuda, wl.num_rows, 512, 3000, 3, h)
    keys = synth.make_batch(synth.Workload("r", (wl.num_rows,), 512, 1.2, "iid", n), 0, n)
    for g, c in enumerate(group):
        check_batch(torch_cuda, c, t, keys, wl.num_rows, 512, 3)
    for c in group:
        c.close()


def test_out_of_range_duplicates_and_u32(torch_cuda):
    N, R = 50_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e4).astype(np.float32)
    t, group = make_group(torch_cuda, N, R, 2000, 2, h)
    keys = np.array([0, 0, 0, N - 1, N, -1, -(1 << 40), 1 << 40, 7, 7, 12345] * 300, dtype=np.int64)
    check_batch(torch_cuda, group[0], t, keys, N, R, 2)
    ku = np.array([0, 5, N, N + 7, 3, 3, 49_999] * 500, dtype=np.int64)
    check_batch(torch_cuda, group[1], t, ku, N, R, 2, key_dtype=np.uint32)
    for c in group:
        c.close()


def test_empty_batch(torch_cuda):
    N, R = 10_000, 512
    t, (c,) = make_group(torch_cuda, N, R, 100, 1, None)
    out = c.extract(torch_cuda.zeros(0, dtype=torch_cuda.int64, device="cuda"))
    assert out.shape == (0, R)
    assert c.last_launch_count() == 0
    per, bad = c.last_batch_stats()
    assert per.sum() == 0 and bad == 0
    c.close()


@pytest.mark.parametrize("C", [0, 10_000])
def test_all_host_and_all_local(torch_cuda, C):
    N, R = 10_000, 512
    h = np.random.default_rng(0).random(N).astype(np.float32)
    t, group = make_group(torch_cuda, N, R, C, 2, h)
    keys = np.random.default_rng(1).integers(0, N, 5000)
    for c in group:
        per = check_batch(torch_cuda, c, t, keys, N, R, 2)
        if C == 0:
            assert per[2] == len(keys)
    for c in group:
        c.close()


@pytest.mark.parametrize("R", [16, 48, 512, 1536, 2064, 6144, 8192])
@pytest.mark.parametrize("bulk", [True, False])
def test_row_sizes(torch_cuda, R, bulk):
    """Row sizes from one 16-B vector to 8 KB, local rows by TMA bulk copies (R <= 6 KB)
    or through registers; several chunk and group boundaries per warp."""
    N = 20_000
    h = (synth.zipf_pmf(N, 1.2) * 1e4).astype(np.float32)[np.random.default_rng(R).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 1500, 2, h)
    keys = np.random.default_rng(2).integers(0, N, 7777)
    for c in group:
        c.set_local_bulk(bulk)
        check_batch(torch_cuda, c, t, keys, N, R, 2)
    for c in group:
        c.close()


def test_host_buffers_e2e_path(torch_cuda):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, (c,) = make_group(torch_cuda, wl.num_rows, 512, wl.capacity_rows, 1, h)
    keys = synth.make_batch(wl, 0, 9)
    pinned_keys = torch_cuda.from_numpy(keys).pin_memory()
    out = torch_cuda.empty((len(keys), 512), dtype=torch_cuda.uint8).pin_memory()
    c.extract(pinned_keys, out)
    torch_cuda.cuda.synchronize()
    ref, _ = oracle.gather(t.ptr, wl.num_rows, 512, keys)
    assert np.array_equal(out.numpy(), ref)
    # pageable numpy buffers too
    out2 = np.empty((len(keys), 512), dtype=np.uint8)
    c.extract(keys, out2)
    torch_cuda.cuda.synchronize()
    assert np.array_equal(out2, ref)
    c.close()


@pytest.mark.parametrize("G", [1, 4])
def test_random_dispatch_mode_parity(torch_cuda, G):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, group = make_group(torch_cuda, wl.num_rows, 512, 4000, G, h)
    for g, c in enumerate(group):
        c.set_mode("random")
        check_batch(torch_cuda, c, t, synth.make_batch(wl, g, 3), wl.num_rows, 512, G)
        assert c.last_launch_count() == 1
        c.set_mode("factored")
    for c in group:
        c.close()


@pytest.mark.parametrize("host_sms,peer_sms", [(1, 1), (1, 36), (100, 1), (4, 12)])
def test_dedication_variants(torch_cuda, host_sms, peer_sms):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, group = make_group(torch_cuda, wl.num_rows, 512, 3000, 4, h)
    for g, c in enumerate(group):
        c.set_dedication(host_sms, peer_sms)
        check_batch(torch_cuda, c, t, synth.make_batch(wl, g, 4), wl.num_rows, 512, 4)
    for c in group:
        c.close()


def test_timing_and_repeated_extracts(torch_cuda):
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, (c,) = make_group(torch_cuda, wl.num_rows, 512, wl.capacity_rows, 1, h)
    c.enable_timing(True)
    keys = synth.make_batch(wl, 0, 5)
    for i in range(20):  # counters re-armed by the kernel itself across launches
        c.set_stream("on" if i % 2 else "off")
        per = check_batch(torch_cuda, c, t, keys, wl.num_rows, 512, 1)
        a, b = c.last_batch_timing()
        # the single pass has no separate locate phase: it is reported as 0
        assert b > 0 and (a == 0 if i % 2 else a > 0)
    c.close()


def test_pa_shaped_scaled_parity(torch_cuda):
    """PA-shaped rows/skew/batch at 1/10 of the rows: 11.1M x 512 B, 500K-unique batch
    scaled to 50K, 10 % cache, G = 8 fake peers."""
    wl = synth.get_workload("gnn_pa@0.1")
    h = synth.hotness(wl)
    t, group = make_group(torch_cuda, wl.num_rows, wl.row_bytes, wl.capacity_rows, 8, h)
    for g in (0, 5):
        check_batch(torch_cuda, group[g], t, synth.make_batch(wl, g, 0), wl.num_rows,
                    wl.row_bytes, 8)
    for c in group:
        c.close()
    t.close()
    _TABLES.pop((wl.num_rows, wl.row_bytes), None)


def test_dlr_shaped_scaled_parity(torch_cuda):
    wl = synth.get_workload("dlr_criteo@0.02")
    h = synth.hotness(wl)
    t, group = make_group(torch_cuda, wl.num_rows, wl.row_bytes, wl.capacity_rows, 4, h)
    check_batch(torch_cuda, group[1], t, synth.make_batch(wl, 1, 0), wl.num_rows, wl.row_bytes, 4)
    for c in group:
        c.close()
    t.close()
    _TABLES.pop((wl.num_rows, wl.row_bytes), None)


@pytest.mark.parametrize("ordered", [True, False])
@pytest.mark.parametrize("host_sms", [1, 3, 16, 147])
def test_host_range_ordering_parity(torch_cuda, ordered, host_sms):
    """Large host bucket (>= kHostSortMin keys): range-ordered and unordered host reads
    give the same bytes, for any number of host CTAs (intra-role barriers)."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(5).permutation(N)]
    t, (c,) = make_group(torch_cuda, N, R, 3000, 1, h)
    c.set_host_ordering(ordered)  # UGACHE_OPT_HOST_ORDERING
    c.set_dedication(host_sms, 0)
    keys = np.random.default_rng(6).integers(0, N, 40_000)
    keys[::50] = -3
    for _ in range(3):  # re-armed range counters across launches
        per = check_batch(torch_cuda, c, t, keys, N, R, 1)
        assert per[1] > 4096
    c.close()


@pytest.mark.parametrize("staged", [False, True])
def test_pinned_host_io_zero_copy_and_staged(torch_cuda, staged):
    """Pinned host keys/out are used in place by the kernels (default) or staged; both
    produce the oracle's bytes, including zero rows of out-of-range keys."""
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(8).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 4000, 2, h)
    keys = np.random.default_rng(9).integers(0, N, 30_000)
    keys[::97] = N + 1
    pk = torch_cuda.from_numpy(keys).pin_memory()
    for g, c in enumerate(group):
        c.set_stage_host_io(staged)
        out = torch_cuda.full((len(keys), R), 7, dtype=torch_cuda.uint8).pin_memory()
        c.extract(pk, out)
        torch_cuda.cuda.synchronize()
        ref, bad = oracle.gather(t.ptr, N, R, keys)
        assert np.array_equal(out.numpy(), ref)
        per, nbad = c.last_batch_stats()
        assert nbad == bad
    for c in group:
        c.close()


@pytest.mark.parametrize("G", [1, 4])
def test_host_tier_parity(torch_cuda, G):
    """UGACHE_FLAG_HOST_TIER: host rows are read from the ctx's rank-ordered pinned copy."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(11).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 3000, G, h, host_tier=True)
    keys = np.random.default_rng(12).integers(-5, N + 5, 40_000)
    for g, c in enumerate(group):
        per = check_batch(torch_cuda, c, t, keys, N, R, G)
        assert per[G] > 4096            # range-ordered host path on the tier
        c.set_host_ordering(False)
        check_batch(torch_cuda, c, t, keys[:999], N, R, G)
    for c in group:
        c.close()


def test_shared_host_tier_buffer(torch_cuda):
    """A caller-built tier (ugache_fill_host_tier) shared by every rank's ctx."""
    from paper_conf_sosp_songz0c23_b200 import (UGache, connect_in_process, fill_host_tier,
                                                host_tier_rows, make_config, solve)
    wl = synth.get_workload("tiny")
    N, R, G = wl.num_rows, wl.row_bytes, 2
    t = table_for(N, R)
    h = synth.hotness(wl)
    cfg = make_config(N, R, wl.capacity_rows, num_gpus=G, host_tier=True)
    plan, order = solve(cfg, h)
    tier = np.empty((host_tier_rows(plan, N), R), dtype=np.uint8)
    fill_host_tier(cfg, order, plan, t, tier)
    group = [UGache(t, N, R, wl.capacity_rows, num_gpus=G, rank=g, plan=plan, order=order,
                    host_tier=tier) for g in range(G)]
    connect_in_process(group)
    for c in group:
        c.fill()
    for g, c in enumerate(group):
        check_batch(torch_cuda, c, t, synth.make_batch(wl, g, 2), N, R, G)
    for c in group:
        c.close()


@pytest.mark.parametrize("G,hw,pw", [(1, 1, 1), (1, 5, 1), (4, 1, 1), (4, 3, 2), (8, 2, 2)])
@pytest.mark.parametrize("big_host", [False, True])
def test_warp_granular_dedication_parity(torch_cuda, G, hw, pw, big_host):
    """UGACHE_DEDICATE_WARPS: host / peer warps on every SM, ordered or strided host reads."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(13).permutation(N)]
    C = 2000 if big_host else 60_000
    t, group = make_group(torch_cuda, N, R, min(C, N // G), G, h)
    keys = np.random.default_rng(14).integers(-3, N + 3, 30_000)
    for g, c in enumerate(group):
        c.set_dedication_mode("warps", host_warps=hw, peer_warps=pw)
        per = check_batch(torch_cuda, c, t, keys, N, R, G)
        if big_host:
            assert per[G] > 4096
    for c in group:
        c.close()


def test_embedding_layer_module(torch_cuda):
    """UGacheEmbedding: [B, T] keys -> [B, T, D] float32 rows, bitwise equal to
    the oracle; no grad (read-only table)."""
    from paper_conf_sosp_songz0c23_b200.layer import UGacheEmbedding
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, (c,) = make_group(torch_cuda, wl.num_rows, 512, wl.capacity_rows, 1, h)
    emb = UGacheEmbedding(c, 128, torch_cuda.float32)
    keys_np = synth.make_batch(wl, 0, 7)[:4096].reshape(64, 64)
    y = emb(torch_cuda.from_numpy(keys_np).cuda())
    assert y.shape == (64, 64, 128) and y.dtype == torch_cuda.float32 and not y.requires_grad
    ref, _ = oracle.gather(t.ptr, wl.num_rows, 512, keys_np.reshape(-1))
    assert np.array_equal(y.view(torch_cuda.uint8).reshape(-1, 512).cpu().numpy(), ref)
    with pytest.raises(ValueError):
        UGacheEmbedding(c, 64, torch_cuda.float32)
    c.close()


def test_block_milp_placement_parity(torch_cuda):
    """Placement from the block-level MILP (section 6.3), which may replicate a block on any
    subset of GPUs and read a stored block from a peer, through ugache_init_with_placement."""
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process, make_config, solve
    from paper_conf_sosp_songz0c23_b200.milp_solver import (make_blocks, placement_from_blocks,
                                                            solve_blocks)
    from oracle.placement import rank_order
    N, R, G, C = 20_000, 512, 4, 900
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(21).permutation(N)]
    cfg = make_config(N, R, C, num_gpus=G)
    plan, order = solve(cfg, h)
    ordr = order.astype(np.int64)
    blocks = make_blocks(h[ordr], G)
    s, a, z, _ = solve_blocks(h[ordr], blocks, C, G, (plan.T_local, plan.T_peer, plan.T_host),
                              (plan.R_local, plan.R_peer, plan.R_host), time_limit=60)
    locs, sks = placement_from_blocks(ordr, blocks, s, a, N, G)
    t = table_for(N, R)
    group = [UGache(t, N, R, C, num_gpus=G, rank=g, placement=(locs[g], sks[g])) for g in range(G)]
    connect_in_process(group)
    for c in group:
        c.fill()
    keys = np.random.default_rng(22).integers(0, N, 20_000)
    for g, c in enumerate(group):
        loc, sk = c.export_placement()
        assert np.array_equal(loc, locs[g]) and np.array_equal(sk, sks[g])
        check_batch(torch_cuda, c, t, keys, N, R, G)
    bad = locs[0].copy()
    bad[int(sks[0][0]) if len(sks[0]) else 0] = np.uint64(G) << np.uint64(56)  # host row != key
    with pytest.raises(Exception):
        UGache(t, N, R, C, num_gpus=G, rank=0, placement=(bad, sks[0]))
    for c in group:
        c.close()


def test_cache_refresh_protocol(torch_cuda):
    """Section 7.2 refresh on G = 3 fake peers: hotness shifts (a new Zipf permutation), the
    Refresher re-solves, and extraction stays bit-exact after every step (transitional
    table -> rewritten content -> new table); the committed placement equals the new one
    and passes the checker; the modeled time of the old placement under the new hotness is
    worse than the new optimum."""
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process
    from paper_conf_sosp_songz0c23_b200.refresh import (HotnessSampler, modeled_time,
                                                        plan_placements, refresh_group,
                                                        should_refresh)
    N, R, G, C = 100_000, 512, 3, 6000
    p = (synth.zipf_pmf(N, 1.2) * 8192).astype(np.float32)
    h1 = p[np.random.default_rng(1).permutation(N)]
    h2 = p[np.random.default_rng(2).permutation(N)]
    kw = dict(num_rows=N, row_bytes=R, capacity_rows=C)
    plan1, pl1 = plan_placements(kw, h1, G)
    t = table_for(N, R)
    group = [UGache(t, N, R, C, num_gpus=G, rank=g, placement=pl1[g]) for g in range(G)]
    connect_in_process(group)
    for c in group:
        c.fill()
    # foreground sampling under the new distribution
    rng = np.random.default_rng(3)
    cdf = np.cumsum(h2.astype(np.float64)) / h2.sum()
    sampler = HotnessSampler(N)
    batches = [np.searchsorted(cdf, rng.random(8192)).astype(np.int64) for _ in range(8)]
    for b in batches:
        sampler.record(b)
    plan2, pl2 = plan_placements(kw, sampler.hotness(), G)
    assert should_refresh([l for l, _ in pl1], h2, plan2)
    assert modeled_time([l for l, _ in pl2], h2, plan2) < modeled_time([l for l, _ in pl1], h2, plan2)

    def foreground():
        for g, c in enumerate(group):
            check_batch(torch_cuda, c, t, batches[g], N, R, G)

    foreground()
    for c, (loc, sk) in zip(group, pl2):
        c.refresh_begin(loc, sk)
    foreground()                                  # transitional tables
    with pytest.raises(Exception):
        group[0].refresh_commit()                 # content step missing -> ESTATE
    for c in group:                               # chunked content, foreground in between
        while c.refresh_content(max_sms=4, max_rows=700) > 0:
            foreground()
    foreground()                                  # new content, transitional tables
    for c in group:
        c.refresh_commit()
    foreground()                                  # new placement
    locs, sks = [], []
    for g, c in enumerate(group):
        loc, sk = c.export_placement()
        assert np.array_equal(loc, pl2[g][0]) and np.array_equal(sk, pl2[g][1])
        locs.append(loc)
        sks.append(sk)
        if len(sk):
            idx = np.linspace(0, len(sk) - 1, 301).astype(np.int64)
            assert np.array_equal(c.read_slab(0, len(sk))[idx], t.array[sk[idx].astype(np.int64)])
    check_placement(np.stack(locs), sks, N, C)
    # refresh back with the group helper
    refresh_group(group, pl1, max_sms=8, max_rows=2500, foreground=foreground)
    foreground()
    for c in group:
        c.close()


@pytest.mark.parametrize("G", [1, 4])
@pytest.mark.parametrize("walk", [True, False])
@pytest.mark.parametrize("key_dtype", [np.int64, np.uint32])
def test_sparse_host_walk_parity(torch_cuda, G, walk, key_dtype):
    """UGACHE_OPT_HOST_WALK: sparse host rows found by an input-order walk of the batch
    (and the bucket path when off) give the oracle's bytes, with duplicates and bad keys."""
    N, R = 400_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(31).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 20_000, G, h)
    rng = np.random.default_rng(32)
    hot = np.argsort(-h, kind="stable")[:15_000]          # cached somewhere (C = 20K per GPU)
    keys = np.concatenate([rng.integers(0, N, 3000), rng.choice(hot, 20_000)])
    rng.shuffle(keys)
    keys[::101] = N + 3
    for g, c in enumerate(group):
        c.set_host_walk(walk)
        per = check_batch(torch_cuda, c, t, keys, N, R, G, key_dtype=key_dtype)
        assert 0 < per[G] < 4096
    for c in group:
        c.close()


@pytest.mark.parametrize("fused", ["on", "off", "stream"])
@pytest.mark.parametrize("G,C,n", [(1, 3000, 1), (1, 3000, 40_000), (4, 2000, 50_001), (3, 40_000, 9_999)])
def test_fused_and_split_launch_parity(torch_cuda, fused, G, C, n):
    """K1+K2 in one cooperative launch (grid barrier) vs two launches vs the single pass:
    same bytes/counts, dense and sparse host buckets, ragged sizes, u32 keys."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(41).permutation(N)]
    t, group = make_group(torch_cuda, N, R, C, G, h)
    keys = np.random.default_rng(42).integers(-2, N + 2, n)
    for g, c in enumerate(group):
        c.set_fused("on" if fused == "stream" else fused)
        c.set_stream("on" if fused == "stream" else "off")
        c.set_local_bulk(g % 2 == 0)
        for kd in (np.int64, np.uint32):
            check_batch(torch_cuda, c, t, np.abs(keys) if kd == np.uint32 else keys, N, R, G, key_dtype=kd)
            assert c.last_launch_count() == (2 if fused == "off" else 1)
            assert c.last_extract_path() == {"off": "split", "on": "fused", "stream": "single_pass"}[fused]
    for c in group:
        c.close()


@pytest.mark.parametrize("G,policy", [(1, "ugache"), (2, "partition"), (4, "ugache"), (8, "partition")])
@pytest.mark.parametrize("fused", ["on", "off"])
def test_message_based_baseline_parity(torch_cuda, G, policy, fused):
    """Message-based baseline: local/host rows by the factored kernels with no
    peer SMs, peer rows through request/serve/reply exchanges and a scatter into key order
     -- same bytes and per-source counts as the oracle, incl. out-of-range keys."""
    from paper_conf_sosp_songz0c23_b200.message import message_extract_group
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    N, R = wl.num_rows, wl.row_bytes
    t, group = make_group(torch_cuda, N, R, 4000, G, h, policy=policy)
    for c in group:
        c.set_fused(fused)
    for b in range(2):
        keys_np = [synth.make_batch(wl, g, b) for g in range(G)]
        keys_np[0][::777] = N + 3
        keys = [torch_cuda.from_numpy(k).cuda() for k in keys_np]
        outs = message_extract_group(group, keys)
        torch_cuda.cuda.synchronize()
        for g, c in enumerate(group):
            ref, bad = oracle.gather(t.ptr, N, R, keys_np[g])
            assert np.array_equal(outs[g].cpu().numpy(), ref)
            per, nbad = c.last_batch_stats()
            loc, _ = c.export_placement()
            ref_cnt, ref_bad = source_counts(loc, keys_np[g], N, G)
            assert nbad == ref_bad == bad and np.array_equal(per, ref_cnt)
            if G > 1 and b == 0:
                assert per[[j for j in range(G) if j != g]].sum() > 0
    # protocol misuse: scatter without the earlier steps -> ESTATE
    from paper_conf_sosp_songz0c23_b200._abi import UGacheError
    from paper_conf_sosp_songz0c23_b200 import message
    with pytest.raises(UGacheError):
        message._scatter(group[0], outs[0], outs[0], None)
    for c in group:
        c.close()


@pytest.mark.parametrize("early", [True, False])
@pytest.mark.parametrize("G,C,n", [(1, 2000, 30_000), (1, 2000, 700_000), (2, 20_000, 120_000),
                                   (4, 60_000, 8_193)])
def test_early_host_walk_parity(torch_cuda, early, G, C, n):
    """Fused launch with CTAs that have no locate tile walking for host rows before the grid
    barrier: dense host buckets (the ordered path must skip the walked prefix), sparse ones
    (the post-barrier walk continues from the shared cursor), and batches with more tiles
    than CTAs (no early walkers)."""
    N, R = 400_000, 512
    h = (synth.zipf_pmf(N, 1.1) * 1e5).astype(np.float32)[np.random.default_rng(43).permutation(N)]
    t, group = make_group(torch_cuda, N, R, C, G, h)
    rng = np.random.default_rng(44)
    for g, c in enumerate(group):
        c.set_fused("on")
        c.set_stream("off")
        c.set_early_walk(early)
        for b in range(3):  # repeated launches: the walk cursor is re-armed by the kernel
            keys = rng.integers(0, N, n)
            keys[:: 997] = N + 1
            per = check_batch(torch_cuda, c, t, keys, N, R, G)
            assert per[G] > 0
    for c in group:
        c.close()


@pytest.mark.parametrize("inline", ["host", "none", "all"])
@pytest.mark.parametrize("G,host_sms,peer_sms", [(1, 12, 0), (1, 148, 0), (2, 12, 60), (4, 1, 1),
                                                 (8, 12, 19), (8, 1, 21)])
def test_single_pass_parity(torch_cuda, inline, G, host_sms, peer_sms):
    """Single-pass extraction (UGACHE_OPT_STREAM): locate + inline local copies + per-source
    queues drained by dedicated SMs.  Every dedication split, including grids whose every SM
    is dedicated (1 + 7 x 21 = 148: every warp is a consumer that also locates), inline and
    queued host / peer rows, ragged and empty chunks, out-of-range keys, u32 keys, and
    repeated launches (queues re-armed to ~0 by their consumers)."""
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(45).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 6000, G, h)
    rng = np.random.default_rng(46)
    for g, c in enumerate(group[:3]):
        c.set_fused("on")
        c.set_stream("on")
        c.set_inline(host=inline != "none", peers=inline == "all")
        if G > 1 or host_sms != 12:
            c.set_dedication(host_sms, peer_sms if G > 1 else 0)
        for b, n in enumerate([1, 63, 64, 65, 5_000, 100_001, 77_777]):
            c.set_local_bulk(b != 6)  # rows through TMA slots, or the register path
            keys = rng.integers(0, N, n)
            keys[:: 613] = N + b
            kd = np.uint32 if b % 2 else np.int64
            per = check_batch(torch_cuda, c, t, keys, N, R, G, key_dtype=kd)
            assert c.last_launch_count() == 1
            if n > 50_000:
                assert per[G] > 0 and (G == 1 or per[[j for j in range(G) if j != g]].sum() > 0)
    for c in group:
        c.close()


def test_stream_auto_switches_on_host_density(torch_cuda):
    """UGACHE_OPT_STREAM = auto picks the path from the previous launch's host count (mirrored
    by the kernel to pinned host memory): a dense-host batch after sparse ones (and back)
    stays bit-exact, and the path taken follows the density (single pass: no locate phase)."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(47).permutation(N)]
    t, (c,) = make_group(torch_cuda, N, R, 30_000, 1, h)
    c.set_fused("on")
    c.set_stream("auto")
    c.enable_timing(True)
    rng = np.random.default_rng(48)
    loc, _ = c.export_placement()
    host_keys = np.nonzero((loc >> 56) == 1)[0]
    local_keys = np.nonzero((loc >> 56) == 0)[0]
    # before any launch the choice comes from the plan's expected host keys
    prev_dense = 200_000 * c.plan.host_mass_frac >= 4096
    for b in range(7):
        dense = b in (2, 3, 4)
        keys = rng.choice(host_keys if dense else local_keys, 200_000)
        if not dense:
            keys[:50] = host_keys[:50]
        per = check_batch(torch_cuda, c, t, keys, N, R, 1)
        assert per[1] == (200_000 if dense else 50)
        a, _ = c.last_batch_timing()
        assert (a > 0) == prev_dense   # ordered path after a dense batch, single pass otherwise
        assert c.last_extract_path() == ("fused" if prev_dense else "single_pass")
        prev_dense = dense
    c.close()


@pytest.mark.parametrize("G", [1, 4])
@pytest.mark.parametrize("k", ["1", "2"])
@pytest.mark.parametrize("sched", ["0", "1", "2", "3"])
def test_single_pass_static_schedule_and_chunk_sizes(torch_cuda, monkeypatch, G, k, sched):
    """Single pass with every chunk schedule (UGACHE_STREAM_STATIC: 0 dynamic cursor, 1
    static, 2/3 static rounds then a dynamic tail), both chunk sizes (UGACHE_STREAM_K),
    queued peers and inline host rows."""
    monkeypatch.setenv("UGACHE_STREAM_STATIC", sched)
    monkeypatch.setenv("UGACHE_STREAM_K", k)
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(49).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 6000, G, h)
    rng = np.random.default_rng(50)
    for g, c in enumerate(group[:2]):
        c.set_fused("on")
        c.set_stream("on")
        for n in (1, 100, 60_001, 300_000):
            keys = rng.integers(0, N, n)
            keys[::101] = N + 9
            check_batch(torch_cuda, c, t, keys, N, R, G)
    for c in group:
        c.close()


def test_stream_auto_with_peers(torch_cuda):
    """auto keeps the two-phase kernel when peer rows are queued to dedicated SMs (G > 1,
    default, batches above 32768 keys) and takes the single pass once peers are inline or the
    batch is small; all bit-exact."""
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(51).permutation(N)]
    # partition of 2 x 95,000 rows: 5 % of uniform keys go to the host (a sparse bucket)
    t, group = make_group(torch_cuda, N, R, 95_000, 2, h, policy="partition")
    c = group[0]
    c.set_stream("auto")
    keys = np.random.default_rng(52).integers(0, N, 40_000)
    for peers_inline, want in ((False, "fused"), (True, "single_pass")):
        c.set_inline(host=True, peers=peers_inline)
        for _ in range(2):
            per = check_batch(torch_cuda, c, t, keys, N, R, 2)
            assert per[1] > 0 and 0 < per[2] < 3000, per
        assert c.last_extract_path() == want
    # a small batch (<= 32768 keys, latency-bound) takes the single pass with its peer rows
    # read inline even when peers are otherwise queued to dedicated SMs
    c.set_inline(host=True, peers=False)
    for n in (1, 8_192, 32_768):
        per = check_batch(torch_cuda, c, t, keys[:n], N, R, 2)
        assert c.last_extract_path() == "single_pass", n
    check_batch(torch_cuda, c, t, keys[:32_769], N, R, 2)
    assert c.last_extract_path() == "fused"
    for g in group:
        g.close()


@pytest.mark.parametrize("G", [1, 4])
def test_single_pass_register_store_retire(torch_cuda, monkeypatch, G):
    """Single pass with landed slots leaving by warp-wide 16-B stores (UGACHE_STREAM_REGSTORE)
    instead of bulk copies: bit-exact incl. 1536-B rows (8 slots per warp)."""
    monkeypatch.setenv("UGACHE_STREAM_REGSTORE", "1")
    for R in (512, 1536):
        N = 100_000
        h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(53).permutation(N)]
        t, group = make_group(torch_cuda, N, R, 8000, G, h)
        c = group[0]
        c.set_stream("on")
        c.set_inline(host=True, peers=G > 2)
        for n in (5, 20_000, 120_001):
            keys = np.random.default_rng(n).integers(0, N + 3, n)
            check_batch(torch_cuda, c, t, keys, N, R, G)
        for g in group:
            g.close()


@pytest.mark.parametrize("prefetch", ["1", "2"])
@pytest.mark.parametrize("sched", ["0", "1", "2"])
@pytest.mark.parametrize("key_dtype", [np.int64, np.uint32])
def test_single_pass_locate_pipeline(torch_cuda, monkeypatch, prefetch, sched, key_dtype):
    """Single pass with the locating warps pipelined (UGACHE_STREAM_PREFETCH: 1 registers,
    2 shared memory via cp.async): every chunk's entries are the ones of its own keys, for
    both key types, every chunk schedule, queued peers, inline host rows, out-of-range keys,
    ragged and tiny batches."""
    monkeypatch.setenv("UGACHE_STREAM_PREFETCH", prefetch)
    monkeypatch.setenv("UGACHE_STREAM_STATIC", sched)
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(57).permutation(N)]
    for G in (1, 4):
        t, group_ = make_group(torch_cuda, N, R, 6000, G, h)
        c = group_[0]
        c.set_stream("on")
        for n in (1, 31, 33, 4_999, 150_001, 700_000):
            keys = np.random.default_rng(n).integers(0, N + 2, n)
            if key_dtype == np.int64:
                keys[::97] = -5
            check_batch(torch_cuda, c, t, keys, N, R, G, key_dtype=key_dtype)
        for g in group_:
            g.close()


@pytest.mark.parametrize("G", [1, 4])
def test_sparse_host_bucket_walk_or_order(torch_cuda, G):
    """A sparse host bucket (far below the ordering threshold) on the two-phase kernel: with
    G = 1 every SM walks the batch in input order (no ordering stamp); with peer roles holding
    most SMs (G = 4) the walkers would be few, so the bucket is range-ordered instead (the
    ordering stamp is set).  Bit-exact either way, out-of-range keys included."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(58).permutation(N)]
    C = 295_000 // G   # ~1.7 % of uniform keys on the host: < 4096 of 200K
    t, group = make_group(torch_cuda, N, R, C, G, h, policy="partition")
    c = group[0]
    c.enable_timing(True)
    c.set_stream("off")
    rng = np.random.default_rng(59)
    for n in (200_000, 77_777):
        keys = rng.integers(0, N + 2, n)
        per = check_batch(torch_cuda, c, t, keys, N, R, G)
        assert 0 < per[G] < 4096, per
        assert c.last_extract_path() == "fused"
        _, ordered, _, _, _ = c.last_batch_phases()
        assert (ordered > 0) == (G > 1), (G, ordered)
    for g in group:
        g.close()


@pytest.mark.parametrize("G", [1, 4])
def test_role_timeline(torch_cuda, G):
    """ugache_last_batch_timeline after a fused launch: one row per SM; role counts match
    the dedication (host CTAs = calibrated host SMs for a dense bucket, peer_sms per peer,
    the rest local); per CTA start <= gather start <= role done <= done <= the launch end;
    ESTATE after a single-pass launch or with timing off."""
    from paper_conf_sosp_songz0c23_b200._abi import UGacheError
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(66).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 20_000, G, h)
    c = group[0]
    c.set_stream("off")
    keys = np.random.default_rng(67).integers(0, N, 200_000)     # dense host bucket
    c.enable_timing(False)
    check_batch(torch_cuda, c, t, keys, N, R, G)
    with pytest.raises(UGacheError):
        c.last_batch_timeline()
    c.enable_timing(True)
    check_batch(torch_cuda, c, t, keys, N, R, G)
    tl = c.last_batch_timeline()
    end = c.last_batch_phases()[4]
    S = torch_cuda.cuda.get_device_properties(0).multi_processor_count
    assert tl.shape == (S, 5)
    roles = tl[:, 0].astype(int)
    assert set(roles.tolist()) <= set(range(G + 1))
    assert (roles == G).sum() == c.plan.host_sms
    for j in range(1, G):
        assert (roles == j).sum() == c.plan.peer_sms, (j, (roles == j).sum())
    assert np.all(tl[:, 1] <= tl[:, 2]) and np.all(tl[:, 2] <= tl[:, 3]) and np.all(tl[:, 3] <= tl[:, 4])
    assert tl[:, 4].max() <= end + 1e-3
    c.set_stream("on")
    check_batch(torch_cuda, c, t, keys[:5000], N, R, G)
    with pytest.raises(UGacheError):
        c.last_batch_timeline()
    for g in group:
        g.close()


@pytest.mark.parametrize("ck", ["8", "16", "32", "0"])
@pytest.mark.parametrize("G", [1, 4])
def test_single_pass_register_kernel(torch_cuda, monkeypatch, ck, G):
    """K3r, the lean register single pass (sparse host bucket, every source inline;
    UGACHE_REG_KERNEL_CK = keys per chunk, 0 = K3's own register path): bit-exact with
    out-of-range keys, both key types, ragged and tiny batches, G = 1 and G = 4 with peer
    rows inline; per-source counts exact."""
    monkeypatch.setenv("UGACHE_REG_KERNEL_CK", ck)
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(68).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 190_000 // G, G, h, policy="partition")
    c = group[0]
    c.set_stream("auto")
    c.set_inline(host=True, peers=True)
    rng = np.random.default_rng(69)
    for n in (1, 33, 8_191, 50_000, 70_001):
        keys = rng.integers(-3, N + 3, n)
        for kd in (np.int64, np.uint32):
            per = check_batch(torch_cuda, c, t, np.abs(keys) if kd == np.uint32 else keys, N, R, G, key_dtype=kd)
            if n >= 50_000:
                assert 0.005 * n <= per[G] < 4096, per
                assert c.last_extract_path() == "single_pass"
    for g in group:
        g.close()


def test_fused_phase_stamps(torch_cuda):
    """ugache_last_batch_phases: after a fused launch with a dense host bucket the stamps are
    ordered (locate <= host ordered <= host copies done <= the launch's event time); after a
    single-pass launch the call reports ESTATE."""
    from paper_conf_sosp_songz0c23_b200._abi import UGacheError
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(54).permutation(N)]
    t, (c,) = make_group(torch_cuda, N, R, 10_000, 1, h)
    c.enable_timing(True)
    c.set_stream("off")
    keys = np.random.default_rng(55).integers(0, N, 200_000)   # ~97 % host keys: dense
    check_batch(torch_cuda, c, t, keys, N, R, 1)
    loc_ms, gat_ms = c.last_batch_timing()
    a, b, d, la, e = c.last_batch_phases()
    assert 0 < la <= a <= b <= d <= e <= (loc_ms + gat_ms) * 1.05 + 0.01
    c.set_stream("on")
    check_batch(torch_cuda, c, t, keys[:5000], N, R, 1)
    with pytest.raises(UGacheError):
        c.last_batch_phases()
    c.close()


@pytest.mark.parametrize("group", ["2", "3", "8"])
@pytest.mark.parametrize("sched", ["0", "1"])
def test_single_pass_host_first_groups(torch_cuda, monkeypatch, group, sched):
    """Single pass with groups of chunks whose non-local rows go first (UGACHE_STREAM_GROUP):
    every chunk processed exactly once (static and dynamic schedules), queued peers and
    inline host rows, ragged and tiny batches."""
    monkeypatch.setenv("UGACHE_STREAM_GROUP", group)
    monkeypatch.setenv("UGACHE_STREAM_STATIC", sched)
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(56).permutation(N)]
    for G in (1, 4):
        t, group_ = make_group(torch_cuda, N, R, 6000, G, h)
        c = group_[0]
        c.set_stream("on")
        for n in (3, 4_999, 150_001, 700_000):
            keys = np.random.default_rng(n).integers(0, N + 2, n)
            check_batch(torch_cuda, c, t, keys, N, R, G)
        for g in group_:
            g.close()


@pytest.mark.parametrize("fused", ["on", "off"])
@pytest.mark.parametrize("G,tier", [(1, False), (1, True), (2, False), (4, True)])
def test_preorder_parity(torch_cuda, fused, G, tier):
    """UGACHE_OPT_PREORDER: the host range histogram is built while locating and every CTA
    scatters a slice of the host bucket; bit-exact against the oracle and against the host
    CTAs' own ordering, on the fused and split paths, with and without the host tier, and
    across dense -> sparse -> dense launches (the histogram is re-armed either way)."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(60).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 4000, G, h, host_tier=tier)
    rng = np.random.default_rng(61)
    for g, c in enumerate(group):
        c.set_stream("off")
        c.set_fused(fused)
        for pre in (True, False, True):
            c.set_preorder(pre)
            for n, dense in ((150_000, True), (3_000, False), (120_001, True)):
                keys = rng.integers(-3, N + 3, n)
                per = check_batch(torch_cuda, c, t, keys, N, R, G)
                assert (per[G] >= 4096) == dense
    for c in group:
        c.close()


def test_preorder_phase_stamps(torch_cuda):
    """With pre-ordering, host copies begin right after the locate boundary: the host bucket
    is ordered before the copies start, every stamp is inside the launch."""
    N, R = 300_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(62).permutation(N)]
    t, (c,) = make_group(torch_cuda, N, R, 10_000, 1, h, host_tier=True)
    c.enable_timing(True)
    c.set_stream("off")
    c.set_fused("on")
    keys = np.random.default_rng(63).integers(0, N, 200_000)
    for _ in range(3):
        check_batch(torch_cuda, c, t, keys, N, R, 1)
        loc_ms, gat_ms = c.last_batch_timing()
        located, ordered, host_done, last_loc, end = c.last_batch_phases()
        assert 0 < last_loc <= located <= ordered <= host_done <= end <= (loc_ms + gat_ms) * 1.05 + 0.01
    c.close()


def test_first_batch_path_from_plan(torch_cuda):
    """UGACHE_OPT_STREAM = auto before any launch: the path follows the plan's expected host
    keys (n x host_mass_frac vs the ordering threshold), not a default."""
    N, R = 400_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(64).permutation(N)]
    for C, n in ((8_000, 200_000), (300_000, 20_000)):
        t, (c,) = make_group(torch_cuda, N, R, C, 1, h)
        expect_dense = n * c.plan.host_mass_frac >= 4096
        assert expect_dense == (C == 8_000)
        keys = np.random.default_rng(65).choice(N, n, p=h / h.sum())
        check_batch(torch_cuda, c, t, keys, N, R, 1)
        assert c.last_extract_path() == ("fused" if expect_dense else "single_pass")
        c.close()


@pytest.mark.parametrize("inline", ["host", "none"])
def test_fresh_ctx_on_nonblocking_stream(torch_cuda, inline):
    """The scratch (queue sentinels, sub-queue counters) of a fresh ctx is initialised on the
    extract stream: the first launches on a non-blocking stream are bit-exact, including
    queued host rows (inline none) and a batch that grows the scratch."""
    N, R = 200_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(66).permutation(N)]
    t, (c,) = make_group(torch_cuda, N, R, 20_000, 1, h)
    c.set_stream("on")
    c.set_inline(host=inline == "host", peers=False)
    s = torch_cuda.cuda.Stream()
    for n in (30_000, 250_000):
        keys_np = np.random.default_rng(n).integers(0, N, n)
        keys = torch_cuda.from_numpy(keys_np).cuda()
        torch_cuda.cuda.synchronize()
        out = torch_cuda.empty((n, R), dtype=torch_cuda.uint8, device="cuda")
        c.extract(keys, out, s)
        s.synchronize()
        ref, _ = oracle.gather(t.ptr, N, R, keys_np)
        assert np.array_equal(out.cpu().numpy(), ref)
    c.close()


def test_init_rejects_bad_order_plan_and_alignment(torch_cuda):
    """ugache_init_with_plan: an order that is not a permutation, or a plan larger than the
    config's capacity, is EINVAL; a host table that is not 16-byte aligned is EINVAL (the
    kernels read rows with 16-byte vector loads and bulk copies)."""
    from paper_conf_sosp_songz0c23_b200 import UGache, make_config, solve
    from paper_conf_sosp_songz0c23_b200._abi import UGACHE_EINVAL, UGacheError
    N, R, C = 20_000, 512, 1000
    t = table_for(N, R)
    h = (synth.zipf_pmf(N, 1.2) * 1e4).astype(np.float32)
    cfg = make_config(N, R, C, host_tier=True)
    plan, order = solve(cfg, h)
    bad = order.copy()
    bad[5] = bad[6]                                   # duplicate key, one key missing
    with pytest.raises(UGacheError) as e:
        UGache(t, N, R, C, plan=plan, order=bad, host_tier=True)
    assert e.value.status == UGACHE_EINVAL
    big_cfg = make_config(N, R, 2 * C)
    big_plan, big_order = solve(big_cfg, h)
    with pytest.raises(UGacheError) as e:
        UGache(t, N, R, C, plan=big_plan, order=big_order)
    assert e.value.status == UGACHE_EINVAL
    raw = np.empty(N * R + 16, dtype=np.uint8)
    off = (-raw.ctypes.data) % 16 + 8                 # 8 bytes past a 16-byte boundary
    mis = raw[off: off + N * R]
    with pytest.raises(UGacheError) as e:
        UGache(mis, N, R, C, hotness=h)
    assert e.value.status == UGACHE_EINVAL
    ok = UGache(t, N, R, C, plan=plan, order=order, host_tier=True)   # the valid pair works
    ok.fill()
    check_batch(torch_cuda, ok, t, np.arange(0, N, 7), N, R, 1)
    ok.close()


@pytest.mark.parametrize("protocol", ["chunked", "whole"])
@pytest.mark.parametrize("G", [1, 3])
def test_cache_refresh_with_host_tier(torch_cuda, protocol, G):
    """Section 7.2 refresh on a host-tier ctx (the shipped configuration): keys evicted from
    the cache are redirected to their slot of the tier (which holds every row), extraction
    stays bit-exact through every step of the chunked (stage / evict / fill / install per
    slot range) and whole-table (begin / content / commit) protocols, and the committed table
    equals the new placement with host rows mapped to tier slots."""
    from paper_conf_sosp_songz0c23_b200 import UGache, connect_in_process, make_config, solve
    from paper_conf_sosp_songz0c23_b200.refresh import plan_placements, refresh_group
    N, R, C = 120_000, 512, 7000
    p = (synth.zipf_pmf(N, 1.2) * 8192).astype(np.float32)
    h1 = p[np.random.default_rng(71).permutation(N)]
    h2 = p[np.random.default_rng(72).permutation(N)]
    t = table_for(N, R)
    group = [UGache(t, N, R, C, hotness=h1, num_gpus=G, rank=g, host_tier=True) for g in range(G)]
    connect_in_process(group)
    for c in group:
        c.fill()
    plan1, order1 = solve(make_config(N, R, C, num_gpus=G, host_tier=True), h1)
    be1 = int(plan1.band_end)
    tier_slot = np.empty(N, dtype=np.uint64)
    tier_slot[order1.astype(np.int64)] = (np.arange(N, dtype=np.uint64) + np.uint64(N - be1)) % np.uint64(N)
    _, pl2 = plan_placements(dict(num_rows=N, row_bytes=R, capacity_rows=C), h2, G)
    rng = np.random.default_rng(73)
    cdf = np.cumsum(h2.astype(np.float64)) / h2.sum()
    batches = [np.searchsorted(cdf, rng.random(30_000)).astype(np.int64) for _ in range(G)]
    n_fg = [0]

    def foreground():
        for g, c in enumerate(group):
            check_batch(torch_cuda, c, t, batches[g], N, R, G)
        n_fg[0] += 1

    foreground()
    if protocol == "chunked":
        refresh_group(group, pl2, max_sms=4, max_rows=2000, foreground=foreground)
        assert n_fg[0] >= 1 + (C + 1999) // 2000
    else:
        for c, (loc, sk) in zip(group, pl2):
            c.refresh_begin(loc, sk)
        foreground()
        for c in group:
            while c.refresh_content(max_sms=4, max_rows=3000) > 0:
                foreground()
        torch_cuda.cuda.synchronize()
        foreground()
        for c in group:
            c.refresh_commit()
    foreground()
    host = np.uint64(G) << np.uint64(56)
    for g, c in enumerate(group):
        loc, sk = c.export_placement()
        want = pl2[g][0].copy()
        is_host = (want >> np.uint64(56)) == np.uint64(G)
        want[is_host] = host | tier_slot[is_host]
        assert np.array_equal(loc, want) and np.array_equal(sk, pl2[g][1])
    for c in group:
        c.close()


@pytest.mark.parametrize("G", [1, 2])
def test_calibrate(torch_cuda, G):
    """ugache_calibrate (A0): host bandwidth vs SMs over the swept counts, the recommended
    host SMs is the first point within 90 % of the best, local gather beats the host link,
    and with peers the all-to-all ingress curve is measured; extraction is unaffected."""
    N, R = 400_000, 512
    h = (synth.zipf_pmf(N, 1.2) * 1e5).astype(np.float32)[np.random.default_rng(81).permutation(N)]
    t, group = make_group(torch_cuda, N, R, 20_000, G, h, host_tier=True)
    cal = group[0].calibrate(16384)
    ks = [k for k, _ in cal["host_curve"]]
    bws = [b for _, b in cal["host_curve"]]
    assert ks == sorted(ks) and ks[0] == 1 and len(ks) >= 8 and all(b > 0 for b in bws)
    first90 = next(k for k, b in cal["host_curve"] if b >= 0.9 * max(bws))
    assert cal["host_sms"] == first90 and cal["bw_host"] >= 0.9 * max(bws)
    assert cal["bw_local"] > cal["bw_host"] and cal["sample_rows"] == 16384
    if G > 1:
        assert cal["peer_curve"] and cal["peer_sms"] >= 1 and cal["bw_peer"] > 0
    else:
        assert cal["peer_curve"] == [] and cal["peer_sms"] == 0
    check_batch(torch_cuda, group[0], t, np.random.default_rng(82).integers(0, N, 50_000), N, R, G)
    for c in group:
        c.close()


@pytest.mark.parametrize("stream_mode", ["on", "off"])
def test_cuda_graph_capture_and_replay(torch_cuda, stream_mode):
    """ugache_extract can be captured into a CUDA graph (no host synchronisation, no
    allocation after the first call; the single-pass and the cooperative two-phase launches
    both capture) and replayed on new key contents, bit-exact every time."""
    torch = torch_cuda
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    t, (c,) = make_group(torch, wl.num_rows, wl.row_bytes, wl.capacity_rows, 1, h)
    c.set_stream(stream_mode)
    n = 8192
    keys = torch.from_numpy(synth.make_batch(wl, 0, 0)).cuda()
    out = torch.empty((n, wl.row_bytes), dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        c.extract(keys, out, s)          # warm-up: scratch allocated outside the capture
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        c.extract(keys, out, s)
    for b in range(1, 5):
        kb = synth.make_batch(wl, 0, b)
        keys.copy_(torch.from_numpy(kb))
        g.replay()
        torch.cuda.synchronize()
        ref, _ = oracle.gather(t.ptr, wl.num_rows, wl.row_bytes, kb)
        assert np.array_equal(out.cpu().numpy(), ref), b
    c.close()


@pytest.mark.slow
def test_full_size_gnn_pa_sampled_parity(torch_cuda):
    """BASELINE configs[1] at full size in the benched launch configuration (111M x 512 B
    rows, 500K unique Zipf(1.2) keys, c = 10 %, host tier, auto path = the fused kernel):
    per-source counts equal the oracle's over the whole batch, and 8,192 sampled output rows
    (plus the first and last) equal the oracle's gather of the same keys byte for byte."""
    wl = synth.get_workload("gnn_pa")
    N, R = wl.num_rows, wl.row_bytes
    table = synth.HostTable(N, R)
    table.fill()
    from paper_conf_sosp_songz0c23_b200 import UGache
    c = UGache(table, N, R, wl.capacity_rows, hotness=synth.hotness(wl), host_tier=True)
    c.fill()
    keys_np = synth.make_batch(wl, 0, 0)
    keys = torch_cuda.from_numpy(keys_np).cuda()
    out = c.extract(keys)
    torch_cuda.cuda.synchronize()
    assert c.last_extract_path() == "fused"
    per, bad = c.last_batch_stats()
    loc, _ = c.export_placement()
    ref_cnt, ref_bad = source_counts(loc, keys_np, N, 1)
    del loc
    assert bad == ref_bad == 0 and np.array_equal(per, ref_cnt) and per[1] > 50_000
    idx = np.concatenate([[0, len(keys_np) - 1], np.random.default_rng(91).choice(len(keys_np), 8192, replace=False)])
    ref, _ = oracle.gather(table.ptr, N, R, keys_np[idx])
    got = out[torch_cuda.from_numpy(idx).cuda()].cpu().numpy()
    assert np.array_equal(got, ref)
    c.close()
    table.close()
