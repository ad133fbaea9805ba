"""CPU tests of the shared input generators (synth/)."""
import os

import numpy as np
import pytest

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_splitmix64_reference_vectors():
    """The C word generator reproduces Vigna's published splitmix64 outputs."""
    rows = []
    with open(os.path.join(GOLDEN, "splitmix64_vectors.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            i, hx = line.split()
            rows.append((int(i), int(hx, 16)))
    gamma = 0x9E3779B97F4A7C15
    # word(k, w) with seed 0, W = 1 (row_bytes 4) and k = i*gamma is lo32(splitmix64(i*gamma));
    # keys are int64 so use rows whose index equals the needed value where representable:
    # use seed = i*gamma and key 0 instead (seed ^ 0 = i*gamma).
    for i, ref in rows:
        seed = (i * gamma) & ((1 << 64) - 1)
        r = synth.rows_for_keys(np.array([0]), 1, 4, seed=seed)
        assert int(r.view(np.uint32)[0, 0]) == ref & 0xFFFFFFFF
        r2 = synth.rows_for_keys_numpy(np.array([0]), 1, 4, seed=seed)
        assert int(r2.view(np.uint32)[0, 0]) == ref & 0xFFFFFFFF


def test_c_generator_matches_numpy_generator():
    rng = np.random.default_rng(1)
    for R in (16, 512, 1536):
        N = 5000
        keys = rng.integers(-3, N + 3, size=777)
        a = synth.rows_for_keys(keys, N, R)
        b = synth.rows_for_keys_numpy(keys, N, R)
        assert np.array_equal(a, b)
        t = synth.make_table(N, R)
        valid = (keys >= 0) & (keys < N)
        assert np.array_equal(t.array[keys[valid]], a[valid])
        assert not a[~valid].any()
        t.close()


def test_table_contains_nan_patterns():
    t = synth.make_table(2000, 512)
    f = t.array.view(np.float32)
    assert np.isnan(f).any()
    t.close()


@pytest.mark.parametrize("N", [1, 2, 97, 100_000, 30_769_231])
def test_bijection_is_a_permutation_and_invertible(N):
    r = np.arange(min(N, 200_000), dtype=np.int64)
    k = synth.rank_to_key(r, N, table_idx=3)
    assert np.all((k >= 0) & (k < N))
    assert len(np.unique(k)) == len(k)
    assert np.array_equal(synth.key_to_rank(k, N, table_idx=3), r)


def test_zipf_pmf_closed_form_coverage():
    # tiny replication at 10 % cache: sum_{r<=10000} p(r) for N=1e5, alpha 1.2
    p = synth.zipf_pmf(100_000, 1.2)
    assert abs(p.sum() - 1) < 1e-12
    assert abs(p[:10_000].sum() - 0.94256) < 1e-4
    assert np.all(np.diff(p) < 0)


def test_zipf_sampler_frequencies():
    rng = np.random.Generator(np.random.PCG64(7))
    N, m = 50, 400_000
    r = synth.sample_ranks(rng, N, 1.2, m)
    freq = np.bincount(r, minlength=N) / m
    p = synth.zipf_pmf(N, 1.2)
    sd = np.sqrt(p * (1 - p) / m)
    assert np.all(np.abs(freq - p) < 6 * sd + 1e-9)


def test_batches_are_deterministic_and_shaped():
    wl = synth.get_workload("tiny")
    a = synth.make_batch(wl, 0, 3)
    b = synth.make_batch(wl, 0, 3)
    c = synth.make_batch(wl, 1, 3)
    assert np.array_equal(a, b) and not np.array_equal(a, c)
    assert a.dtype == np.int64 and len(a) == 8192
    assert np.all((a >= 0) & (a < wl.num_rows))


def test_unique_batch():
    wl = synth.Workload("u", (200_000,), 512, 1.2, "unique", 5000)
    keys, draws = synth.make_batch(wl, 0, 0, return_draws=True)
    assert len(keys) == 5000 and len(np.unique(keys)) == 5000
    m = synth.expected_draws_unique(200_000, 1.2, 5000)
    assert 0.7 * m < draws < 1.3 * m


def test_dlr_batch_layout():
    wl = synth.get_workload("dlr_criteo@0.001")
    keys = synth.make_batch(wl, 2, 0)
    T = wl.num_tables
    assert len(keys) == wl.batch_n * T
    offs = synth.table_offsets(wl)
    k2 = keys.reshape(wl.batch_n, T)
    for t in range(T):
        assert np.all((k2[:, t] >= offs[t]) & (k2[:, t] < offs[t] + wl.table_rows[t]))


def test_hotness_orders_by_rank():
    wl = synth.get_workload("tiny")
    h = synth.hotness(wl)
    ranks = synth.key_to_rank(np.arange(wl.num_rows), wl.num_rows)
    hr = np.empty_like(h)
    hr[ranks] = h
    assert np.all(np.diff(hr.astype(np.float64)) <= 0)
    assert abs(h.sum() - 8192) < 1.0


def test_aliased_table_rows_repeat_the_physical_prefix():
    """AliasedHostTable: a full-size span backed by phys_rows physical rows mapped repeatedly;
    row k is the generator's row k mod phys_rows, writes through one alias show in all."""
    N, R, P = 20_000, 512, 4096
    t = synth.AliasedHostTable(N, R, P)
    t.fill()
    assert t.phys_rows == P and t.copies == 5 and t.array.shape == (N, R)
    keys = np.array([0, 1, P - 1, P, P + 7, 3 * P + 11, N - 1])
    want = synth.rows_for_keys(keys % P, N, R)
    assert np.array_equal(t.array[keys], want)
    t.array[5, :4] = 7                     # shared physical page
    assert np.all(t.array[P + 5, :4] == 7) and np.all(t.array[4 * P + 5, :4] == 7)
    t.close()
