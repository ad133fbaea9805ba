"""Pins for the CPU gather oracle (oracle/gather.c): checked against the generator's
re-derivation of every row and against numpy fancy indexing -- not against itself."""
import numpy as np
import pytest

import oracle
import synth


@pytest.mark.parametrize("R", [16, 512, 1536])
def test_gather_equals_generator_rows(R):
    N = 3000
    t = synth.make_table(N, R)
    rng = np.random.default_rng(R)
    keys = rng.integers(0, N, size=4099)
    keys[::97] = -1
    keys[5::211] = N
    keys[7::333] = 1 << 40
    out, bad = oracle.gather(t.ptr, N, R, keys)
    assert bad == int(np.sum((keys < 0) | (keys >= N)))
    assert np.array_equal(out, synth.rows_for_keys(keys, N, R))
    valid = (keys >= 0) & (keys < N)
    assert np.array_equal(out[valid], t.array[keys[valid]])   # numpy fancy indexing
    assert not out[~valid].any()
    t.close()


def test_gather_u32_keys_and_empty():
    N, R = 1000, 512
    t = synth.make_table(N, R)
    keys = np.array([0, 999, 1000, 5, 5, 5], dtype=np.uint32)
    out, bad = oracle.gather(t.ptr, N, R, keys)
    assert bad == 1
    assert np.array_equal(out, synth.rows_for_keys(keys.astype(np.int64), N, R))
    out0, bad0 = oracle.gather(t.ptr, N, R, np.zeros(0, dtype=np.int64))
    assert out0.shape == (0, R) and bad0 == 0
    t.close()


def test_gather_duplicates_keep_key_order():
    N, R = 100, 64
    t = synth.make_table(N, R)
    keys = np.array([3, 1, 3, 3, 99, 0, 1], dtype=np.int64)
    out, _ = oracle.gather(t.ptr, N, R, keys)
    for i, k in enumerate(keys):
        assert np.array_equal(out[i], t.array[k])
    t.close()
