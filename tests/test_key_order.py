"""The packed-key order the sweep's FP64-pipe max relies on (`kmax64`).

A key is float_bits(w) << 32 | col with w > 0 finite (validate_level >= 1 rejects anything else)
or 0 (a zeroed self-loop / padding).  Read as an IEEE double, such a bit pattern is non-negative,
finite and never NaN, and its double order must equal the unsigned integer order of the bits --
then DSETP + FSEL computes exactly the u64 max.  Checked here on the host with numpy (the same
IEEE comparison), including ties in w, subnormal weights, the largest finite float and key 0.
"""
import numpy as np
import pytest


def _keys(w, col):
    wb = np.asarray(w, dtype=np.float32).view(np.uint32).astype(np.uint64)
    return (wb << np.uint64(32)) | np.asarray(col, dtype=np.uint64)


def _check_order(keys):
    d = keys.view(np.float64)
    assert np.all(np.isfinite(d)) and np.all(d >= 0.0)
    i, j = np.triu_indices(len(keys), 1)
    assert np.array_equal(keys[i] > keys[j], d[i] > d[j])
    assert np.array_equal(keys[i] == keys[j], d[i] == d[j])
    # the max of any subset agrees bit for bit
    rng = np.random.default_rng(5)
    for _ in range(200):
        sub = rng.choice(len(keys), size=rng.integers(1, len(keys)), replace=False)
        assert keys[sub].max() == d[sub].max().view(np.uint64)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_uniform_weights(seed):
    rng = np.random.default_rng(seed)
    w = rng.random(300, dtype=np.float32) + np.float32(1e-7)
    col = rng.integers(0, 2**31 - 1, size=300)
    _check_order(_keys(w, col))


def test_ties_extremes_and_zero():
    tiny = np.float32(np.finfo(np.float32).smallest_subnormal)
    w = [0.125, 0.125, 0.125, 1.0, 1.0, tiny, tiny, np.finfo(np.float32).tiny,
         np.finfo(np.float32).max, np.finfo(np.float32).max, 3.0e-39, 0.999]
    col = [0, 7, 2**31 - 2, 5, 6, 0, 1, 9, 3, 4, 8, 11]
    keys = np.concatenate([_keys(w, col), np.array([0], dtype=np.uint64)])
    _check_order(keys)


def test_paper_three_decimal_weights():
    # weights with three decimals in [0, 1] -> heavy ties broken by the column
    rng = np.random.default_rng(9)
    w = (rng.integers(1, 1001, size=400) / 1000.0).astype(np.float32)
    col = rng.integers(0, 1 << 26, size=400)
    _check_order(_keys(w, col))
