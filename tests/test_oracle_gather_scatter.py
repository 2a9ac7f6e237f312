"""Pins for the gather-scatter microbenchmark oracle (f2, reading F2):
closed forms with x = 1 and table = k, and numpy's own add.at / bincount."""
import numpy as np


def test_single_point_closed_forms(orc):
    rng = np.random.default_rng(0)
    K = 97
    keys = rng.integers(0, K, 5000).astype(np.int32)
    acc = np.zeros(K)
    out = orc.gather_scatter(keys, np.ones(5000), np.arange(K, dtype=np.float64), acc)
    assert np.array_equal(out, keys.astype(np.float64))          # gather = table[k] = k
    assert np.array_equal(acc, np.bincount(keys, minlength=K))   # scatter of ones = counts


def test_stencil_closed_forms(orc):
    K, nx = 10 * 12, 12
    keys = np.repeat(np.arange(K, dtype=np.int32), 7)
    acc = np.zeros(K)
    out = orc.gather_scatter(keys, np.ones(keys.size), np.arange(K, dtype=np.float64), acc, nx)
    interior = (keys >= nx + 1) & (keys < K - nx - 1)
    assert np.array_equal(out[interior], 5.0 * keys[interior])   # k + (k-1) + (k+1) + (k-nx) + (k+nx)
    assert np.all(acc == 5 * 7)                                   # every key is in 5 stencils x 7 copies


def test_random_values_match_numpy(orc):
    rng = np.random.default_rng(1)
    K, nx = 1000, 25
    keys = rng.integers(0, K, 20000).astype(np.int32)
    x = rng.standard_normal(20000)
    table = rng.standard_normal(K)
    acc = np.zeros(K)
    out = orc.gather_scatter(keys, x, table, acc, nx)
    k = keys.astype(np.int64)
    pts = [k, (k - 1) % K, (k + 1) % K, (k - nx) % K, (k + nx) % K]
    want = np.zeros(K)
    for pnt in pts:
        np.add.at(want, pnt, x)
    assert np.allclose(acc, want, rtol=1e-12, atol=1e-12)
    assert np.allclose(out, sum(table[pnt] for pnt in pts), rtol=1e-14, atol=1e-14)
