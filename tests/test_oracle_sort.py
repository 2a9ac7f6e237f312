"""Pins for the oracle's sorts (Alg. 1, Alg. 2).

What fixes the expected values here (not the oracle itself):
* a hand-worked example (tests/golden/sort_worked_example.json);
* the paper's prose invariants: strided output "is split into one or more
  strictly monotonically increasing subsets"; tiled: "each chunk
  contains one or more repeating tiles where all keys in each tile are in
  strided sort order";
* the lexicographic characterisation (r, k) / (floor(k/T), r, k) derived in
  DESIGN.md, checked by brute force over every short key sequence against
  Python's own sorted() on tuples;
* special cases: all-distinct keys -> strided == standard; all-equal -> identity.
"""
import itertools
import json
import os

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden", "sort_worked_example.json")


def ranks(keys):
    seen = {}
    r = []
    for k in keys:
        r.append(seen.get(k, 0))
        seen[k] = seen.get(k, 0) + 1
    return r


def lex_perm(keys, order, T=1):
    r = ranks(keys)
    idx = range(len(keys))
    if order == 0:
        return sorted(idx, key=lambda i: (keys[i], i))
    if order == 1:
        return sorted(idx, key=lambda i: (r[i], keys[i]))
    if order == 2:
        return sorted(idx, key=lambda i: (keys[i] // T, r[i], keys[i]))
    return list(idx)


def test_worked_example(orc):
    g = json.load(open(GOLD))
    keys = g["keys"]
    nk, perm = orc.sort_keys(keys, orc.SORT_STRIDED)
    assert nk.tolist() == g["strided"]["new_keys"]
    assert perm.tolist() == g["strided"]["perm"]
    assert [keys[i] for i in perm] == g["strided"]["sorted_keys"]
    nk, perm = orc.sort_keys(keys, orc.SORT_TILED, g["tiled"]["tile_sz"])
    assert nk.tolist() == g["tiled"]["new_keys"]
    assert perm.tolist() == g["tiled"]["perm"]
    nk, perm = orc.sort_keys(keys, orc.SORT_STANDARD)
    assert perm.tolist() == g["standard"]["perm"]
    assert nk.tolist() == keys


@pytest.mark.parametrize("offset", [0, 5, 13])
def test_bruteforce_small(orc, offset):
    """Every sequence of length <= 6 over a 4-letter alphabet (shifted by
    offset), every order, T in {1,2,3,5}: the oracle's permutation equals the
    lexicographic characterisation and all adjusted keys are unique."""
    count = 0
    for n in range(0, 7):
        for seq in itertools.product(range(4), repeat=n):
            keys = [s + offset for s in seq]
            for order, Ts in ((0, [1]), (1, [1]), (2, [1, 2, 3, 5]), (3, [1])):
                for T in Ts:
                    nk, perm = orc.sort_keys(keys, order, T)
                    assert perm.tolist() == lex_perm(keys, order, T), (keys, order, T)
                    if order in (1, 2):
                        assert len(set(nk.tolist())) == len(keys)
                    count += 1
    assert count > 5000


def _runs(seq):
    """Split into maximal strictly increasing runs."""
    out, cur = [], []
    for k in seq:
        if cur and k <= cur[-1]:
            out.append(cur)
            cur = []
        cur.append(k)
    if cur:
        out.append(cur)
    return out


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_strided_invariant(orc, seed):
    rng = np.random.default_rng(seed)
    keys = rng.integers(100, 400, 5000).astype(np.int32)
    _, perm = orc.sort_keys(keys, orc.SORT_STRIDED)
    out = keys[perm]
    runs = _runs(out.tolist())
    counts = np.bincount(keys)
    # strictly increasing subsets; subset r holds every key seen > r times
    assert len(runs) == counts.max()
    for r, run in enumerate(runs):
        assert run == sorted(np.nonzero(counts > r)[0].tolist())
    assert sorted(perm.tolist()) == list(range(keys.size))


@pytest.mark.parametrize("T", [7, 64, 1000])
def test_tiled_invariant(orc, T):
    rng = np.random.default_rng(T)
    keys = rng.integers(0, 3000, 20000).astype(np.int32)
    _, perm = orc.sort_keys(keys, orc.SORT_TILED, T)
    out = keys[perm]
    chunk = out // T
    assert np.all(np.diff(chunk) >= 0)  # chunks ascending, contiguous
    counts = np.bincount(keys, minlength=3000)
    for c in np.unique(chunk):
        seg = out[chunk == c].tolist()
        runs = _runs(seg)
        ck = counts[c * T:(c + 1) * T]
        # repeating tiles, each in strided (strictly increasing) order
        assert len(runs) == ck.max()
        for r, run in enumerate(runs):
            assert run == (np.nonzero(ck > r)[0] + c * T).tolist()


def test_special_cases(orc):
    rng = np.random.default_rng(0)
    distinct = rng.permutation(1000).astype(np.int32)
    _, p_std = orc.sort_keys(distinct, orc.SORT_STANDARD)
    _, p_str = orc.sort_keys(distinct, orc.SORT_STRIDED)
    _, p_til = orc.sort_keys(distinct, orc.SORT_TILED, 10**6)
    assert (p_std == p_str).all() and (p_std == p_til).all()
    assert (distinct[p_std] == np.arange(1000)).all()
    same = np.full(777, 42, np.int32)
    for order in range(4):
        _, p = orc.sort_keys(same, order, 3)
        assert (p == np.arange(777)).all()
    nk, p = orc.sort_keys(np.zeros(0, np.int32), orc.SORT_TILED, 4)
    assert nk.size == 0 and p.size == 0


def test_standard_is_stable_textbook(orc):
    """Standard order == numpy's stable argsort (a library routine)."""
    rng = np.random.default_rng(9)
    keys = rng.integers(0, 50, 10000).astype(np.int32)
    _, p = orc.sort_keys(keys, orc.SORT_STANDARD)
    assert (p == np.argsort(keys, kind="stable")).all()


def test_new_keys_int64(orc):
    """Reading R5: the strided stride is max_k + 1 and keys are int64."""
    keys = np.array([2**30, 2**30, 2**30, 5], np.int32)
    nk, _ = orc.sort_keys(keys, orc.SORT_STRIDED)
    assert nk.tolist() == [2**30 - 5, 2**30 - 5 + (2**30 + 1), 2**30 - 5 + 2 * (2**30 + 1), 0]


def test_sort_particles_counts(orc):
    from paper_conf_sc_tanlta25_b200 import inputs
    g = inputs.GridSpec(4, 3, 2)
    p = inputs.random_particles(g, 500, 3)
    out, counts, nk, perm = orc.sort_particles(g, p, orc.SORT_STANDARD)
    assert (counts == np.bincount(p["i"], minlength=g.nv)).all()
    assert (out.view(np.uint8).reshape(-1, 32) == p[perm].view(np.uint8).reshape(-1, 32)).all()
    assert np.all(np.diff(out["i"]) >= 0)
