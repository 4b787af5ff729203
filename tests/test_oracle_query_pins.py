"""Pins of the oracle's query form (oracle.query: WHERE predicate, ORDER BY a ranking
function, LIMIT k -- the paper's §5 database integration, queries 1-3 of
§6.8; readings R17/R18).  CPU only.

Independent references:
  * numpy does the filter (boolean mask / numpy.isin) and the projection (float32
    ufuncs, each operation rounded to float32), torch.sort(stable=True) the ordering
    (NaN greatest, -0 == +0, ties by position) -- no code shared with the oracle;
  * closed forms: selectivity 0 (no rows), a range over a row-id column (= the top-k of
    a slice, with its base), integer-valued ranking columns where a + w*b is exact and
    equals the float64 value, w = 0 (f = a).
A dropped predicate, an inverted range bound, a wrong IN bit, a transposed ranking
operand or a missing weight fails at least one of these.
"""
import numpy as np
import pytest
import torch

import oracle


def lib_query(a, k, largest, rank_b=None, w=0.0, keep=None):
    """numpy filter + projection, torch stable sort; indices refer to the input rows."""
    rows = np.arange(a.shape[0], dtype=np.int64)
    f = a if rank_b is None else (a + np.float32(w) * rank_b).astype(np.float32)
    if rank_b is not None:  # R18: computed NaNs are the canonical quiet NaN
        f = f.copy()
        f[np.isnan(f)] = np.uint32(0x7FC00000).view(np.float32)
    if keep is not None:
        rows, f = rows[keep], f[keep]
    m = min(k, rows.shape[0])
    if m == 0:
        return f[:0], rows[:0]
    _, order = torch.sort(torch.from_numpy(f.astype(np.float64) if f.dtype == np.uint32 else f),
                          stable=True, descending=largest)
    order = order[:m].numpy()
    return f[order], rows[order]


def check(a, k, largest, rank_b=None, w=0.0, pred=None, keep=None):
    v, i, m = oracle.query(a, k, largest, rank_b=rank_b, rank_w=w, pred=pred)
    rv, ri = lib_query(a, k, largest, rank_b, w, keep)
    assert m == ri.shape[0]
    assert np.array_equal(i[:m], ri), (i[:m], ri)
    assert v[:m].tobytes() == rv.tobytes()
    assert np.all(i[m:] == -1)
    assert not np.any(v[m:].view(np.uint8))


@pytest.mark.parametrize("largest", [True, False])
@pytest.mark.parametrize("dtype", [np.float32, np.uint32, np.float64])
def test_range_predicate_vs_numpy(largest, dtype):
    rng = np.random.default_rng(11)
    n = 5000
    if dtype == np.uint32:
        a = rng.integers(0, 50, n).astype(np.uint32)  # heavy ties
    else:
        a = (rng.integers(0, 1 << 10, n) / 1024.0).astype(dtype)
    col = rng.integers(0, 1000, n).astype(np.uint32)
    for lo, hi in [(0, 1000), (100, 400), (999, 1000), (500, 500), (0, 1)]:
        keep = (col >= lo) & (col < hi)
        for k in (1, 7, 64, 300):
            check(a, k, largest, pred=("range", col, lo, hi), keep=keep)


@pytest.mark.parametrize("largest", [True, False])
def test_in_predicate_vs_numpy(largest):
    rng = np.random.default_rng(12)
    n = 4000
    a = rng.random(n, dtype=np.float32)
    col = rng.integers(0, 80, n).astype(np.uint32)  # codes >= 64 never match
    for cats in ([3, 5], [0], [63], list(range(64)), [70]):
        mask = 0
        for c in cats:
            if c < 64:
                mask |= 1 << c
        keep = np.isin(col, [c for c in cats if c < 64])
        for k in (1, 50, 256):
            check(a, k, largest, pred=("in", col, mask), keep=keep)


@pytest.mark.parametrize("largest", [True, False])
def test_ranking_function_vs_numpy(largest):
    rng = np.random.default_rng(13)
    n = 6000
    a = rng.random(n, dtype=np.float32)
    b = rng.random(n, dtype=np.float32) * 3
    a[:8] = [np.nan, -0.0, 0.0, np.inf, -np.inf, 1e-40, -1e-40, 2.0]
    b[:8] = [1.0, 0.0, -0.0, -1.0, 5.0, 1e-40, 0.0, np.nan]
    for w in (0.5, -1.25, 3.0e-3):
        for k in (1, 32, 500):
            check(a, k, largest, rank_b=b, w=w)
    col = rng.integers(0, 10, n).astype(np.uint32)
    check(a, 64, largest, rank_b=b, w=0.5, pred=("range", col, 2, 7), keep=(col >= 2) & (col < 7))


def test_integer_ranking_is_exact():
    """retweet_count + 0.5 * likes_count on integer counts: exact in float32
    below 2^23, so the float64 value sorted by numpy.lexsort is the closed form."""
    rng = np.random.default_rng(14)
    n = 3000
    a = rng.integers(0, 1000, n).astype(np.float32)
    b = rng.integers(0, 1000, n).astype(np.float32)
    f64 = a.astype(np.float64) + 0.5 * b.astype(np.float64)
    order = np.lexsort((np.arange(n), -f64))[:100]
    v, i, m = oracle.query(a, 100, True, rank_b=b, rank_w=0.5)
    assert m == 100 and np.array_equal(i, order)
    assert np.array_equal(v.astype(np.float64), f64[order])
    # transposed operands give a different answer (the pin can see it)
    _, i2, _ = oracle.query(b, 100, True, rank_b=a, rank_w=0.5)
    assert not np.array_equal(i2, order)


def test_closed_forms():
    rng = np.random.default_rng(15)
    n = 10000
    a = rng.random(n, dtype=np.float32)
    rowid = np.arange(n, dtype=np.uint32)
    # selectivity 0: no result rows
    v, i, m = oracle.query(a, 10, True, pred=("range", rowid, 5, 5))
    assert m == 0 and np.all(i == -1) and not np.any(v.view(np.uint8))
    v, i, m = oracle.query(a, 10, True, pred=("in", rowid, 0))
    assert m == 0
    # a range over the row id = the top-k of a slice with base lo
    lo, hi = 1234, 5678
    v, i, m = oracle.query(a, 40, True, pred=("range", rowid, lo, hi))
    sv, si = oracle.topk(a[lo:hi], 40, True, base=lo)
    assert m == 40 and np.array_equal(i, si) and v.tobytes() == sv.tobytes()
    # fewer matches than k: every match, best first, then -1
    v, i, m = oracle.query(a, 50, False, pred=("range", rowid, 100, 120))
    assert m == 20 and np.array_equal(np.sort(i[:20]), np.arange(100, 120))
    assert np.all(np.diff(v[:20]) >= 0) and np.all(i[20:] == -1)
    # w = 0 with non-negative finite b: f = a exactly
    b = rng.random(n, dtype=np.float32)
    v, i, m = oracle.query(a, 64, True, rank_b=b, rank_w=0.0)
    sv, si = oracle.topk(a, 64, True)
    assert np.array_equal(i, si) and v.tobytes() == sv.tobytes()


# ---- compound keys (KKV; R19) ----

def lex_ref(k1, k2, k, l1, l2):
    """numpy.lexsort (last key primary) on NaN-free columns: the library pin."""
    s1 = -k1.astype(np.float64) if l1 else k1.astype(np.float64)
    s2 = -k2.astype(np.float64) if l2 else k2.astype(np.float64)
    order = np.lexsort((np.arange(k1.shape[0]), s2, s1))[:k]
    return order


@pytest.mark.parametrize("l1", [True, False])
@pytest.mark.parametrize("l2", [True, False])
def test_compound_keys_vs_lexsort(l1, l2):
    rng = np.random.default_rng(21)
    n = 5000
    k1 = (rng.integers(0, 40, n) / 8).astype(np.float32)  # heavy ties on the first key
    k2 = (rng.integers(0, 1 << 12, n) / 4096).astype(np.float32)
    k2[::7] = k2[3]  # ties on both keys -> the row id decides
    for k in (1, 10, 100, 1000):
        v1, v2, i = oracle.topk_kk(k1, k2, k, l1, l2)
        ref = lex_ref(k1, k2, k, l1, l2)
        assert np.array_equal(i, ref)
        assert v1.tobytes() == k1[ref].tobytes() and v2.tobytes() == k2[ref].tobytes()


def test_compound_keys_special_values_brute_force():
    """Tiny inputs over special floats vs Python's sort of (code1, code2, -idx) tuples
    built from torch's stable sort ranks (an independent order for NaN / -0)."""
    sp = np.array([np.nan, -np.inf, -0.0, 0.0, 1.0, np.inf], dtype=np.float32)
    rng = np.random.default_rng(22)
    for trial in range(200):
        n = int(rng.integers(1, 12))
        k1 = sp[rng.integers(0, sp.shape[0], n)]
        k2 = sp[rng.integers(0, sp.shape[0], n)]
        # dense rank of each value under "NaN greatest, -0 == +0" via torch.sort
        def rank(a):
            t = torch.from_numpy(a)
            _, order = torch.sort(t, stable=True)
            r = np.empty(n, dtype=np.int64)
            cur = -1
            prev = None
            for pos in order.numpy():
                x = a[pos]
                same = prev is not None and ((np.isnan(x) and np.isnan(prev)) or x == prev)
                if not same:
                    cur += 1
                r[pos] = cur
                prev = x
            return r
        r1, r2 = rank(k1), rank(k2)
        for l1 in (True, False):
            for l2 in (True, False):
                key = sorted(range(n), key=lambda i: ((-r1[i]) if l1 else r1[i],
                                                      (-r2[i]) if l2 else r2[i], i))
                k = int(rng.integers(1, n + 1))
                _, _, i = oracle.topk_kk(k1, k2, k, l1, l2)
                assert list(i) == key[:k], (k1, k2, l1, l2)


def test_compound_keys_reduce_to_single_key():
    """Constant second key: the single-key oracle (pinned above) decides."""
    rng = np.random.default_rng(23)
    k1 = rng.random(3000, dtype=np.float32)
    k2 = np.full(3000, 0.25, dtype=np.float32)
    for l1 in (True, False):
        _, _, i = oracle.topk_kk(k1, k2, 64, l1, True)
        _, si = oracle.topk(k1, 64, l1)
        assert np.array_equal(i, si)


@pytest.mark.parametrize("orders", [(True, True, True), (False, True, False), (True, False, True)])
def test_three_keys_vs_lexsort(orders):
    """KKKV: numpy.lexsort on three NaN-free tie-heavy columns."""
    rng = np.random.default_rng(24)
    n = 4000
    cols = [(rng.integers(0, m, n) / m).astype(np.float32) for m in (6, 5, 50)]
    sk = [-c.astype(np.float64) if l else c.astype(np.float64) for c, l in zip(cols, orders)]
    for k in (1, 17, 300, 2048):
        ref = np.lexsort((np.arange(n), sk[2], sk[1], sk[0]))[:k]
        v1, v2, v3, i = oracle.topk_kkk(*cols, k, orders)
        assert np.array_equal(i, ref)
        assert v3.tobytes() == cols[2][ref].tobytes()


def test_three_keys_reduce_to_two():
    """A constant third key: the (pinned) two-key oracle decides."""
    rng = np.random.default_rng(25)
    a = (rng.integers(0, 9, 3000) / 9).astype(np.float32)
    b = rng.random(3000, dtype=np.float32)
    c = np.zeros(3000, dtype=np.float32)
    _, _, _, i = oracle.topk_kkk(a, b, c, 100, (True, False, True))
    _, _, i2 = oracle.topk_kk(a, b, 100, True, False)
    assert np.array_equal(i, i2)
