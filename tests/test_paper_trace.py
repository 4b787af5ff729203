"""Pin of the reconstructed operators (R6-R9) on the CPU.

A step-by-step, pure-Python transcription of the paper's three operators -- local sort
(Alg. 2), merge (Alg. 3) and rebuild (Alg. 4, index math
and direction rule verbatim, `@` read as XOR) -- must (a) reproduce every state of the
hand-worked top-4-of-16 trace (tests/golden/trace_top4_of_16.txt, Fig. 5 shape) and
(b) return exactly the oracle's top-k on random and 0-1 inputs (0-1 principle), for
every power-of-two k.  The GPU network (csrc/network.cuh) uses the same index math with
the mirrored direction convention (best-first run 0).

This file is test code only; it is not the oracle and not the product.
"""
import os

import numpy as np

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def worse(a, b):
    """x0 < x1 of Alg. 4 line 9 under the total order: a is worse than b."""
    (va, ia), (vb, ib) = a, b
    return va < vb or (va == vb and ia > ib)


def step(L, inc, dir_):
    n = len(L)
    for t in range(n // 2):
        low = t & (inc - 1)                 # Alg. 4 line 5
        i = (t << 1) - low                  # line 6
        reverse = (dir_ & i) == 0           # line 7
        x0, x1 = L[i], L[i + inc]           # line 8
        swap = reverse ^ worse(x0, x1)      # line 9 (XOR reading, R8)
        if swap:
            x0, x1 = x1, x0                 # line 10
        L[i], L[i + inc] = x0, x1           # line 11


def local_sort(L, k):                       # Alg. 2 (reconstructed)
    length = 1
    while length < k:
        inc = length
        while inc > 0:
            step(L, inc, length << 1)
            inc >>= 1
        length <<= 1


def merge(L, k):                            # Alg. 3 (reconstructed): keep the better
    out = []
    for t in range(len(L) // 2):
        i = (t << 1) - (t & (k - 1))
        a, b = L[i], L[i + k]
        out.append(a if worse(b, a) else b)
    return out


def rebuild(L, k):                          # Alg. 4
    inc = k >> 1
    while inc > 0:
        step(L, inc, k)
        inc >>= 1


def paper_topk(vals, k):
    L = [(v, i) for i, v in enumerate(vals)]
    states = []
    local_sort(L, k)
    states.append(list(L))
    while len(L) > k:
        L = merge(L, k)
        states.append(list(L))
        rebuild(L, k)
        states.append(list(L))
    return states, L[::-1]                  # final run is worst first


def parse(tok):
    v, i = tok.split("@")
    return (float(v), int(i))


def test_golden_trace_every_state():
    rows = {}
    with open(os.path.join(GOLDEN, "trace_top4_of_16.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            name, *vals = line.split()
            rows.setdefault(name, []).append(vals)
    k = int(rows["k"][0][0])
    vals = [parse(t)[0] for t in rows["input"][0]]
    states, result = paper_topk(vals, k)
    want = [rows["localsort"][0], rows["merge"][0], rows["rebuild"][0], rows["merge"][1],
            rows["rebuild"][1]]
    assert [[(v, i) for v, i in s] for s in states] == [[parse(t) for t in w] for w in want]
    assert result == [parse(t) for t in rows["result"][0]]


def test_operators_equal_oracle_random_and_01():
    rng = np.random.default_rng(2)
    for logn in range(0, 8):
        n = 1 << logn
        for logk in range(0, logn + 1):
            k = 1 << logk
            for trial in range(6):
                if trial < 3:
                    vals = rng.integers(0, 2, n).astype(np.float32)  # 0-1 principle
                else:
                    vals = rng.integers(0, 5, n).astype(np.float32)
                _, res = paper_topk(vals.tolist(), k)
                ov, oi = oracle.topk(vals, k, True)
                assert [i for _, i in res] == oi.tolist()
