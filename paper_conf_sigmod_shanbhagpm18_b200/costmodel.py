"""The paper's hardware-conscious cost model (§7), as host-side planning
arithmetic (no device work): predicted times of radix-select top-k (§7.1) and bitonic
top-k (§7.2) from the global-memory bandwidth B_G, the shared-memory bandwidth B_S, the
key width w, the data size D and the thread count n_t.

bench.py prints these predictions next to the measured times of topk_radix and topk
(SURVEY §2.1 A13/A14); ``choose`` is the model-based dispatch the paper's evaluation
implies (bitonic for small K, radix for large K).  Pinned in
tests/test_costmodel.py against the numbers P:341 prints (T_g = 8.96 ms on Titan X).
"""
from __future__ import annotations

import math
from dataclasses import dataclass


@dataclass
class Hardware:
    b_g: float    # global-memory bandwidth, bytes/s (P:309 B_G)
    b_s: float    # shared-memory bandwidth, bytes/s (P:309 B_S)
    n_t: int      # threads in flight (P:309 n_t)


# Titan X Maxwell as the paper measured it: B_S = 2.9 TBps, B_G = 251 GBps.
TITAN_X = Hardware(b_g=251 * 2**30, b_s=2.9e12, n_t=24 * 2048)


def b200(hbm_gbs: float, sm_clock_ghz: float = 1.965, sms: int = 148) -> Hardware:
    """B200: measured HBM bandwidth; smem 128 B/clk/SM (32 banks x 4 B)."""
    return Hardware(b_g=hbm_gbs * 1e9, b_s=sms * 128 * sm_clock_ghz * 1e9, n_t=sms * 2048)


def radix_passes(n: int, w: int, etas: list[float] | None = None) -> list[tuple[float, float]]:
    """(D_i1, eta_i) for each pass: D_11 = D, then D_(i+1)1 = eta_i * D_i1.
    ``etas`` default: uniform keys, each 8-bit digit keeps 1/256 of the candidates."""
    npass = w  # one pass per 8-bit digit: w bytes ("at most w/8" for w in bits)
    etas = etas if etas is not None else [1.0 / 256] * npass
    d = float(n * w)
    out = []
    for i in range(npass):
        out.append((d, etas[i]))
        d *= etas[i]
    return out


def radix_time(n: int, w: int, hw: Hardware, etas: list[float] | None = None) -> float:
    """§7.1: T = sum_i T_i1 + T_i2 + T_i3."""
    t = 0.0
    hist = 16 * 4 * hw.n_t  # "16 integers per thread"
    for d, eta in radix_passes(n, w, etas):
        t += d / hw.b_g + hist / hw.b_g               # T_i1: read + per-thread counts
        t += 2 * hist / hw.b_g                         # T_i2: prefix sum
        if eta < 1.0:                                  # T_i3 (skipped if eta = 1)
            t += d / hw.b_g + eta * d / hw.b_g
    return t


def bitonic_tg(n: int, w: int, hw: Hardware, x: int = 8) -> float:
    """§7.2 global-memory term of the SortReducer: T_g = D/B_G + D/(x B_G)."""
    d = n * w
    return d / hw.b_g + d / (x * hw.b_g)


def sortreducer_smem_factor(k: int) -> float:
    """The bank-conflict-weighted step sum of T_k = f * D / B_S.  The paper prints
    f = 17.5 for top-32; other K scale with the combined-step count of the
    local sort + merges, (L+1)(L+2)/2, normalised to that point."""
    L = max(0, int(math.log2(k)))
    return 17.5 * ((L + 1) * (L + 2) / 2) / 21.0


def bitonic_time(n: int, w: int, k: int, hw: Hardware, x: int = 8) -> float:
    """§7.2: max(T_g, T_k) for the SortReducer; the BitonicReducers work on
    D/x and are folded in as a geometric tail (x / (x - 1))."""
    tk = sortreducer_smem_factor(k) * n * w / hw.b_s
    return max(bitonic_tg(n, w, hw, x), tk) * (x / (x - 1))


def choose(n: int, w: int, k: int, hw: Hardware) -> str:
    """Model-based dispatch (the paper's models): the smaller predicted time."""
    return "bitonic" if bitonic_time(n, w, k, hw) <= radix_time(n, w, hw) else "radix"


def bitonic_b200_time(n: int, w: int, hw: Hardware) -> float:
    """This repo's B200 pass: every key read from HBM once, the network
    run on the buffer filler's survivors only (~0.1 % of the keys on uniform data), the
    intermediate runs on chip / in L2 -- bounded below by T_g's first term, D / B_G.
    The paper's T_k (every key through shared memory) no longer applies."""
    return n * w / hw.b_g


def choose_b200(n: int, w: int, k: int, hw: Hardware) -> str:
    """Dispatch with the B200 bitonic model against the paper's radix model."""
    return "bitonic" if bitonic_b200_time(n, w, hw) <= radix_time(n, w, hw) else "radix"
