"""Seeded synthetic inputs shared by the CUDA path's tests/bench and by the oracle.

This module holds NO top-k arithmetic: it only defines the inputs (DESIGN.md §3,
"Input recipe").  It is plain PyTorch integer code that runs identically on the CPU
and on a CUDA device, so the oracle (host) and the kernels (device) see bit-identical
keys; ``tests/test_datagen.py`` pins it against a pure-Python splitmix64 and, on the
GPU, device output against host output.

Counter-based generator: row ``i`` of a stream with seed ``s`` is
``z_i = splitmix64_mix(s + GAMMA * (i + 1))`` -- the standard splitmix64 output
sequence -- so any shard ``[base, base + n)`` can be generated independently.

Distributions (the paper's workloads):
  * ``uniform``     f32 U(0,1) on a 2^-24 grid: ``(z >> 40) * 2^-24``
  * ``uniform``     u32 U(0, 2^32-1): ``z >> 32``
  * ``uniform``     f64 U(0,1): ``(z >> 11) * 2^-53``
  * ``increasing``  sorted U(0,1) as the closed-form ramp floor(i*2^24/n)*2^-24
  * ``decreasing``  its mirror
  * ``fewdistinct`` 16 distinct values (z % 16) / 16 ("many duplicates", BJ cfg 3)
  * ``bucketkiller`` all 1.0 except 4 keys that each differ in one 8-bit digit
"""
from __future__ import annotations

import torch

GAMMA = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB
_CHUNK = 1 << 24

DISTS = ("uniform", "increasing", "decreasing", "fewdistinct", "bucketkiller")
DTYPES = {"f32": torch.float32, "u32": torch.uint32, "f64": torch.float64}


def _s64(v: int) -> int:
    v &= (1 << 64) - 1
    return v - (1 << 64) if v >= 1 << 63 else v


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 lanes holding uint64 bit patterns."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def mix(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 output function on int64 lanes (two's-complement wraparound)."""
    x = (x ^ _srl(x, 30)) * _s64(_M1)
    x = (x ^ _srl(x, 27)) * _s64(_M2)
    return x ^ _srl(x, 31)


def stream(seed: int, lo: int, hi: int, device) -> torch.Tensor:
    """z_i for rows i in [lo, hi) as int64 bit patterns."""
    i = torch.arange(lo, hi, dtype=torch.int64, device=device)
    return mix((i + 1) * _s64(GAMMA) + _s64(seed))


def _f32_from_grid(g: torch.Tensor) -> torch.Tensor:
    # g in [0, 2^24): exact in float32
    return g.to(torch.float32) * (2.0 ** -24)


def _fill(dist: str, dtype: str, seed: int, n_total: int, lo: int, hi: int, device):
    if dist == "uniform":
        z = stream(seed, lo, hi, device)
        if dtype == "f32":
            return _f32_from_grid(_srl(z, 40))
        if dtype == "u32":
            return _srl(z, 32).to(torch.uint32)
        return _srl(z, 11).to(torch.float64) * (2.0 ** -53)
    if dist in ("increasing", "decreasing"):
        i = torch.arange(lo, hi, dtype=torch.int64, device=device)
        if dist == "decreasing":
            i = (n_total - 1) - i
        if dtype == "u32":
            return i.to(torch.uint32)  # distinct keys: key = rank
        g = (i << 24) // n_total
        if dtype == "f32":
            return _f32_from_grid(g)
        return g.to(torch.float64) * (2.0 ** -24)
    if dist == "fewdistinct":
        z = stream(seed, lo, hi, device)
        v = z & 15
        if dtype == "u32":
            return v.to(torch.uint32)
        return (v.to(torch.float64) / 16.0).to(DTYPES[dtype])
    raise ValueError(dist)


def bucketkiller_specials(seed: int, n_total: int):
    """Positions and bit patterns of the 4 non-1.0 keys (reading R12).

    Key j replaces byte j of 1.0f (0x3F800000) by (byte XOR 0x5A): 0x3F80005A,
    0x3F805A00, 0x3FDA0000, 0x65800000 -- all > 1.0 ("each of which differ from
    1.0 in one 8-bit digit")."""
    z = stream(seed ^ 0xB0C4E7, 0, 4, "cpu")
    pos = [int(_srl(z[j:j + 1], 1).item()) % n_total for j in range(4)]
    bits = []
    for j in range(4):
        b = (0x3F800000 >> (8 * j)) & 0xFF
        bits.append((0x3F800000 & ~(0xFF << (8 * j))) | ((b ^ 0x5A) << (8 * j)))
    return pos, bits


def generate(dist: str, n: int, dtype: str = "f32", seed: int = 0x5EED0001, device="cpu",
             base: int = 0, n_total: int | None = None, out: torch.Tensor | None = None
             ) -> torch.Tensor:
    """Rows [base, base + n) of the global input of length ``n_total`` (default n)."""
    if n_total is None:
        n_total = base + n
    if out is None:
        out = torch.empty(n, dtype=DTYPES[dtype], device=device)
    if dist == "bucketkiller":
        if dtype != "f32":
            raise ValueError("bucketkiller is defined for f32 (P:262)")
        out.fill_(1.0)
        pos, bits = bucketkiller_specials(seed, n_total)
        for p, b in zip(pos, bits):
            if base <= p < base + n:
                out[p - base] = torch.tensor([b], dtype=torch.int32).view(torch.float32)[0]
        return out
    for lo in range(0, n, _CHUNK):
        hi = min(n, lo + _CHUNK)
        out[lo:hi] = _fill(dist, dtype, seed, n_total, base + lo, base + hi, out.device)
    return out


def payload(n: int, seed: int = 0x5EED0001, device="cpu", base: int = 0) -> torch.Tensor:
    """KV payload (32-bit row id stand-in, != the index so tests can tell them apart)."""
    out = torch.empty(n, dtype=torch.uint32, device=device)
    for lo in range(0, n, _CHUNK):
        hi = min(n, lo + _CHUNK)
        out[lo:hi] = _srl(stream(seed ^ 0x7A7A7A7A, base + lo, base + hi, out.device), 32
                          ).to(torch.uint32)
    return out


def config_seed(config_id: int, run: int = 0) -> int:
    """Seeds 0x5EED0001 + 16*config + run."""
    return 0x5EED0001 + 16 * config_id + run
