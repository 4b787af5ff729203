"""CPU oracle for bitonic top-k -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference`` arm) may import this package.  The product package
``paper_conf_sigmod_shanbhagpm18_b200`` never imports it and has no CPU fallback.

The arithmetic lives in ``topk_oracle.cpp`` (plain C++17, std::partial_sort under the
total order of DESIGN.md R1-R4; see its header for the paper passages it follows).
This module only marshals numpy arrays through ctypes.

Parity status: every function here is pinned by ``tests/test_oracle_pins.py``
(brute force, library sorts, closed forms, the paper-shaped golden trace); none is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "topk_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

DT_F32, DT_U32, DT_F64 = 0, 1, 2
_NP2DT = {np.dtype(np.float32): DT_F32, np.dtype(np.uint32): DT_U32, np.dtype(np.float64): DT_F64}

_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with g++ (no CUDA).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-shared",
                               "-fPIC", "-pthread",
                               "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        lib.oracle_topk.argtypes = [i32, vp, vp, u64, u64, u32, i32, vp, vp, i32]
        lib.oracle_topk.restype = i32
        lib.oracle_certificate.argtypes = [i32, vp, u64, u64, u32, i32, vp, vp]
        lib.oracle_certificate.restype = i32
        lib.oracle_codes.argtypes = [i32, vp, u64, i32, vp]
        lib.oracle_codes.restype = None
        lib.oracle_query.argtypes = [i32, vp, vp, ctypes.c_float, i32, vp, u32, u32, u64, u64,
                                     u32, i32, vp, vp, i32]
        lib.oracle_query.restype = i32
        lib.oracle_topk_kk.argtypes = [vp, vp, u64, u32, i32, i32, vp, vp, vp]
        lib.oracle_topk_kk.restype = i32
        lib.oracle_topk_kkk.argtypes = [vp, vp, vp, u64, u32, i32, i32, i32, vp, vp, vp, vp]
        lib.oracle_topk_kkk.restype = i32
        lib.oracle_threads.argtypes = []
        lib.oracle_threads.restype = i32
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def topk(keys: np.ndarray, k: int, largest: bool = True, base: int = 0,
         idx: np.ndarray | None = None, threads: int = 0):
    """Exact top-k of ``keys`` (1-D float32 / uint32 / float64), best first.

    Returns ``(values, indices)``; indices are ``base + row`` (int64) unless an explicit
    ``idx`` array (int64, same length) supplies the source index of every row.
    """
    keys = np.ascontiguousarray(keys)
    dt = _NP2DT[keys.dtype]
    n = keys.shape[0]
    if idx is not None:
        idx = np.ascontiguousarray(idx, dtype=np.int64)
        assert idx.shape[0] == n
    out_k = np.empty(k, dtype=keys.dtype)
    out_i = np.empty(k, dtype=np.int64)
    r = _load().oracle_topk(dt, _ptr(keys), _ptr(idx), n, base, k, 0 if largest else 1,
                            _ptr(out_k), _ptr(out_i), threads)
    if r < 0:
        raise ValueError(f"oracle_topk: invalid arguments (n={n}, k={k})")
    return out_k, out_i


PRED_NONE, PRED_RANGE, PRED_IN = 0, 1, 2


def query(keys: np.ndarray, k: int, largest: bool = True, rank_b: np.ndarray | None = None,
          rank_w: float = 0.0, pred: tuple | None = None, threads: int = 0):
    """``SELECT WHERE pred ORDER BY f LIMIT k`` (R17/R18).

    ``pred``: None, ``("range", col_u32, lo, hi)`` (lo <= col < hi) or
    ``("in", col_u32, mask64)`` (col < 64 and bit col of mask).  ``rank_b``: None
    (f = keys) or a float32 column (f = keys + rank_w * rank_b, each op rounded to f32).
    Returns ``(values, indices, m)``: m = result rows (<= k); rows j >= m have index -1
    and zero key bits.
    """
    keys = np.ascontiguousarray(keys)
    dt = _NP2DT[keys.dtype]
    n = keys.shape[0]
    kind, col, lo, hi, mask = PRED_NONE, None, 0, 0, 0
    if pred is not None:
        if pred[0] == "range":
            kind, col, lo, hi = PRED_RANGE, pred[1], int(pred[2]), int(pred[3])
        elif pred[0] == "in":
            kind, col, mask = PRED_IN, pred[1], int(pred[2])
        else:
            raise ValueError(pred[0])
        col = np.ascontiguousarray(col, dtype=np.uint32)
        assert col.shape[0] == n
    if rank_b is not None:
        rank_b = np.ascontiguousarray(rank_b, dtype=np.float32)
        assert rank_b.shape[0] == n
    out_k = np.empty(k, dtype=keys.dtype)
    out_i = np.empty(k, dtype=np.int64)
    m = _load().oracle_query(dt, _ptr(keys), _ptr(rank_b), float(rank_w), kind, _ptr(col),
                             lo, hi, mask, n, k, 0 if largest else 1, _ptr(out_k), _ptr(out_i),
                             threads)
    if m < 0:
        raise ValueError("oracle_query: invalid arguments")
    return out_k, out_i, m


def topk_kk(k1: np.ndarray, k2: np.ndarray, k: int, largest1: bool = True,
            largest2: bool = True):
    """Compound-key top-k (ORDER BY k1, k2 LIMIT k; KKV): lexicographic on
    the two float32 columns' order codes, then the lowest row id.  Returns
    ``(v1, v2, indices)``."""
    k1 = np.ascontiguousarray(k1, dtype=np.float32)
    k2 = np.ascontiguousarray(k2, dtype=np.float32)
    assert k1.shape == k2.shape
    o1 = np.empty(k, dtype=np.float32)
    o2 = np.empty(k, dtype=np.float32)
    oi = np.empty(k, dtype=np.int64)
    r = _load().oracle_topk_kk(_ptr(k1), _ptr(k2), k1.shape[0], k, 0 if largest1 else 1,
                               0 if largest2 else 1, _ptr(o1), _ptr(o2), _ptr(oi))
    if r < 0:
        raise ValueError("oracle_topk_kk: invalid arguments")
    return o1, o2, oi


def topk_kkk(k1, k2, k3, k: int, largest=(True, True, True)):
    """Three compound keys (KKKV): ORDER BY k1, k2, k3 LIMIT k.  Returns
    ``(v1, v2, v3, indices)``."""
    cols = [np.ascontiguousarray(c, dtype=np.float32) for c in (k1, k2, k3)]
    assert cols[0].shape == cols[1].shape == cols[2].shape
    outs = [np.empty(k, dtype=np.float32) for _ in range(3)]
    oi = np.empty(k, dtype=np.int64)
    r = _load().oracle_topk_kkk(*[_ptr(c) for c in cols], cols[0].shape[0], k,
                                *[0 if l else 1 for l in largest], *[_ptr(o) for o in outs],
                                _ptr(oi))
    if r < 0:
        raise ValueError("oracle_topk_kkk: invalid arguments")
    return outs[0], outs[1], outs[2], oi


def certificate(keys: np.ndarray, k: int, out_keys: np.ndarray, out_idx: np.ndarray,
                largest: bool = True, base: int = 0) -> int:
    """O(n) check that (out_keys, out_idx) is exactly the top-k; 0 = certified."""
    keys = np.ascontiguousarray(keys)
    out_keys = np.ascontiguousarray(out_keys, dtype=keys.dtype)
    out_idx = np.ascontiguousarray(out_idx, dtype=np.int64)
    return _load().oracle_certificate(_NP2DT[keys.dtype], _ptr(keys), keys.shape[0], base, k,
                                      0 if largest else 1, _ptr(out_keys), _ptr(out_idx))


def codes(keys: np.ndarray, largest: bool = True) -> np.ndarray:
    """The oracle's order code of every key (uint64; larger = better)."""
    keys = np.ascontiguousarray(keys)
    out = np.empty(keys.shape[0], dtype=np.uint64)
    _load().oracle_codes(_NP2DT[keys.dtype], _ptr(keys), keys.shape[0], 0 if largest else 1,
                         _ptr(out))
    return out


def threads() -> int:
    """Host threads the oracle uses by default (the process affinity mask)."""
    return _load().oracle_threads()
