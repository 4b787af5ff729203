"""B200-native bitonic top-k (Shanbhag, Pirk, Madden, SIGMOD 2018).

Thin Python binding over the C ABI in ``include/topk.h`` (``libtopk_b200.so``): the
functions below only marshal torch tensors (device memory, current stream) into the
C calls; every step of the top-k runs in the library's sm_100a kernels.

    values, indices = topk(x, k, largest=True)          # x: 1-D cuda f32/u32/f64
    values, indices, pay = topk(x, k, payload=p)        # key + 32-bit payload
    values, indices = merge(cand_vals, cand_idx, k)     # global step
    values, indices = query(a, k, rank_b=b, rank_w=0.5, pred=("range", t, 0, X))
                                                        # WHERE / ORDER BY f(A1, A2)
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib

__all__ = ["topk", "topk_host", "merge", "query", "topk_kk", "topk_kkk", "topk_radix", "Workspace", "launch_count", "workspace_bytes"]

_DT = {torch.float32: _lib.F32, torch.uint32: _lib.U32, torch.float64: _lib.F64}


def _dtype_code(t: torch.Tensor) -> int:
    try:
        return _DT[t.dtype]
    except KeyError:
        raise TypeError(f"unsupported key dtype {t.dtype} (float32, uint32, float64)") from None


def _stream_ptr(device) -> ctypes.c_void_p:
    return ctypes.c_void_p(torch.cuda.current_stream(device).cuda_stream)


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def _check_col(t, n, dtype, device, what):
    """A CUDA column the kernels read: dtype, length, device and layout are checked here,
    so a wrong tensor raises instead of turning into an out-of-bounds device access."""
    if t is None:
        return None
    if not t.is_cuda or t.device != device:
        raise ValueError(f"{what}: must be a CUDA tensor on {device}")
    if t.dtype != dtype or t.dim() != 1 or t.shape[0] != n:
        raise ValueError(f"{what}: expected a 1-D {dtype} tensor of length {n}")
    return t.contiguous()


def _check_out(t, k, dtype, device, what):
    if t is None:
        return None
    if not t.is_cuda or t.device != device or t.dtype != dtype or t.numel() < k \
            or not t.is_contiguous():
        raise ValueError(f"{what}: expected a contiguous CUDA {dtype} tensor of >= {k} "
                         f"elements on {device}")
    return t


def workspace_bytes(dtype: torch.dtype, n: int, k: int) -> int:
    return int(_lib.load().topk_workspace_bytes(_DT[dtype], n, k))


class Workspace:
    """Device workspace for topk() (zero-filled once; each call leaves it zeroed).
    Must not be shared by concurrent calls on different streams."""

    def __init__(self, nbytes: int, device):
        self.nbytes = max(256, int(nbytes))
        self.buf = torch.zeros(self.nbytes, dtype=torch.uint8, device=device)

    def ptr(self):
        return ctypes.c_void_p(self.buf.data_ptr())


_ws_cache: dict = {}


def _workspace(device, nbytes: int) -> Workspace:
    key = (device.index, torch.cuda.current_stream(device).cuda_stream)
    ws = _ws_cache.get(key)
    if ws is None or ws.nbytes < nbytes:
        ws = Workspace(max(nbytes, 1 << 20), device)
        _ws_cache[key] = ws
    return ws


def topk(x: torch.Tensor, k: int, largest: bool = True, payload: torch.Tensor | None = None,
         base: int = 0, mode: str = "filter", out=None, workspace: Workspace | None = None):
    """Exact top-k of a 1-D CUDA tensor, best first; ties -> lowest index.

    Returns ``(values, indices)`` or ``(values, indices, payload_out)``; indices are
    ``base + position`` as int64.  ``mode``: "filter" (default) or "pure" (the paper's
    data-independent network on every key); both give identical results.
    """
    if not x.is_cuda or x.dim() != 1:
        raise ValueError("topk expects a 1-D CUDA tensor (no CPU path)")
    lib = _lib.load()
    dt = _dtype_code(x)
    n = x.shape[0]
    x = x if x.is_contiguous() else x.contiguous()
    if mode not in ("filter", "pure"):
        raise ValueError(f"mode must be 'filter' or 'pure', not {mode!r}")
    dev = x.device
    payload = _check_col(payload, n, torch.uint32, dev, "payload")
    if out is None:
        vals = torch.empty(k, dtype=x.dtype, device=dev)
        idx = torch.empty(k, dtype=torch.int64, device=dev)
        pay = torch.empty(k, dtype=torch.uint32, device=dev) if payload is not None else None
    else:
        vals, idx, pay = out
        vals = _check_out(vals, k, x.dtype, dev, "out values")
        idx = _check_out(idx, k, torch.int64, dev, "out indices")
        pay = _check_out(pay, k, torch.uint32, dev, "out payload")
        if pay is not None and payload is None:
            raise ValueError("out payload given without an input payload")
    with torch.cuda.device(dev):
        need = int(lib.topk_workspace_bytes(dt, n, k))
        if need == 0:
            raise _lib.TopkError(f"invalid arguments for topk (n={n}, k={k})")
        ws = workspace if workspace is not None else _workspace(dev, need)
        st = lib.topk_select(dt, _ptr(x), _ptr(payload), n, base, k,
                             _lib.LARGEST if largest else _lib.SMALLEST,
                             _lib.MODE_FILTER if mode == "filter" else _lib.MODE_PURE,
                             _ptr(vals), _ptr(pay), _ptr(idx), ws.ptr(), ws.nbytes,
                             _stream_ptr(dev))
    _lib.check(st, "topk_select")
    return (vals, idx) if payload is None else (vals, idx, pay)


def query(keys: torch.Tensor, k: int, largest: bool = True, rank_b: torch.Tensor | None = None,
          rank_w: float = 0.0, pred: tuple | None = None, payload: torch.Tensor | None = None,
          workspace: Workspace | None = None):
    """``SELECT WHERE pred ORDER BY f DESC|ASC LIMIT k`` fused into one streaming pass
    (the paper's §5: filter as the buffer filler, ranking function inside the pass).

    ``pred``: ``("range", col, lo, hi)`` (lo <= col < hi) or ``("in", col, mask64)``
    (col < 64 and bit col of mask); ``col`` a CUDA uint32 tensor.  ``rank_b``: None
    (f = keys) or a CUDA float32 tensor (f = keys + rank_w * rank_b, f32, each op
    rounded).  Every column 16-byte aligned.  Returns ``(values, indices)`` or
    ``(values, indices, payload_out)``; rows beyond the matches have index -1.
    """
    if not keys.is_cuda or keys.dim() != 1:
        raise ValueError("query expects 1-D CUDA tensors (no CPU path)")
    lib = _lib.load()
    dt = _dtype_code(keys)
    n = keys.shape[0]
    cols = [keys]
    pr = None
    if pred is not None:
        if pred[0] == "range":
            pr = _lib.Pred(_lib.PRED_RANGE, pred[1].data_ptr(), int(pred[2]), int(pred[3]), 0)
        elif pred[0] == "in":
            pr = _lib.Pred(_lib.PRED_IN, pred[1].data_ptr(), 0, 0, int(pred[2]))
        else:
            raise ValueError(f"unknown predicate kind {pred[0]!r}")
        if pred[1].dtype != torch.uint32 or pred[1].shape[0] != n or not pred[1].is_contiguous():
            raise ValueError("predicate column: contiguous CUDA uint32 of the same length")
        cols.append(pred[1])
    if rank_b is not None:
        if rank_b.dtype != torch.float32 or rank_b.shape[0] != n or not rank_b.is_contiguous():
            raise ValueError("rank_b: contiguous CUDA float32 of the same length")
        cols.append(rank_b)
    if payload is not None:
        payload = _check_col(payload, n, torch.uint32, keys.device, "payload")
        cols.append(payload)
    if any(not c.is_contiguous() or c.device != keys.device for c in cols):
        raise ValueError("columns must be contiguous and on the keys' device")
    vals = torch.empty(k, dtype=keys.dtype, device=keys.device)
    idx = torch.empty(k, dtype=torch.int64, device=keys.device)
    pay = torch.empty(k, dtype=torch.uint32, device=keys.device) if payload is not None else None
    with torch.cuda.device(keys.device):
        need = int(lib.topk_workspace_bytes(dt, n, k))
        if need == 0:
            raise _lib.TopkError(f"invalid arguments for query (n={n}, k={k})")
        ws = workspace if workspace is not None else _workspace(keys.device, need)
        st = lib.topk_query(dt, _ptr(keys), _ptr(rank_b), float(rank_w),
                            ctypes.byref(pr) if pr is not None else None, _ptr(payload), n, k,
                            _lib.LARGEST if largest else _lib.SMALLEST, _ptr(vals), _ptr(pay),
                            _ptr(idx), ws.ptr(), ws.nbytes, _stream_ptr(keys.device))
    _lib.check(st, "topk_query")
    return (vals, idx) if payload is None else (vals, idx, pay)


def _pred_struct(pred, n):
    if pred is None:
        return None
    if pred[1].dtype != torch.uint32 or pred[1].shape[0] != n or not pred[1].is_contiguous():
        raise ValueError("predicate column: contiguous CUDA uint32 of the same length")
    if pred[0] == "range":
        return _lib.Pred(_lib.PRED_RANGE, pred[1].data_ptr(), int(pred[2]), int(pred[3]), 0)
    if pred[0] == "in":
        return _lib.Pred(_lib.PRED_IN, pred[1].data_ptr(), 0, 0, int(pred[2]))
    raise ValueError(f"unknown predicate kind {pred[0]!r}")


def topk_kk(k1: torch.Tensor, k2: torch.Tensor, k: int, largest1: bool = True,
            largest2: bool = True, pred: tuple | None = None,
            payload: torch.Tensor | None = None, workspace: Workspace | None = None):
    """Compound-key top-k, ``ORDER BY k1, k2 LIMIT k`` over two CUDA float32 columns
    (KKV), lexicographic, ties to the lowest row.  Returns
    ``(v1, v2, indices)`` or ``(v1, v2, indices, payload_out)``."""
    if not (k1.is_cuda and k2.is_cuda) or k1.dim() != 1 or k1.shape != k2.shape:
        raise ValueError("topk_kk expects two 1-D CUDA float32 tensors of one length")
    if k1.dtype != torch.float32 or k2.dtype != torch.float32:
        raise TypeError("topk_kk: float32 key columns")
    lib = _lib.load()
    n = k1.shape[0]
    pr = _pred_struct(pred, n)
    dev = k1.device
    v1 = torch.empty(k, dtype=torch.float32, device=dev)
    v2 = torch.empty(k, dtype=torch.float32, device=dev)
    idx = torch.empty(k, dtype=torch.int64, device=dev)
    pay = torch.empty(k, dtype=torch.uint32, device=dev) if payload is not None else None
    payload = _check_col(payload, n, torch.uint32, dev, "payload")
    if k2.device != dev or (pred is not None and pred[1].device != dev):
        raise ValueError("topk_kk: every column on the same device")
    with torch.cuda.device(dev):
        need = int(lib.topk_workspace_bytes(_lib.F64, n, k))
        if need == 0:
            raise _lib.TopkError(f"invalid arguments for topk_kk (n={n}, k={k})")
        ws = workspace if workspace is not None else _workspace(dev, need)
        st = lib.topk_kk(_ptr(k1.contiguous()), _ptr(k2.contiguous()),
                         ctypes.byref(pr) if pr is not None else None, _ptr(payload), n, k,
                         _lib.LARGEST if largest1 else _lib.SMALLEST,
                         _lib.LARGEST if largest2 else _lib.SMALLEST, _ptr(v1), _ptr(v2),
                         _ptr(pay), _ptr(idx), ws.ptr(), ws.nbytes, _stream_ptr(dev))
    _lib.check(st, "topk_kk")
    return (v1, v2, idx) if payload is None else (v1, v2, idx, pay)


def topk_kkk(k1: torch.Tensor, k2: torch.Tensor, k3: torch.Tensor, k: int,
             largest=(True, True, True), pred: tuple | None = None,
             payload: torch.Tensor | None = None, workspace: Workspace | None = None):
    """Three compound keys, ``ORDER BY k1, k2, k3 LIMIT k`` (KKKV).  Returns
    ``(v1, v2, v3, indices)`` or ``(v1, v2, v3, indices, payload_out)``."""
    cols = (k1, k2, k3)
    if any(not c.is_cuda or c.dim() != 1 or c.shape != k1.shape or c.dtype != torch.float32
           for c in cols):
        raise ValueError("topk_kkk expects three 1-D CUDA float32 tensors of one length")
    lib = _lib.load()
    n = k1.shape[0]
    pr = _pred_struct(pred, n)
    dev = k1.device
    outs = [torch.empty(k, dtype=torch.float32, device=dev) for _ in range(3)]
    idx = torch.empty(k, dtype=torch.int64, device=dev)
    pay = torch.empty(k, dtype=torch.uint32, device=dev) if payload is not None else None
    payload = _check_col(payload, n, torch.uint32, dev, "payload")
    if any(c.device != dev for c in cols) or (pred is not None and pred[1].device != dev):
        raise ValueError("topk_kkk: every column on the same device")
    o = [_lib.LARGEST if l else _lib.SMALLEST for l in largest]
    with torch.cuda.device(dev):
        need = int(lib.topk_workspace_bytes(_lib.F64, n, k))
        if need == 0:
            raise _lib.TopkError(f"invalid arguments for topk_kkk (n={n}, k={k})")
        ws = workspace if workspace is not None else _workspace(dev, need)
        st = lib.topk_kkk(*[_ptr(c.contiguous()) for c in cols],
                          ctypes.byref(pr) if pr is not None else None, _ptr(payload), n, k, *o,
                          *[_ptr(t) for t in outs], _ptr(pay), _ptr(idx), ws.ptr(), ws.nbytes,
                          _stream_ptr(dev))
    _lib.check(st, "topk_kkk")
    return (*outs, idx) if payload is None else (*outs, idx, pay)


def topk_radix(x: torch.Tensor, k: int, largest: bool = True, out=None):
    """Radix-select top-k (the paper's selection-based method): the same
    result as :func:`topk`, by MSD passes over 8-bit digits of the order code."""
    if not x.is_cuda or x.dim() != 1:
        raise ValueError("topk_radix expects a 1-D CUDA tensor (no CPU path)")
    lib = _lib.load()
    dt = _dtype_code(x)
    n = x.shape[0]
    x = x.contiguous()
    dev = x.device
    if out is not None:
        vals = _check_out(out[0], k, x.dtype, dev, "out values")
        idx = _check_out(out[1], k, torch.int64, dev, "out indices")
    else:
        vals = torch.empty(k, dtype=x.dtype, device=dev)
        idx = torch.empty(k, dtype=torch.int64, device=dev)
    with torch.cuda.device(dev):
        need = int(lib.topk_radix_workspace_bytes(dt, n, k))
        if need == 0:
            raise _lib.TopkError(f"invalid arguments for topk_radix (n={n}, k={k})")
        key = ("radix", dev.index, torch.cuda.current_stream(dev).cuda_stream)
        ws = _ws_cache.get(key)
        if ws is None or ws.nbytes < need:
            ws = Workspace(need, dev)
            _ws_cache[key] = ws
        st = lib.topk_radix(dt, _ptr(x), n, k, _lib.LARGEST if largest else _lib.SMALLEST,
                            _ptr(vals), _ptr(idx), ws.ptr(), ws.nbytes, _stream_ptr(dev))
    _lib.check(st, "topk_radix")
    return vals, idx


def topk_host(x: torch.Tensor, k: int, largest: bool = True, chunk_keys: int = 1 << 26,
              device=None, out=None):
    """Exact top-k of a 1-D HOST tensor (pinned recommended), streamed to the GPU in
    chunks that overlap the reductive pass.  Returns host tensors
    ``(values, indices)``; they are valid after the current stream synchronises."""
    if x.is_cuda or x.dim() != 1:
        raise ValueError("topk_host expects a 1-D host tensor")
    lib = _lib.load()
    dt = _dtype_code(x)
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else device
    n = x.shape[0]
    chunk_keys = max(4096, min(int(chunk_keys), n + (-n) % 4))
    chunk_keys += (-chunk_keys) % 4
    need = int(lib.topk_host_workspace_bytes(dt, n, k, chunk_keys))
    if need == 0:
        raise _lib.TopkError(f"invalid arguments for topk_host (n={n}, k={k})")
    key = ("host", dev.index, need)
    ws = _ws_cache.get(key)
    if ws is None:
        ws = Workspace(need, dev)
        _ws_cache[key] = ws
    if out is None:
        vals = torch.empty(k, dtype=x.dtype, pin_memory=True)
        idx = torch.empty(k, dtype=torch.int64, pin_memory=True)
    else:
        vals, idx = out
    x = x.contiguous()
    with torch.cuda.device(dev):
        st = lib.topk_select_host(dt, _ptr(x), n, k, _lib.LARGEST if largest else _lib.SMALLEST,
                                  _ptr(vals), _ptr(idx), chunk_keys, ws.ptr(), ws.nbytes,
                                  _stream_ptr(dev))
    _lib.check(st, "topk_select_host")
    return vals, idx


def merge(cand_keys: torch.Tensor, cand_idx: torch.Tensor, k: int, largest: bool = True,
          cand_payload: torch.Tensor | None = None, runs: int = 1, sorted_runs: bool = False):
    """Exact top-k of candidate entries (key, global int64 index[, payload]) -- the
    global step after per-partition top-k (multi-GPU all-gather result).  With
    ``sorted_runs`` every one of the ``runs`` equal-length runs must be sorted best first
    (as :func:`topk` returns them): only the merge + rebuild rounds run."""
    if not cand_keys.is_cuda or cand_keys.dim() != 1:
        raise ValueError("merge expects 1-D CUDA candidate tensors (no CPU path)")
    lib = _lib.load()
    dt = _dtype_code(cand_keys)
    total = cand_keys.shape[0]
    if runs < 1 or total % runs:
        raise ValueError("candidates must be runs * run_len long")
    cand_keys = cand_keys.contiguous()
    dev = cand_keys.device
    cand_idx = _check_col(cand_idx, total, torch.int64, dev, "cand_idx")
    cand_payload = _check_col(cand_payload, total, torch.uint32, dev, "cand_payload")
    vals = torch.empty(k, dtype=cand_keys.dtype, device=dev)
    idx = torch.empty(k, dtype=torch.int64, device=dev)
    pay = torch.empty(k, dtype=torch.uint32, device=dev) if cand_payload is not None else None
    with torch.cuda.device(dev):
        fn = lib.topk_merge_sorted if sorted_runs else lib.topk_merge
        st = fn(dt, _ptr(cand_keys), _ptr(cand_idx), _ptr(cand_payload), runs,
                total // runs, k, _lib.LARGEST if largest else _lib.SMALLEST,
                _ptr(vals), _ptr(pay), _ptr(idx), None, 0, _stream_ptr(dev))
    _lib.check(st, "topk_merge")
    return (vals, idx) if cand_payload is None else (vals, idx, pay)


def launch_count() -> int:
    """Kernels launched by libtopk_b200.so so far in this process."""
    return int(_lib.load().topk_launch_count())
