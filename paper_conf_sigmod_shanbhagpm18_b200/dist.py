"""Multi-GPU shard-and-gather driver.

The partitioned top-k of the paper: "each processor compute[s] a per-partition top-k and
[the] global top-k [is computed] from the m per-partition heaps" (§1); "the top-k
elements emitted by the individual core are combined in a final global step".
On B200s: one process per GPU, rank r holds the rows [base_r, base_r + n_r) of the global
input; the local top-k runs in the select kernel with ``base = base_r`` (global row ids),
the k (value, id) candidates of every rank are all-gathered over NCCL (NVLink 5 /
NVSwitch), and every rank reduces them with the merge kernel -- the same local sort /
merge / rebuild network -- to the identical exact result (ties by global id).

``local_fn`` / ``merge_fn`` default to the CUDA library; tests inject CPU stand-ins to
exercise the host logic (ranks, offsets, gather layout) with the gloo backend.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def _default_local(x, k, largest, base):
    from . import topk
    return topk(x, k, largest, base=base)


def _default_merge(vals, idx, k, largest, runs):
    from . import merge
    return merge(vals, idx, k, largest, runs=runs)


def shard_bounds(n_total: int, world: int, rank: int):
    """Contiguous shard of rank r: rows [r*n/G, (r+1)*n/G)."""
    lo = n_total * rank // world
    hi = n_total * (rank + 1) // world
    return lo, hi


def sharded_topk(x_local: torch.Tensor, k: int, largest: bool = True, base: int = 0,
                 group=None, local_fn=None, merge_fn=None):
    """Exact top-k of the union of every rank's ``x_local`` (global ids = base + row).

    Every rank must hold at least k keys.  Returns (values, int64 global ids), identical on
    every rank.
    """
    local_fn = local_fn or _default_local
    merge_fn = merge_fn or _default_merge
    world = dist.get_world_size(group)
    v, i = local_fn(x_local, k, largest, base)
    v = v.contiguous()
    i = i.to(torch.int64).contiguous()
    if world == 1:
        return v, i
    gv = torch.empty(world * k, dtype=v.dtype, device=v.device)
    gi = torch.empty(world * k, dtype=torch.int64, device=i.device)
    dist.all_gather_into_tensor(gv, v, group=group)
    dist.all_gather_into_tensor(gi, i, group=group)
    return merge_fn(gv, gi, k, largest, world)


class NcclComm:
    """An NCCL communicator owned by the C ABI (topk_nccl_comm_init) for
    topk_select_sharded.  Rank 0 makes the unique id; it reaches the other ranks through
    ``group`` (any torch.distributed backend -- only the 128-byte id travels there)."""

    def __init__(self, group=None, device=None):
        import ctypes
        from . import _lib
        lib = _lib.load()
        on = dist.is_available() and dist.is_initialized()
        self.rank = dist.get_rank(group) if on else 0
        self.world = dist.get_world_size(group) if on else 1
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None \
            else torch.device(device)
        uid = ctypes.create_string_buffer(128)
        if self.rank == 0:
            _lib.check(lib.topk_nccl_unique_id(uid), "topk_nccl_unique_id")
        obj = [bytes(uid.raw)]
        if self.world > 1:
            dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0)
                                       if group is not None else 0, group=group)
        uid = ctypes.create_string_buffer(obj[0], 128)
        comm = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            _lib.check(lib.topk_nccl_comm_init(uid, self.world, self.rank, ctypes.byref(comm)),
                       "topk_nccl_comm_init")
        self.ptr = comm
        self._ws = None

    def workspace(self, dtype_code: int, n_local: int, k: int):
        from . import _lib
        from . import Workspace
        need = int(_lib.load().topk_sharded_workspace_bytes(dtype_code, n_local, k, self.world))
        if need == 0:
            raise _lib.TopkError(f"invalid sharded arguments (n_local={n_local}, k={k})")
        if self._ws is None or self._ws.nbytes < need:
            self._ws = Workspace(need, self.device)
        return self._ws

    def close(self):
        from . import _lib
        if self.ptr:
            _lib.load().topk_nccl_comm_destroy(self.ptr)
            self.ptr = None


def sharded_topk_native(x_local: torch.Tensor, k: int, comm: NcclComm, largest: bool = True,
                        base: int = 0, payload: torch.Tensor | None = None, out=None):
    """Exact top-k of the union of every rank's shard through the C ABI's
    topk_select_sharded: local select kernel -> ncclAllGather of the k candidates ->
    merge kernel, all enqueued on the current stream (no host synchronisation).
    Returns (values, int64 global ids[, payload]) on every rank."""
    import ctypes
    from . import _lib, _dtype_code, _ptr, _stream_ptr, _check_col, _check_out
    if not x_local.is_cuda or x_local.dim() != 1:
        raise ValueError("sharded_topk_native expects a 1-D CUDA tensor")
    if x_local.device != comm.device:
        raise ValueError(f"shard on {x_local.device}, communicator on {comm.device}")
    lib = _lib.load()
    dt = _dtype_code(x_local)
    n = x_local.shape[0]
    dev = x_local.device
    x_local = x_local.contiguous()
    payload = _check_col(payload, n, torch.uint32, dev, "payload")
    if out is None:
        vals = torch.empty(k, dtype=x_local.dtype, device=dev)
        idx = torch.empty(k, dtype=torch.int64, device=dev)
        pay = torch.empty(k, dtype=torch.uint32, device=dev) if payload is not None else None
    else:
        vals = _check_out(out[0], k, x_local.dtype, dev, "out values")
        idx = _check_out(out[1], k, torch.int64, dev, "out indices")
        pay = _check_out(out[2], k, torch.uint32, dev, "out payload")
    with torch.cuda.device(dev):
        ws = comm.workspace(dt, n, k)
        st = lib.topk_select_sharded(dt, _ptr(x_local), _ptr(payload), n, base, k,
                                     _lib.LARGEST if largest else _lib.SMALLEST, _ptr(vals),
                                     _ptr(pay), _ptr(idx), comm.ptr, ws.ptr(), ws.nbytes,
                                     _stream_ptr(dev))
    _lib.check(st, "topk_select_sharded")
    return (vals, idx) if payload is None else (vals, idx, pay)
