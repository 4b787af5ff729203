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
