"""bench.py's multi-GPU plan on CPU: weak (2^29 per rank) and strong (--n-total, BJ
configs[4]: 2^32 split over 1/2/4/8 GPUs) shards tile the global input exactly, in rank
order (the merge kernel's "ordered runs" fast path relies on that), and a world-size-2
gloo run of the plan agrees across ranks -- the torchrun launch without the GPU work."""
import os
import socket
import sys

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("n_total", [None, 1 << 32, (1 << 32) + 7, 1000])
def test_shards_tile_the_input(world, n_total):
    got = [bench.shard_plan(r, world, n_total) for r in range(world)]
    total = got[0][0]
    assert all(g[0] == total for g in got)
    assert total == (world * bench.N_PER_GPU if n_total is None else n_total)
    assert got[0][1] == 0 and got[-1][2] == total
    for a, b in zip(got, got[1:]):
        assert a[2] == b[1] and a[1] <= a[2]
    if n_total is None:
        assert all(g[2] - g[1] == bench.N_PER_GPU for g in got)  # weak: fixed per rank
    else:
        sizes = [g[2] - g[1] for g in got]
        assert max(sizes) - min(sizes) <= 1  # strong: balanced


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n_total, q):
    sys.path.insert(0, ROOT)
    import torch
    import bench as b
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    r, w, _ = b.dist_env()
    mine = torch.tensor(list(b.shard_plan(r, w, n_total)), dtype=torch.int64)
    allp = [torch.zeros(3, dtype=torch.int64) for _ in range(w)]
    dist.all_gather(allp, mine)
    q.put((rank, [tuple(int(v) for v in t) for t in allp]))
    dist.destroy_process_group()


@pytest.mark.parametrize("n_total", [None, 1 << 32])
def test_plan_under_gloo_world2(n_total):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n_total, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    plans = [r[1] for r in sorted(res)]
    assert plans[0] == plans[1]
    (t0, lo0, hi0), (t1, lo1, hi1) = plans[0]
    assert t0 == t1 and lo0 == 0 and hi0 == lo1 and hi1 == t0
