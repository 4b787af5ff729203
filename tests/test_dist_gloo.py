"""Host logic of the multi-GPU shard-and-gather driver with world_size 2 on CPU (gloo).

The CUDA local / merge steps are replaced by the oracle (test-only injection) so the
rank offsets, gather layout and merge inputs are checked without a GPU: the sharded
result must equal the oracle on the whole input, bit-exact, on every rank."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import oracle
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen
    from paper_conf_sigmod_shanbhagpm18_b200.dist import shard_bounds, sharded_topk

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)

    def local_fn(x, k, largest, base):
        v, i = oracle.topk(x.numpy(), k, largest, base=base)
        return torch.from_numpy(v), torch.from_numpy(i)

    def merge_fn(vals, idx, k, largest, runs):
        v, i = oracle.topk(vals.numpy(), k, largest, idx=idx.numpy())
        return torch.from_numpy(v), torch.from_numpy(i)

    res = []
    for dist_name, n_total, k, largest in [("fewdistinct", 100003, 64, True),
                                           ("uniform", 65536, 256, False),
                                           ("increasing", 50000, 7, True)]:
        lo, hi = shard_bounds(n_total, world, rank)
        x = datagen.generate(dist_name, hi - lo, "f32", base=lo, n_total=n_total)
        v, i = sharded_topk(x, k, largest, base=lo, local_fn=local_fn, merge_fn=merge_fn)
        res.append((v.numpy().tobytes(), i.numpy().tolist()))
    q.put((rank, res))
    dist.destroy_process_group()


def test_sharded_topk_world2_gloo():
    import oracle
    from paper_conf_sigmod_shanbhagpm18_b200 import datagen
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=180) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cases = [("fewdistinct", 100003, 64, True), ("uniform", 65536, 256, False),
             ("increasing", 50000, 7, True)]
    for ci, (dname, n_total, k, largest) in enumerate(cases):
        x = datagen.generate(dname, n_total, "f32").numpy()
        ov, oi = oracle.topk(x, k, largest)
        for r in range(2):
            vb, il = out[r][ci]
            assert il == oi.tolist(), (dname, r)
            assert vb == ov.tobytes()


def _comm_worker(rank, world, port, q):
    """NcclComm's host logic: rank 0's unique id reaches every rank through the torch
    group and each rank initialises its communicator with (id, world, rank).  The two
    C calls are replaced by recorders (no GPU / NCCL here)."""
    import ctypes
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib, dist as tkdist

    calls = []

    class FakeLib:
        def topk_nccl_unique_id(self, buf):
            ctypes.memmove(buf, bytes(range(7, 7 + 128)), 128)
            return 0

        def topk_nccl_comm_init(self, uid, nranks, r, out):
            calls.append((bytes(uid.raw), nranks, r))
            return 0

    _lib.load = lambda build_if_missing=True: FakeLib()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)

    class _Dev:  # torch.cuda.device(...) needs no GPU for this check
        def __init__(self, *a):
            pass

        def __enter__(self):
            return self

        def __exit__(self, *a):
            return False

    torch.cuda.device = _Dev
    tkdist.NcclComm(device="cpu")
    q.put((rank, calls))
    dist.destroy_process_group()


def test_nccl_comm_id_broadcast_world2_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_comm_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=180) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = bytes(range(7, 7 + 128))
    for r in range(2):
        assert out[r] == [(want, 2, r)]
