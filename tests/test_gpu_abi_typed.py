"""The typed C-ABI entries SURVEY §8(b) lists -- topk_f32, topk_u32, topk_f64,
topk_u32_kv, topk_f64_kv, topk_f32_sharded -- called with data through ctypes (device
pointers from torch, the caller-owned workspace zero-filled once with
topk_workspace_init), against the CPU oracle: bit-exact key bits, indices, payloads."""
import ctypes

import numpy as np
import pytest
import torch

import oracle
from paper_conf_sigmod_shanbhagpm18_b200 import _lib, datagen

pytestmark = pytest.mark.gpu

DT = {"f32": (torch.float32, _lib.F32), "u32": (torch.uint32, _lib.U32),
      "f64": (torch.float64, _lib.F64)}


def host(t):
    if t.dtype == torch.uint32:
        return t.cpu().view(torch.int32).numpy().view(np.uint32)
    return t.cpu().numpy()


def P(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def workspace(lib, code, n, k, dev):
    nb = int(lib.topk_workspace_bytes(code, n, k))
    assert nb > 0
    ws = torch.empty(nb, dtype=torch.uint8, device=dev)
    assert lib.topk_workspace_init(P(ws), nb, None) == 0  # legacy default stream
    return ws, nb


@pytest.mark.parametrize("dt", ["f32", "u32", "f64"])
@pytest.mark.parametrize("n", [1000, (1 << 20) + 3, 1 << 24])
def test_typed_entry(cuda_device, dt, n):
    lib = _lib.load()
    tdt, code = DT[dt]
    fn = {"f32": lib.topk_f32, "u32": lib.topk_u32, "f64": lib.topk_f64}[dt]
    x = datagen.generate("uniform" if n > 1000 else "fewdistinct", n, dt, seed=n + 17,
                         device=cuda_device)
    keys = host(x)
    for k, order in ((1, _lib.LARGEST), (100, _lib.SMALLEST), (min(n, 1024), _lib.LARGEST)):
        ws, nb = workspace(lib, code, n, k, cuda_device)
        ok = torch.empty(k, dtype=tdt, device=cuda_device)
        oi = torch.empty(k, dtype=torch.int64, device=cuda_device)
        torch.cuda.synchronize()
        assert fn(P(x), n, k, order, P(ok), P(oi), P(ws), nb, None) == 0
        torch.cuda.synchronize()
        ev, ei = oracle.topk(keys, k, order == _lib.LARGEST)
        assert np.array_equal(oi.cpu().numpy(), ei)
        assert host(ok).tobytes() == ev.tobytes()
        # the same workspace serves the next call without re-initialisation
        assert fn(P(x), n, k, order, P(ok), P(oi), P(ws), nb, None) == 0
        torch.cuda.synchronize()
        assert np.array_equal(oi.cpu().numpy(), ei)


@pytest.mark.parametrize("dt", ["u32", "f64"])
def test_typed_kv_entry(cuda_device, dt):
    lib = _lib.load()
    tdt, code = DT[dt]
    fn = lib.topk_u32_kv if dt == "u32" else lib.topk_f64_kv
    n = (1 << 22) + 1
    x = datagen.generate("uniform", n, dt, seed=4242, device=cuda_device)
    p = datagen.payload(n, seed=4242, device=cuda_device)
    keys, ph = host(x), host(p)
    for k, order in ((64, _lib.LARGEST), (64, _lib.SMALLEST), (2048, _lib.LARGEST)):
        ws, nb = workspace(lib, code, n, k, cuda_device)
        ok = torch.empty(k, dtype=tdt, device=cuda_device)
        op = torch.empty(k, dtype=torch.uint32, device=cuda_device)
        oi = torch.empty(k, dtype=torch.int64, device=cuda_device)
        torch.cuda.synchronize()
        assert fn(P(x), P(p), n, k, order, P(ok), P(op), P(oi), P(ws), nb, None) == 0
        torch.cuda.synchronize()
        ev, ei = oracle.topk(keys, k, order == _lib.LARGEST)
        assert np.array_equal(oi.cpu().numpy(), ei)
        assert host(ok).tobytes() == ev.tobytes()
        assert np.array_equal(host(op), ph[ei])


def test_typed_entries_reject_bad_arguments(cuda_device):
    lib = _lib.load()
    x = torch.zeros(100, dtype=torch.float32, device=cuda_device)
    ws, nb = workspace(lib, _lib.F32, 100, 10, cuda_device)
    assert lib.topk_f32(P(x), 100, 0, 0, None, None, P(ws), nb, None) == 1      # k = 0
    assert lib.topk_f32(P(x), 100, 101, 0, None, None, P(ws), nb, None) == 1    # k > n
    assert lib.topk_f32(P(x), 100, 10, 7, None, None, P(ws), nb, None) == 1     # order
    assert lib.topk_f32(P(x), 100, 10, 0, None, None, P(ws), 16, None) == 3     # ws size
    assert lib.topk_f64(ctypes.c_void_p(x.data_ptr() + 4), 10, 1, 0, None, None, P(ws), nb,
                        None) == 1                                               # f64 align


def test_f32_sharded_one_rank(cuda_device):
    """topk_f32_sharded (local select -> ncclAllGather -> merge) on a one-rank
    communicator: global ids = base + i."""
    from paper_conf_sigmod_shanbhagpm18_b200.dist import NcclComm
    lib = _lib.load()
    comm = NcclComm(device=cuda_device)
    try:
        n, base, k = (1 << 21) + 5, 3 << 32, 300
        x = datagen.generate("uniform", n, "f32", seed=77, device=cuda_device)
        nb = int(lib.topk_sharded_workspace_bytes(_lib.F32, n, k, 1))
        ws = torch.zeros(nb, dtype=torch.uint8, device=cuda_device)
        ok = torch.empty(k, dtype=torch.float32, device=cuda_device)
        oi = torch.empty(k, dtype=torch.int64, device=cuda_device)
        torch.cuda.synchronize()
        assert lib.topk_f32_sharded(P(x), n, base, k, _lib.LARGEST, P(ok), P(oi), comm.ptr,
                                    P(ws), nb, None) == 0
        torch.cuda.synchronize()
        ev, ei = oracle.topk(host(x), k, True, base=base)
        assert np.array_equal(oi.cpu().numpy(), ei)
        assert host(ok).tobytes() == ev.tobytes()
    finally:
        comm.close()
