"""TOPK_MODE_PURE -- the paper's data-independent method (every key through local sort,
merge and rebuild) -- against the CPU oracle, bit-exact.  For 32-bit keys and k <= 32 it
runs the register/warp-shuffle kernel (csrc/pure.cuh: keys-only network on the order
codes, folds across lanes, exact index recovery by ballots); larger k and f64 use the
streaming kernel with the filter off.  Covers every k <= 32 (powers of two and not),
ragged chunk tails, tie-heavy inputs (the index recovery of equal codes), both orders,
u32 keys, payloads, base offsets and special values."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

pytestmark = pytest.mark.gpu


def host(t):
    if t.dtype == torch.uint32:
        return t.cpu().view(torch.int32).numpy().view(np.uint32)
    return t.cpu().numpy()


def check(x_cpu, k, largest=True, payload=None, base=0):
    x = x_cpu.cuda()
    keys = host(x_cpu)
    if payload is not None:
        v, i, pv = tk.topk(x, k, largest, payload=payload.cuda(), base=base, mode="pure")
    else:
        v, i = tk.topk(x, k, largest, base=base, mode="pure")
    ov, oi = oracle.topk(keys, k, largest, base=base)
    gi = i.cpu().numpy()
    assert np.array_equal(gi, oi), (k, largest, np.nonzero(gi != oi)[0][:5])
    assert host(v).tobytes() == ov.tobytes()
    if payload is not None:
        assert np.array_equal(host(pv), host(payload)[oi - base])


@pytest.mark.parametrize("n", [1, 31, 32, 33, 1000, 1024, 1025, 4097, 65536 + 77, (1 << 20) + 13])
def test_pure_every_small_k(cuda_device, n):
    x = datagen.generate("uniform", n, "f32", seed=n + 5)
    for k in range(1, min(n, 32) + 1):
        check(x, k, True)
    for k in (1, 5, 16, 17, 32):
        if k <= n:
            check(x, k, False)


@pytest.mark.parametrize("dist", ["fewdistinct", "increasing", "decreasing", "bucketkiller"])
@pytest.mark.parametrize("largest", [True, False])
def test_pure_ties_and_sorted(cuda_device, dist, largest):
    n = (1 << 21) + 333
    x = datagen.generate(dist, n, "f32", seed=77)
    for k in (1, 2, 7, 8, 31, 32):
        check(x, k, largest)


def test_pure_all_equal(cuda_device):
    x = torch.full((300001,), 0.5, dtype=torch.float32)
    for k in (1, 3, 32):
        check(x, k, True)
        check(x, k, False)


def test_pure_u32_payload_base(cuda_device):
    n = (1 << 22) + 9
    x = datagen.generate("uniform", n, "u32", seed=88)
    p = datagen.payload(n, seed=88)
    for k in (1, 19, 32):
        check(x, k, True, payload=p, base=12345678901)
        check(x, k, False, payload=p)
    xf = datagen.generate("fewdistinct", n, "u32", seed=89)
    check(xf, 32, True)


def test_pure_special_values(cuda_device):
    rng = np.random.default_rng(3)
    specials = np.array([np.nan, -np.nan, np.inf, -np.inf, 0.0, -0.0, 1.0, -1.0, 1e-45,
                         -1e-45, 3.4e38], np.float32)
    nan_payloads = np.array([0x7FC00001, 0xFFC00002, 0x7F800003], np.uint32).view(np.float32)
    x = torch.from_numpy(rng.choice(np.concatenate([specials, nan_payloads]), 100003))
    for k in (1, 4, 32):
        check(x, k, True)
        check(x, k, False)


@pytest.mark.parametrize("k", [33, 64, 100, 128, 129, 200, 256])
def test_pure_entry_network(cuda_device, k):
    """32 < k <= 256: the (code, index) entry network (pure64_kernel)."""
    for n, dist in (((1 << 20) + 333, "uniform"), ((1 << 19) + 5, "fewdistinct"),
                    (4097, "uniform"), ((1 << 21) + 1, "decreasing")):
        x = datagen.generate(dist, n, "f32", seed=n + k)
        check(x, k, True)
        check(x, k, False)
    xu = datagen.generate("uniform", (1 << 20) + 7, "u32", seed=k)
    p = datagen.payload((1 << 20) + 7, seed=k)
    check(xu, k, True, payload=p, base=77)


@pytest.mark.parametrize("offset", [1, 2, 3])
@pytest.mark.parametrize("k", [1, 32, 64, 256])
def test_pure_misaligned_pointer(cuda_device, offset, k):
    """Keys not 16-byte aligned: the chunk loads bypass the TMA ring (direct loads)."""
    n = (1 << 20) + 77
    x = datagen.generate("uniform", n, "f32", seed=offset * 100 + k)
    full = x.cuda()
    xs = full[offset:]
    keys = x.numpy()[offset:]
    v, i = tk.topk(xs, k, True, mode="pure")
    ov, oi = oracle.topk(keys, k, True)
    assert np.array_equal(i.cpu().numpy(), oi)
    assert v.cpu().numpy().tobytes() == ov.tobytes()
    if k <= 32:  # filter mode on a small input takes the pure kernel too
        v, i = tk.topk(xs, k, False)
        ov, oi = oracle.topk(keys, k, False)
        assert np.array_equal(i.cpu().numpy(), oi)
