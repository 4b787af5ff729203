"""GPU parity of the radix-select top-k (topk_radix: the paper's selection-based method,
P:93) against the CPU oracle -- bit-exact values and rows under the same
total order as topk_select (R1-R5).  Covers the three ways its result is
assembled: the bucket path (digit-1 bucket written, ties collected from it), tie
overflow (more ties at the k-th code than the collect buffer holds -> the input pass),
and the skipped bucket (digit-1 bucket larger than the workspace -> input passes)."""
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


def check(x_cpu, k, largest=True, offset=0):
    x = x_cpu.to("cuda")[offset:]
    v, i = tk.topk_radix(x, k, largest)
    torch.cuda.synchronize()
    ov, oi = oracle.topk(host(x_cpu)[offset:], k, largest)
    gi = i.cpu().numpy()
    assert np.array_equal(gi, oi), f"rows differ (k={k}): first at {np.nonzero(gi != oi)[0][:5]}"
    assert host(v).tobytes() == ov.tobytes()


N = (1 << 20) + 4096 * 5 + 11


@pytest.mark.parametrize("k", [1, 2, 31, 32, 100, 256, 257, 1000, 1024, 1500, 2048])
def test_every_k(cuda_device, k):
    x = datagen.generate("uniform", N, "f32", seed=401)
    check(x, k, True)
    check(x, k, False)


@pytest.mark.parametrize("dist", ["uniform", "increasing", "decreasing", "fewdistinct",
                                  "bucketkiller"])
@pytest.mark.parametrize("largest", [True, False])
def test_distributions(cuda_device, dist, largest):
    x = datagen.generate(dist, N, "f32", seed=402)
    for k in (1, 64, 256, 1024):
        check(x, k, largest)


@pytest.mark.parametrize("dt", ["u32", "f64"])
@pytest.mark.parametrize("dist", ["uniform", "fewdistinct", "increasing"])
def test_dtypes(cuda_device, dt, dist):
    x = datagen.generate(dist, N, dt, seed=403)
    for k in (1, 64, 777):
        check(x, k, True)
        check(x, k, False)


def test_all_equal_skips_bucket(cuda_device):
    """Every key equal: the digit-1 bucket is the whole input (> the workspace's
    n/16): no scatter, every digit reads the input, the ties come from the input pass
    (the first k rows)."""
    x = torch.full((N,), 0.5, dtype=torch.float32)
    check(x, 1000, True)
    check(x, 3, False)


def test_special_values_and_small_n(cuda_device):
    sp = torch.tensor([float("nan"), -float("nan"), -float("inf"), -0.0, 0.0, 1.0,
                       float("inf"), 1e-40], dtype=torch.float32)
    g = torch.Generator().manual_seed(5)
    for n in (1, 2, 15, 16, 17, 4095, 4097, 70001):
        x = sp[torch.randint(0, sp.shape[0], (n,), generator=g)]
        for k in sorted({1, min(n, 5), min(n, 64)}):
            check(x, k, True)
            check(x, k, False)


@pytest.mark.parametrize("offset", [1, 2, 3])
def test_misaligned(cuda_device, offset):
    x = datagen.generate("uniform", 300001, "f32", seed=404)
    check(x, 100, True, offset)


def test_repeated_calls(cuda_device):
    x = datagen.generate("uniform", N, "f32", seed=405)
    y = datagen.generate("fewdistinct", N, "f32", seed=406)
    for _ in range(3):
        check(x, 256, True)
        check(y, 128, True)


@pytest.mark.slow
def test_full_size_matches_oracle(cuda_device):
    """2^29 uniform f32 (BJ configs[1], the bench's radix_vs_bitonic launch): bit-exact
    against the CPU oracle (and therefore identical to the bitonic path's result)."""
    x = datagen.generate("uniform", 1 << 29, "f32", seed=datagen.config_seed(2), device="cuda")
    keys = x.cpu().numpy()
    ov, oi = oracle.topk(keys, 1024, True)
    for k in (32, 256, 1024):
        v1, i1 = tk.topk_radix(x, k)
        assert np.array_equal(i1.cpu().numpy(), oi[:k])
        assert v1.cpu().numpy().tobytes() == ov[:k].tobytes()
    ov, oi = oracle.topk(keys, 256, False)
    v1, i1 = tk.topk_radix(x, 256, False)
    assert np.array_equal(i1.cpu().numpy(), oi)
