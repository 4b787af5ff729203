"""GPU parity at the sizes and launch configurations bench.py times (VERDICT r1 "weak #1").

The select kernel changes shape with the input size: a launch with ntiles >= 16 * #SM
claims blocks of 8 tiles, visits the waves of blocks in the Feistel order (perm_h > 0)
and requests the tile-12 rank-bound refresh; the tie-heavy bag limit only matters when a
CTA streams many tiles.  Every case here compares the CUDA path (through the C ABI, the
launch the bench times) with the CPU oracle element by element: bit-exact key bits and
int64 indices (DESIGN.md §6 parity bar).  Expected values come only from oracle/.

* non-slow: 2^25 f32 and 2^24 f64 (ntiles = 4370 >= 16 * 148) -- every GPUTEST run
  reaches blk = 8, the Feistel order and the refresh;
* slow (-m "gpu and slow"): BJ configs[2] at 2^29 (increasing, decreasing, fewdistinct,
  bucketkiller; k = 256, 1024, 2048; both orders), configs[3] (2^28 u32 + payload and
  2^28 f64, LIMIT 64), configs[4] at G = 1 (2^32 f32: two 2^31-key launches + merge).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

pytestmark = pytest.mark.gpu


def host(t: torch.Tensor) -> np.ndarray:
    if t.dtype == torch.uint32:
        return t.cpu().view(torch.int32).numpy().view(np.uint32)
    return t.cpu().numpy()


def sms():
    return torch.cuda.get_device_properties(0).multi_processor_count


def compare_prefixes(xd, keys, ks, largest, payload_d=None, payload_h=None, mode="filter"):
    """The oracle's top-max(ks) once; every smaller k must equal its prefix (the result
    is best first under a total order, so top-k is a prefix of top-K)."""
    kmax = max(ks)
    ov, oi = oracle.topk(keys, kmax, largest)
    for k in ks:
        if payload_d is not None:
            v, i, pv = tk.topk(xd, k, largest, payload=payload_d, mode=mode)
        else:
            v, i = tk.topk(xd, k, largest, mode=mode)
        gi = i.cpu().numpy()
        assert np.array_equal(gi, oi[:k]), \
            f"k={k} largest={largest}: indices differ first at {np.nonzero(gi != oi[:k])[0][:5]}"
        assert host(v).tobytes() == ov[:k].tobytes(), f"k={k}: key bits differ"
        if payload_d is not None:
            assert np.array_equal(host(pv), payload_h[oi[:k]])


@pytest.mark.parametrize("dist", ["uniform", "increasing", "decreasing", "fewdistinct",
                                  "bucketkiller"])
def test_2p25_f32_block_claiming(cuda_device, dist):
    n = 1 << 25
    assert (n + 7679) // 7680 >= 16 * sms()  # blk = 8, perm_h > 0, refresh at tile 12
    xd = datagen.generate(dist, n, "f32", seed=datagen.config_seed(3, 7), device=cuda_device)
    keys = host(xd)
    for largest in (True, False):
        compare_prefixes(xd, keys, (1, 32, 256, 1000, 2048), largest)


def test_2p25_f32_ragged_payload(cuda_device):
    n = (1 << 25) + 4095  # ragged last tile and a < 16-byte tail
    xd = datagen.generate("uniform", n, "f32", seed=991, device=cuda_device)
    pd = datagen.payload(n, seed=991, device=cuda_device)
    compare_prefixes(xd, host(xd), (64, 777), True, pd, host(pd))
    compare_prefixes(xd[1:], host(xd)[1:], (64,), False, pd[1:], host(pd)[1:])  # misaligned


@pytest.mark.parametrize("dist", ["uniform", "increasing", "fewdistinct"])
def test_2p24_f64_block_claiming(cuda_device, dist):
    n = 1 << 24
    assert (n + 3839) // 3840 >= 16 * sms()
    xd = datagen.generate(dist, n, "f64", seed=datagen.config_seed(4, 7), device=cuda_device)
    keys = host(xd)
    for largest in (True, False):
        compare_prefixes(xd, keys, (1, 64, 1024), largest)


def test_2p25_u32_payload(cuda_device):
    n = 1 << 25
    xd = datagen.generate("uniform", n, "u32", seed=992, device=cuda_device)
    pd = datagen.payload(n, seed=992, device=cuda_device)
    for largest in (True, False):
        compare_prefixes(xd, host(xd), (64, 512), largest, pd, host(pd))


def test_2p25_pure_mode(cuda_device):
    """The paper's data-independent method (TOPK_MODE_PURE) at a size with many tiles
    per CTA, against the oracle."""
    n = 1 << 25
    xd = datagen.generate("uniform", n, "f32", seed=993, device=cuda_device)
    keys = host(xd)
    for largest in (True, False):
        compare_prefixes(xd, keys, (1, 32, 256, 1024), largest, mode="pure")
    xd = datagen.generate("fewdistinct", n, "f32", seed=994, device=cuda_device)
    compare_prefixes(xd, host(xd), (32, 256), True, mode="pure")


# ---------------- full BJ sizes (-m slow) ----------------

@pytest.mark.slow
@pytest.mark.parametrize("dist", ["increasing", "decreasing", "fewdistinct", "bucketkiller"])
def test_config3_2p29_adversarial(cuda_device, dist):
    """BJ configs[2]: 2^29 f32 sorted increasing / decreasing / many duplicates, the
    bench's adversarial_k256 launch, plus k = 1024, 2048 (the tie-bag flush limit)."""
    n = 1 << 29
    xd = datagen.generate(dist, n, "f32", seed=datagen.config_seed(3), device=cuda_device)
    keys = host(xd)
    for largest in (True, False):
        compare_prefixes(xd, keys, (256, 1024, 2048), largest)


@pytest.mark.slow
def test_config2_2p29_uniform_sweep(cuda_device):
    """BJ configs[1]: every k of the bench's sweep on the bench's input."""
    n = 1 << 29
    xd = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device=cuda_device)
    keys = host(xd)
    compare_prefixes(xd, keys, (1, 8, 32, 64, 128, 256, 512, 1024, 2048), True)
    compare_prefixes(xd, keys, (256,), False)


@pytest.mark.slow
def test_config4a_2p28_u32_payload(cuda_device):
    """BJ configs[3] (a): 2^28 u32 key + 32-bit row-id payload, DESC LIMIT 64."""
    n = 1 << 28
    xd = datagen.generate("uniform", n, "u32", seed=datagen.config_seed(4), device=cuda_device)
    pd = datagen.payload(n, seed=datagen.config_seed(4), device=cuda_device)
    for largest in (True, False):
        compare_prefixes(xd, host(xd), (64,), largest, pd, host(pd))


@pytest.mark.slow
def test_config4b_2p28_f64(cuda_device):
    """BJ configs[3] (b): 2^28 f64 keys, DESC LIMIT 64."""
    n = 1 << 28
    xd = datagen.generate("uniform", n, "f64", seed=datagen.config_seed(4), device=cuda_device)
    keys = host(xd)
    for largest in (True, False):
        compare_prefixes(xd, keys, (64, 1024), largest)


@pytest.mark.slow
def test_config5_2p32_two_chunks(cuda_device):
    """BJ configs[4] at G = 1: 2^32 uniform f32 in one call -- two 2^31-key launches with
    base offsets + the merge kernel.  Expected: the oracle per 2^29-row piece (generated
    piecewise on the host side of the same counter-based stream), then the oracle's
    global step over the pieces' candidates with their global ids -- the decomposition
    pinned by tests/test_oracle_pins.py (topk(A u B) == topk(topk(A) u topk(B)))."""
    n, k = 1 << 32, 256
    seed = datagen.config_seed(5)
    free, _ = torch.cuda.mem_get_info()
    if free < n * 4 + (1 << 30):
        pytest.skip("needs 17 GiB of free device memory")
    xd = datagen.generate("uniform", n, "f32", seed=seed, device=cuda_device)
    v, i = tk.topk(xd, k, True)
    gv, gi = host(v), i.cpu().numpy()
    piece = 1 << 29
    cv, ci = [], []
    for p in range(n // piece):
        keys = host(xd[p * piece:(p + 1) * piece])
        pv, pi = oracle.topk(keys, k, True, base=p * piece)
        cv.append(pv)
        ci.append(pi)
    ov, oi = oracle.topk(np.concatenate(cv), k, True, idx=np.concatenate(ci))
    assert np.array_equal(gi, oi)
    assert gv.tobytes() == ov.tobytes()
    # and sampled rows: the device generator equals the host generator at global rows
    rows = np.random.default_rng(5).integers(0, n, 16)
    for r in rows:
        h = datagen.generate("uniform", 1, "f32", seed=seed, base=int(r), n_total=n)
        assert host(h)[0] == host(xd[int(r):int(r) + 1])[0]


@pytest.mark.parametrize("dt,lg,k,dist", [("f64", 24, 1024, "uniform"), ("f32", 24, 2048, "uniform"),
                                          ("u32", 22, 1024, "uniform"),
                                          ("f32", 27, 256, "decreasing")])
def test_repeated_calls_identical(cuda_device, dt, lg, k, dist):
    """The kernel's schedule (which CTA claims which tiles, which one runs the tail) is
    timing-dependent; the answer must not be.  Regression for the bag reservation race
    (select.cuh reserve(): add-then-undo let a warp append above a failed warp's phantom
    entries -- ~4% wrong answers at f64, 2^24, k = 1024): 60 calls, every one exact.
    Decreasing input (every top-k key in one tile, so most CTAs' sample rows are missing
    or weak): regression for a rank bound that ignored missing samples (~17% wrong answers
    at 2^29, k = 256, during development of the count-greater rank_rows)."""
    n = 1 << lg
    x = datagen.generate(dist, n, dt, seed=n + 17, device=cuda_device)
    ev, ei = oracle.topk(host(x), k, True)
    bad = 0
    for _ in range(60):
        v, i = tk.topk(x, k, True)
        bad += int(not (np.array_equal(i.cpu().numpy(), ei) and host(v).tobytes() == ev.tobytes()))
    assert bad == 0, f"{bad}/60 calls wrong"
