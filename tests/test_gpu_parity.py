"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by
element -- bit-exact key bits and indices (the method is exact, integer-ordered work:
DESIGN.md §7 "Parity bar").  Inputs come from the shared seeded generator; expected
values only from oracle/."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen

pytestmark = pytest.mark.gpu

NP = {torch.float32: np.float32, torch.uint32: np.uint32, torch.float64: np.float64}


def host(t: torch.Tensor) -> np.ndarray:
    if t.dtype == torch.uint32:
        return t.cpu().view(torch.int32).numpy().view(np.uint32)
    return t.cpu().numpy()


def check(x_cpu: torch.Tensor, k: int, largest=True, mode="filter", dev="cuda", base=0,
          payload=None, offset=0):
    """Run on the GPU (optionally from a misaligned offset) and compare with the oracle."""
    full = x_cpu.to(dev)
    x = full[offset:]
    keys = host(x_cpu)[offset:]
    if payload is not None:
        pay_d = payload.to(dev)[offset:]
        v, i, pv = tk.topk(x, k, largest, payload=pay_d, base=base, mode=mode)
    else:
        v, i = tk.topk(x, k, largest, base=base, mode=mode)
    torch.cuda.synchronize()
    ov, oi = oracle.topk(keys, k, largest, base=base)
    gi = i.cpu().numpy()
    gv = host(v)
    assert np.array_equal(gi, oi), f"indices differ (k={k}, largest={largest}, mode={mode}): " \
        f"first mismatch at {np.nonzero(gi != oi)[0][:5]}"
    assert gv.tobytes() == ov.tobytes(), "key bits differ"
    if payload is not None:
        ph = host(payload)[offset:]
        assert np.array_equal(host(pv), ph[oi - base])


def test_config1_uniform_2p20_k32(cuda_device):
    x = datagen.generate("uniform", 1 << 20, "f32", seed=datagen.config_seed(1))
    for mode in ("filter", "pure"):
        check(x, 32, True, mode)


@pytest.mark.parametrize("k", [1, 2, 3, 7, 8, 31, 32, 33, 64, 100, 128, 255, 256, 257, 512,
                               777, 1000, 1024, 1025, 1500, 2047, 2048])
def test_every_k_ragged(cuda_device, k):
    n = (1 << 16) + 4096 * 3 + 13  # several tiles + ragged tail
    x = datagen.generate("uniform", n, "f32", seed=101)
    check(x, k, True)
    check(x, k, False)


@pytest.mark.parametrize("dist", ["uniform", "increasing", "decreasing", "fewdistinct",
                                  "bucketkiller"])
@pytest.mark.parametrize("largest", [True, False])
def test_distributions(cuda_device, dist, largest):
    n = (1 << 20) + 13
    x = datagen.generate(dist, n, "f32", seed=202)
    for k in (1, 64, 256, 1024, 2048):
        check(x, k, largest)
    check(x, 256, largest, mode="pure")


@pytest.mark.parametrize("dt", ["u32", "f64"])
@pytest.mark.parametrize("dist", ["uniform", "increasing", "fewdistinct"])
def test_dtypes(cuda_device, dt, dist):
    n = (1 << 18) + 5
    x = datagen.generate(dist, n, dt, seed=303)
    for k in (1, 64, 1000):
        for largest in (True, False):
            check(x, k, largest)


@pytest.mark.parametrize("dt", ["u32", "f64", "f32"])
def test_key_payload(cuda_device, dt):
    n = (1 << 18) + 3
    x = datagen.generate("uniform", n, dt, seed=404)
    p = datagen.payload(n, seed=404)
    check(x, 64, True, payload=p)
    check(x, 64, False, payload=p)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 7, 31, 1023, 4095, 4096, 4097, 8191, 8193])
def test_small_n(cuda_device, n):
    x = datagen.generate("fewdistinct", n, "f32", seed=n)
    for k in sorted({1, min(n // 2 + 1, 1024), min(n, 1024)}):
        check(x, k, True)
        check(x, k, False)


@pytest.mark.parametrize("offset", [1, 2, 3])
def test_misaligned_pointer(cuda_device, offset):
    x = datagen.generate("uniform", 100003, "f32", seed=505)
    check(x, 50, True, offset=offset)
    xd = datagen.generate("uniform", 50003, "f64", seed=505)
    check(xd, 50, True, offset=1)


def test_special_values(cuda_device):
    rng = np.random.default_rng(0)
    specials = np.array([np.nan, -np.nan, np.inf, -np.inf, 0.0, -0.0, 1.0, -1.0, 1e-45,
                         -1e-45, 3.4e38], np.float32)
    nan_payloads = np.array([0x7FC00001, 0xFFC00002, 0x7F800003], np.uint32).view(np.float32)
    vals = rng.choice(np.concatenate([specials, nan_payloads]), 70001)
    x = torch.from_numpy(vals)
    for k in (1, 5, 100, 1024):
        check(x, k, True)
        check(x, k, False)
    d = torch.from_numpy(rng.choice(specials.astype(np.float64), 30001))
    check(d, 77, True)
    check(d, 77, False)


def test_base_offset(cuda_device):
    x = datagen.generate("uniform", 300000, "f32", seed=606)
    check(x, 100, True, base=123456789012)


def test_merge_kernel(cuda_device):
    rng = np.random.default_rng(4)
    for runs, run_len, k in [(8, 256, 256), (4, 1024, 1000), (3, 5, 7), (16, 64, 64),
                             (1, 9000, 2048), (64, 1024, 1), (30, 2000, 500)]:
        vals = rng.choice(np.array([0.5, 1.0, np.nan, -0.0, 0.0, 2.0], np.float32),
                          runs * run_len)
        idx = rng.choice(10 ** 9, size=runs * run_len, replace=False).astype(np.int64)
        for largest in (True, False):
            v, i = tk.merge(torch.from_numpy(vals).cuda(), torch.from_numpy(idx).cuda(), k,
                            largest, runs=runs)
            ov, oi = oracle.topk(vals, k, largest, idx=idx)
            assert np.array_equal(i.cpu().numpy(), oi)
            assert v.cpu().numpy().tobytes() == ov.tobytes()


@pytest.mark.parametrize("runs,run_len,k", [(8, 256, 256), (2, 256, 256), (8, 1024, 1024),
                                            (4, 2048, 2048), (64, 256, 256), (3, 100, 77),
                                            (5, 300, 64), (16, 64, 1), (1, 512, 500),
                                            (32, 2048, 2048)])
@pytest.mark.parametrize("largest", [True, False])
def test_merge_sorted_runs(cuda_device, runs, run_len, k, largest):
    """topk_merge_sorted: runs sorted best first (each the oracle's top-run_len of a
    random tie-heavy block with distinct global ids) -> merge + rebuild rounds only;
    result == the oracle's top-k of all candidates."""
    rng = np.random.default_rng(runs * 1000 + run_len + k)
    vals, idxs = [], []
    pool = np.array([0.5, 1.0, np.nan, -0.0, 0.0, 2.0, -1.0, np.inf], np.float32)
    gids = rng.choice(10 ** 9, size=runs * run_len * 2, replace=False).astype(np.int64).reshape(runs, -1)
    for r in range(runs):
        block = rng.choice(pool, 2 * run_len)
        v, i = oracle.topk(block, run_len, largest, idx=gids[r])
        vals.append(v)
        idxs.append(i)
    cv, ci = np.concatenate(vals), np.concatenate(idxs)
    pay = rng.integers(0, 2 ** 32, cv.shape[0], dtype=np.uint64).astype(np.uint32)
    v, i, pv = tk.merge(torch.from_numpy(cv).cuda(), torch.from_numpy(ci).cuda(), k, largest,
                        cand_payload=torch.from_numpy(pay.view(np.int32)).cuda().view(torch.uint32),
                        runs=runs, sorted_runs=True)
    ov, oi = oracle.topk(cv, k, largest, idx=ci)
    assert np.array_equal(i.cpu().numpy(), oi)
    assert v.cpu().numpy().tobytes() == ov.tobytes()
    row = {int(g): j for j, g in enumerate(ci)}
    assert np.array_equal(host(pv), pay[[row[int(g)] for g in oi]])


def test_sharded_on_one_gpu(cuda_device):
    """The multi-GPU decomposition (§8(e)) with G virtual shards on one device:
    local top-k with base offsets, then the merge kernel == oracle on the whole."""
    n, k = (1 << 20) + 7, 256
    x = datagen.generate("uniform", n, "f32", seed=707)
    xd = x.cuda()
    for G in (2, 3, 8):
        cuts = [n * r // G for r in range(G + 1)]
        vs, is_ = [], []
        for r in range(G):
            v, i = tk.topk(xd[cuts[r]:cuts[r + 1]], k, True, base=cuts[r])
            vs.append(v)
            is_.append(i)
        ov, oi = oracle.topk(x.numpy(), k, True)
        for sorted_runs in (False, True):
            mv, mi = tk.merge(torch.cat(vs), torch.cat(is_), k, True, runs=G,
                              sorted_runs=sorted_runs)
            assert np.array_equal(mi.cpu().numpy(), oi)
            assert mv.cpu().numpy().tobytes() == ov.tobytes()


def test_repeated_calls_reuse_workspace(cuda_device):
    x = datagen.generate("uniform", 1 << 20, "f32", seed=808).cuda()
    ref = None
    for _ in range(5):
        v, i = tk.topk(x, 128)
        if ref is None:
            ref = i.clone()
        assert torch.equal(i, ref)


@pytest.mark.slow
@pytest.mark.parametrize("k", [32, 256, 1024])
def test_full_size_2p29_certificate(cuda_device, k):
    """BJ config 2 at full size (2^29 f32): the kernel in the bench's launch
    configuration, checked with the oracle's O(n) certificate, plus bit-exact
    equality with the oracle's own top-k."""
    n = 1 << 29
    xd = datagen.generate("uniform", n, "f32", seed=datagen.config_seed(2), device="cuda")
    v, i = tk.topk(xd, k, True)
    keys = xd.cpu().numpy()
    # generator parity device vs host on sampled rows
    rows = np.random.default_rng(1).integers(0, n, 1000)
    hx = np.concatenate([datagen.generate("uniform", 1, "f32", seed=datagen.config_seed(2),
                                          base=int(r), n_total=n).numpy() for r in rows[:50]])
    assert np.array_equal(hx, keys[rows[:50]])
    assert oracle.certificate(keys, k, v.cpu().numpy(), i.cpu().numpy(), True) == 0
    ov, oi = oracle.topk(keys, k, True)
    assert np.array_equal(oi, i.cpu().numpy())


@pytest.mark.parametrize("dt", ["f32", "u32", "f64"])
def test_host_resident_chunked(cuda_device, dt):
    """topk_select_host: pinned host keys streamed in chunks, ragged last chunk."""
    n = (1 << 21) + 12
    x = datagen.generate("uniform", n, dt, seed=909).pin_memory()
    for k, largest in ((1, True), (100, True), (1000, False)):
        v, i = tk.topk_host(x, k, largest, chunk_keys=1 << 18)
        torch.cuda.synchronize()
        ov, oi = oracle.topk(host(x), k, largest)
        assert np.array_equal(i.numpy(), oi)
        assert host(v).tobytes() == ov.tobytes()


def test_chunked_device_path(cuda_device):
    """n above one launch's row range is split into chunks + merge; forced small chunks
    (TOPK_CHUNK_N) exercise the same path on a small input in a subprocess."""
    import subprocess
    import sys
    code = (
        "import sys, numpy as np, torch; sys.path.insert(0, '.');"
        "import oracle; import paper_conf_sigmod_shanbhagpm18_b200 as tk;"
        "from paper_conf_sigmod_shanbhagpm18_b200 import datagen;"
        "x = datagen.generate('fewdistinct', (1<<20)+7, 'f32', seed=5);"
        "p = datagen.payload((1<<20)+7, seed=5);"
        "v, i, pv = tk.topk(x.cuda(), 300, True, payload=p.cuda(), base=11);"
        "ov, oi = oracle.topk(x.numpy(), 300, True, base=11);"
        "assert np.array_equal(i.cpu().numpy(), oi);"
        "assert v.cpu().numpy().tobytes() == ov.tobytes();"
        "pp = p.view(torch.int32).numpy().view(np.uint32);"
        "assert np.array_equal(pv.cpu().view(torch.int32).numpy().view(np.uint32), pp[oi - 11]);"
        "print('ok')")
    import os
    env = dict(os.environ, TOPK_CHUNK_N=str(1 << 18))
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]


@pytest.mark.parametrize("e64", [0, 1])
@pytest.mark.parametrize("Lp", [4, 5, 6, 7, 8, 9])
def test_code_network_order_statistics(cuda_device, e64, Lp):
    """cnet.cuh (the code-only local sort / merge / rebuild that yields the flush bounds)
    returns exactly the 2^Lp largest codes, best first (positions past n count as 0):
    the definition is a descending sort of the codes."""
    import ctypes
    from paper_conf_sigmod_shanbhagpm18_b200 import _lib
    lib = _lib.load()
    lib.topk_debug_cnet.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                    ctypes.c_void_p]
    rng = np.random.default_rng(1000 + 10 * Lp + e64)
    dt = np.uint64 if e64 else np.uint32
    hi = np.iinfo(dt).max
    Kp = 1 << Lp
    for n in (1, 17, 100, 511, 512, 513, 1000, 2048, 3840, 4096):
        cases = [rng.integers(0, hi, n, dtype=dt, endpoint=True),
                 (rng.integers(0, 7, n) * (hi // 7)).astype(dt),          # heavy ties
                 np.arange(n, dtype=dt), np.arange(n, dtype=dt)[::-1].copy(),
                 rng.integers(0, 2, n).astype(dt)]                         # 0/1 principle
        for codes in cases:
            d = torch.from_numpy(codes.view(np.int64 if e64 else np.int32)).to(cuda_device)
            out = torch.empty(Kp, dtype=torch.int64 if e64 else torch.int32, device=cuda_device)
            assert lib.topk_debug_cnet(e64, d.data_ptr(), n, Lp, out.data_ptr()) == 0
            got = out.cpu().numpy().view(dt)
            want = np.zeros(Kp, dtype=dt)
            srt = np.sort(codes)[::-1][:Kp]
            want[:len(srt)] = srt
            assert np.array_equal(got, want), (n, Lp, e64, got[:8], want[:8])


@pytest.mark.parametrize("dt", ["f32", "u32", "f64"])
def test_sharded_c_abi_one_rank(cuda_device, dt):
    """topk_select_sharded (local select -> ncclAllGather -> merge kernel) over a real
    one-rank NCCL communicator: global ids = base + i, bit-exact vs the oracle."""
    from paper_conf_sigmod_shanbhagpm18_b200.dist import NcclComm, sharded_topk_native
    comm = NcclComm(device=cuda_device)
    try:
        n, base = (1 << 20) + 7, 5 << 30
        x = datagen.generate("uniform", n, dt, seed=606)
        p = datagen.payload(n, seed=606)
        keys = host(x)
        for k, largest in ((1, True), (64, False), (1000, True)):
            v, i, pv = sharded_topk_native(x.to(cuda_device), k, comm, largest, base=base,
                                           payload=p.to(cuda_device))
            torch.cuda.synchronize()
            ov, oi = oracle.topk(keys, k, largest, base=base)
            assert np.array_equal(i.cpu().numpy(), oi)
            assert host(v).tobytes() == ov.tobytes()
            assert np.array_equal(host(pv), host(p)[oi - base])
    finally:
        comm.close()


def test_small_inputs_streaming_kernel(cuda_device):
    """Filter-mode calls with n <= 2^22 and k <= 32 run the pure kernel (same result, lower
    fixed cost); TOPK_PURE_SMALL_N=0 keeps them on the streaming kernel, whose small-input
    path (one tile per CTA, boot flush, tail) is checked here in a subprocess."""
    import os
    import subprocess
    import sys
    code = """
import sys
import numpy as np
sys.path.insert(0, '.')
import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import datagen
for n in (1, 7, 4096, 4097, 100003, (1 << 20) + 13):
    for dist in ('uniform', 'fewdistinct'):
        x = datagen.generate(dist, n, 'f32', seed=n)
        for k in (1, 8, 17, 32):
            if k > n:
                continue
            for lg in (True, False):
                v, i = tk.topk(x.cuda(), k, lg)
                ov, oi = oracle.topk(x.numpy(), k, lg)
                assert np.array_equal(i.cpu().numpy(), oi), (n, dist, k, lg)
                assert v.cpu().numpy().tobytes() == ov.tobytes(), (n, dist, k, lg)
print('ok')
"""
    env = dict(os.environ, TOPK_PURE_SMALL_N="0")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], cwd=root, env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]
