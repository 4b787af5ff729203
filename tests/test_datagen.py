"""Pins of the shared input generator (CPU only): splitmix64 against a pure-Python
big-integer implementation, shard consistency, and the closed-form distributions."""
import numpy as np
import torch

from paper_conf_sigmod_shanbhagpm18_b200 import datagen

M = (1 << 64) - 1


def splitmix_ref(state: int) -> int:
    z = state & M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def test_stream_matches_bigint_reference():
    seed = 0x5EED0001
    for lo in (0, 12345, (1 << 32) - 3):
        z = datagen.stream(seed, lo, lo + 64, "cpu")
        for j in range(64):
            i = lo + j
            want = splitmix_ref(seed + 0x9E3779B97F4A7C15 * (i + 1))
            assert (int(z[j]) & M) == want


def test_uniform_f32_grid():
    x = datagen.generate("uniform", 4096, "f32")
    z = datagen.stream(0x5EED0001, 0, 4096, "cpu")
    want = np.array([(int(v) & M) >> 40 for v in z], dtype=np.float64) * 2.0 ** -24
    assert np.array_equal(x.numpy().astype(np.float64), want)
    assert float(x.min()) >= 0.0 and float(x.max()) < 1.0


def test_u32_and_f64():
    z = datagen.stream(7, 0, 256, "cpu")
    u = datagen.generate("uniform", 256, "u32", seed=7)
    assert [int(a) for a in u.to(torch.int64)] == [(int(v) & M) >> 32 for v in z]
    d = datagen.generate("uniform", 256, "f64", seed=7)
    assert np.array_equal(d.numpy(), np.array([((int(v) & M) >> 11) * 2.0 ** -53 for v in z]))


def test_shards_equal_full():
    for dist in ("uniform", "increasing", "decreasing", "fewdistinct"):
        for dt in ("f32", "u32", "f64"):
            full = datagen.generate(dist, 10000, dt)
            parts = [datagen.generate(dist, 2500, dt, base=b, n_total=10000)
                     for b in range(0, 10000, 2500)]
            assert torch.equal(torch.cat(parts), full), (dist, dt)


def test_ramps_and_fewdistinct():
    n = 1 << 20
    inc = datagen.generate("increasing", n, "f32").numpy()
    assert np.all(np.diff(inc) >= 0) and inc[0] == 0.0
    assert np.array_equal(inc, np.floor(np.arange(n) * 2.0 ** 24 / n) * 2.0 ** -24)
    dec = datagen.generate("decreasing", n, "f32").numpy()
    assert np.array_equal(dec, inc[::-1])
    few = datagen.generate("fewdistinct", n, "f32").numpy()
    assert set(np.unique(few).tolist()) == {j / 16 for j in range(16)}


def test_bucketkiller():
    n = 1 << 16
    x = datagen.generate("bucketkiller", n, "f32").numpy()
    pos, bits = datagen.bucketkiller_specials(0x5EED0001, n)
    assert sorted(bits) == sorted([0x3F80005A, 0x3F805A00, 0x3FDA0000, 0x65800000])
    ne = np.nonzero(x != 1.0)[0]
    assert sorted(ne.tolist()) == sorted(pos)
    assert sorted(x[ne].view(np.uint32).tolist()) == sorted(bits)


def test_payload_differs_from_index():
    p = datagen.payload(1000)
    assert (p.to(torch.int64) != torch.arange(1000)).sum() > 990
