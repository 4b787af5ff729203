"""GPU parity of the query form (topk_query: WHERE predicate fused as the buffer
filler, ORDER BY a ranking function evaluated inside the pass -- the paper's §5,
P:216-224) against the oracle's unfused plan (filter, project, top-k), bit-exact in
values and indices.  Inputs from the shared seeded generator; expected values only
from oracle/."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sigmod_shanbhagpm18_b200 as tk
from paper_conf_sigmod_shanbhagpm18_b200 import _lib, datagen

pytestmark = pytest.mark.gpu


def host(t: torch.Tensor) -> np.ndarray:
    if t.dtype == torch.uint32:
        return t.cpu().view(torch.int32).numpy().view(np.uint32)
    return t.cpu().numpy()


def u32col(n, seed, mod=None):
    c = datagen.generate("uniform", n, "u32", seed=seed)
    if mod is not None:
        c = (c.to(torch.int64) % mod).to(torch.uint32)
    return c


def run(keys, k, largest=True, rank_b=None, w=0.0, pred=None, payload=None):
    """GPU query vs oracle.query on the same host columns."""
    dev = "cuda"
    gpred = None if pred is None else (pred[0], pred[1].to(dev), *pred[2:])
    out = tk.query(keys.to(dev), k, largest, rank_b=None if rank_b is None else rank_b.to(dev),
                   rank_w=w, pred=gpred, payload=None if payload is None else payload.to(dev))
    torch.cuda.synchronize()
    hpred = None if pred is None else (pred[0], host(pred[1]), *pred[2:])
    ov, oi, m = oracle.query(host(keys), k, largest,
                             rank_b=None if rank_b is None else host(rank_b), rank_w=w,
                             pred=hpred)
    gi = out[1].cpu().numpy()
    assert np.array_equal(gi, oi), f"indices differ (m={m}): first at {np.nonzero(gi != oi)[0][:5]}"
    assert host(out[0]).tobytes() == ov.tobytes(), "value bits differ"
    if payload is not None:
        ph = host(payload)
        exp = np.where(oi >= 0, ph[np.maximum(oi, 0)], 0).astype(np.uint32)
        assert np.array_equal(host(out[2]), exp)
    return m


N = (1 << 20) + 4096 * 3 + 7  # many tiles, ragged tail (n % 4 != 0)


@pytest.mark.parametrize("dt", ["f32", "u32", "f64"])
@pytest.mark.parametrize("largest", [True, False])
def test_range_predicate_selectivities(cuda_device, dt, largest):
    keys = datagen.generate("uniform", N, dt, seed=301)
    col = u32col(N, 302, 1000)
    for lo, hi in [(0, 1000), (0, 500), (250, 260), (999, 1000), (0, 0)]:
        for k in (1, 50, 256):
            run(keys, k, largest, pred=("range", col, lo, hi))


@pytest.mark.parametrize("k", [1, 7, 32, 64, 100, 256, 512, 1024, 2048])
def test_every_k_in_predicate(cuda_device, k):
    keys = datagen.generate("uniform", N, "f32", seed=303)
    lang = u32col(N, 304, 70)  # dictionary codes; >= 64 never match
    run(keys, k, True, pred=("in", lang, (1 << 3) | (1 << 5)))
    run(keys, k, False, pred=("in", lang, 1 << 63))


@pytest.mark.parametrize("largest", [True, False])
def test_ranking_function(cuda_device, largest):
    a = datagen.generate("uniform", N, "f32", seed=305)
    b = datagen.generate("uniform", N, "f32", seed=306)
    for w in (0.5, -1.25, 3.0e-3):
        for k in (1, 64, 256, 1000):
            run(a, k, largest, rank_b=b, w=w)


def test_ranking_special_values(cuda_device):
    a = datagen.generate("uniform", 100000, "f32", seed=307)
    b = datagen.generate("uniform", 100000, "f32", seed=308)
    sp_a = torch.tensor([float("nan"), -0.0, 0.0, float("inf"), -float("inf"), 1e-40, 2.0, 1.0],
                        dtype=torch.float32)
    sp_b = torch.tensor([1.0, 0.0, -0.0, -1.0, 5.0, 1e-40, float("nan"), float("inf")],
                        dtype=torch.float32)
    for j in range(8):
        a[j * 9973] = sp_a[j]
        b[j * 9973] = sp_b[j]
    for largest in (True, False):
        run(a, 20, largest, rank_b=b, w=0.5)


def test_integer_counts_query2(cuda_device):
    """P:298 query 2: retweet_count + 0.5 * likes_count (integer counts in f32)."""
    rt = (u32col(N, 309, 5000).to(torch.float32))
    likes = (u32col(N, 310, 20000).to(torch.float32))
    run(rt, 50, True, rank_b=likes, w=0.5)


def test_rank_and_predicate(cuda_device):
    a = datagen.generate("uniform", N, "f32", seed=311)
    b = datagen.generate("uniform", N, "f32", seed=312)
    t = u32col(N, 313)
    run(a, 256, True, rank_b=b, w=0.5, pred=("range", t, 0, 1 << 30))
    run(a, 64, False, rank_b=b, w=2.0, pred=("in", (t.to(torch.int64) % 64).to(torch.uint32), 0xF0F0))


def test_fewer_matches_than_k(cuda_device):
    keys = datagen.generate("uniform", N, "f32", seed=314)
    rowid = torch.arange(N, dtype=torch.int64).to(torch.uint32)
    for lo, hi in [(5, 5), (100, 120), (N - 3, N), (N - 1000, N)]:
        m = run(keys, 256, True, pred=("range", rowid, lo, hi))
        assert m == min(256, hi - lo)


@pytest.mark.parametrize("dist", ["increasing", "decreasing", "fewdistinct"])
def test_adversarial_with_time_predicate(cuda_device, dist):
    """Query 1 shape: WHERE tweet_time < X, time = row order (appended log)."""
    keys = datagen.generate(dist, N, "f32", seed=315)
    t = torch.arange(N, dtype=torch.int64).to(torch.uint32)
    for X in (N // 10, N // 2, N):
        run(keys, 50, True, pred=("range", t, 0, X))
        run(keys, 50, False, pred=("range", t, 0, X))


def test_payload_and_small_n(cuda_device):
    for n in (1, 3, 4, 5, 17, 4096, 7681):
        keys = datagen.generate("uniform", n, "f32", seed=316 + n)
        col = u32col(n, 317, 4)
        pay = datagen.payload(n, seed=318)
        k = min(n, 16)
        run(keys, k, True, pred=("range", col, 1, 3), payload=pay)


def test_rejects_bad_arguments(cuda_device):
    keys = torch.rand(1024, device="cuda")
    col = torch.zeros(1024, dtype=torch.uint32, device="cuda")
    with pytest.raises(_lib.TopkError):  # misaligned column
        tk.query(keys[1:], 8, pred=("range", col[1:], 0, 1))
    with pytest.raises(_lib.TopkError):  # ranking function needs f32
        tk.query(keys.double(), 8, rank_b=keys)
    with pytest.raises(_lib.TopkError):  # neither predicate nor ranking function
        tk.query(keys, 8)


@pytest.mark.slow
def test_full_size_query1(cuda_device):
    """2^28 rows (BJ config-4 size): WHERE time < X ORDER BY count DESC LIMIT 50."""
    n = 1 << 28
    keys = datagen.generate("uniform", n, "u32", seed=319)
    t = u32col(n, 320)
    run(keys, 50, True, pred=("range", t, 0, 1 << 31))


# ---- compound keys: ORDER BY k1, k2 LIMIT k (KKV) ----

def run_kk(k1, k2, k, l1=True, l2=True, pred=None, payload=None):
    dev = "cuda"
    gpred = None if pred is None else (pred[0], pred[1].to(dev), *pred[2:])
    out = tk.topk_kk(k1.to(dev), k2.to(dev), k, l1, l2, pred=gpred,
                     payload=None if payload is None else payload.to(dev))
    torch.cuda.synchronize()
    h1, h2 = host(k1), host(k2)
    if pred is None:
        o1, o2, oi = oracle.topk_kk(h1, h2, k, l1, l2)
    else:  # the plain plan: filter, then the compound top-k over the survivors
        c = host(pred[1])
        keep = (c >= pred[2]) & (c < pred[3]) if pred[0] == "range" else \
            (c < 64) & (((np.uint64(pred[2]) >> np.minimum(c, 63).astype(np.uint64)) & np.uint64(1)) == 1)
        rows = np.nonzero(keep)[0]
        m = min(k, rows.shape[0])
        oi = np.full(k, -1, dtype=np.int64)
        o1 = np.zeros(k, dtype=np.float32)
        o2 = np.zeros(k, dtype=np.float32)
        if m:
            a1, a2, ii = oracle.topk_kk(h1[rows], h2[rows], m, l1, l2)
            oi[:m], o1[:m], o2[:m] = rows[ii], a1, a2
    gi = out[2].cpu().numpy()
    assert np.array_equal(gi, oi), f"indices differ: first at {np.nonzero(gi != oi)[0][:5]}"
    assert host(out[0]).tobytes() == o1.tobytes() and host(out[1]).tobytes() == o2.tobytes()
    if payload is not None:
        ph = host(payload)
        exp = np.where(oi >= 0, ph[np.maximum(oi, 0)], 0).astype(np.uint32)
        assert np.array_equal(host(out[3]), exp)


@pytest.mark.parametrize("l1", [True, False])
@pytest.mark.parametrize("l2", [True, False])
def test_compound_keys(cuda_device, l1, l2):
    k1 = datagen.generate("fewdistinct", N, "f32", seed=321)  # 16 values: k2 decides
    k2 = datagen.generate("uniform", N, "f32", seed=322)
    for k in (1, 8, 64, 256, 1024, 2048):
        run_kk(k1, k2, k, l1, l2)


def test_compound_keys_ties_and_specials(cuda_device):
    k1 = datagen.generate("fewdistinct", N, "f32", seed=323)
    k2 = datagen.generate("fewdistinct", N, "f32", seed=324)  # full ties: row id decides
    run_kk(k1, k2, 300, True, False)
    k1 = datagen.generate("uniform", 200000, "f32", seed=325)
    k2 = datagen.generate("uniform", 200000, "f32", seed=326)
    for j, (a, b) in enumerate([(float("nan"), 1.0), (float("nan"), float("nan")), (-0.0, 2.0),
                                (0.0, 2.0), (float("inf"), -float("inf")), (1.0, float("nan"))]):
        k1[j * 31337] = a
        k2[j * 31337] = b
    for l1 in (True, False):
        for l2 in (True, False):
            run_kk(k1, k2, 16, l1, l2)


@pytest.mark.parametrize("dist", ["uniform", "increasing", "decreasing"])
def test_compound_keys_predicate_payload(cuda_device, dist):
    k1 = datagen.generate(dist, N, "f32", seed=327)
    k2 = datagen.generate("uniform", N, "f32", seed=328)
    col = u32col(N, 329, 100)
    pay = datagen.payload(N, seed=330)
    run_kk(k1, k2, 64, True, True, pred=("range", col, 10, 60), payload=pay)
    run_kk(k1, k2, 64, False, True, pred=("in", col, (1 << 7) | (1 << 40)), payload=pay)


# ---- three compound keys: ORDER BY k1, k2, k3 LIMIT k (KKKV) ----

def run_kkk(cols, k, orders=(True, True, True), pred=None, payload=None):
    dev = "cuda"
    gpred = None if pred is None else (pred[0], pred[1].to(dev), *pred[2:])
    out = tk.topk_kkk(*[c.to(dev) for c in cols], k, orders, pred=gpred,
                      payload=None if payload is None else payload.to(dev))
    torch.cuda.synchronize()
    h = [host(c) for c in cols]
    oi = np.full(k, -1, dtype=np.int64)
    ov = [np.zeros(k, dtype=np.float32) for _ in range(3)]
    rows = np.arange(h[0].shape[0])
    if pred is not None:  # the plain plan: filter, then the compound top-k
        c = host(pred[1])
        rows = np.nonzero((c >= pred[2]) & (c < pred[3]))[0]
    m = min(k, rows.shape[0])
    if m:
        r = oracle.topk_kkk(*[x[rows] for x in h], m, orders)
        oi[:m] = rows[r[3]]
        for j in range(3):
            ov[j][:m] = r[j]
    gi = out[3].cpu().numpy()
    assert np.array_equal(gi, oi), f"indices differ: first at {np.nonzero(gi != oi)[0][:5]}"
    for j in range(3):
        assert host(out[j]).tobytes() == ov[j].tobytes()
    if payload is not None:
        ph = host(payload)
        assert np.array_equal(host(out[4]), np.where(oi >= 0, ph[np.maximum(oi, 0)], 0).astype(np.uint32))


@pytest.mark.parametrize("orders", [(True, True, True), (False, True, False), (True, False, True)])
def test_three_keys(cuda_device, orders):
    cols = [datagen.generate("fewdistinct", N, "f32", seed=331),
            datagen.generate("fewdistinct", N, "f32", seed=332),
            datagen.generate("uniform", N, "f32", seed=333)]
    for k in (1, 64, 256, 2048):
        run_kkk(cols, k, orders)


def test_three_keys_full_ties_predicate_payload(cuda_device):
    # three independent 16-value columns: 16^3 = 4096 distinct tuples over N rows, so
    # every tuple repeats and key 2 / key 3 / the row id all decide somewhere
    cols = [datagen.generate("fewdistinct", N, "f32", seed=334 + 10 * j) for j in range(3)]
    h = [c.numpy() for c in cols]
    assert len({(a, b) for a, b in zip(h[0][:4096], h[1][:4096])}) > 16  # columns differ
    run_kkk(cols, 500, (True, True, False))
    col = u32col(N, 335, 10)
    pay = datagen.payload(N, seed=336)
    run_kkk(cols, 64, (False, False, True), pred=("range", col, 3, 8), payload=pay)


@pytest.mark.parametrize("form", ["kk", "kkk", "rank", "pred"])
def test_query_forms_repeated_calls_identical(form):
    """The boot sample (select.cuh) runs in every query form: the first tile's best row per
    thread is flushed, the bag emptied and the tile re-read against the bound weakened by
    one entry step (E32 / E64 / E96 words).  The schedule is timing-dependent, the answer
    must not be: 12 calls each, every one equal to the oracle."""
    n = (1 << 22) + 4
    a, b, c = (datagen.generate("uniform", n, "f32", seed=31 + j) for j in range(3))
    col = u32col(n, 34)
    ad, bd, cd, cold = a.cuda(), b.cuda(), c.cuda(), col.cuda()
    if form == "kk":
        f, exp = lambda: tk.topk_kk(ad, bd, 300)[2], oracle.topk_kk(host(a), host(b), 300)[2]
    elif form == "kkk":
        f = lambda: tk.topk_kkk(ad, bd, cd, 300)[3]
        exp = oracle.topk_kkk(host(a), host(b), host(c), 300)[3]
    elif form == "rank":
        f = lambda: tk.query(ad, 300, True, rank_b=bd, rank_w=0.5)[1]
        exp = oracle.query(host(a), 300, True, rank_b=host(b), rank_w=0.5)[1]
    else:
        f = lambda: tk.query(ad, 300, True, pred=("range", cold, 0, 1 << 31))[1]
        exp = oracle.query(host(a), 300, True, pred=("range", host(col), 0, 1 << 31))[1]
    bad = sum(int(not np.array_equal(f().cpu().numpy(), exp)) for _ in range(12))
    assert bad == 0, f"{bad}/12 calls wrong"
