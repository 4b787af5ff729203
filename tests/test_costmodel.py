"""The paper's cost model (§7) against the numbers it prints (CPU only).

P:341: for top-32 on 2^29 floats on Titan X, T_g = 8.96 ms, T_k = 12.1 ms, estimate
max = 12.1 ms (actual 14.2 ms); the first radix kernel "should take 8.6 ms based
on model".  The paper's own units are not consistent: T_g = 8.96 ms
needs B_G = 251 GiB/s, the 8.6 ms radix kernel needs 251 GB/s -- both are pinned with
the unit each needs."""
import math

import pytest

from paper_conf_sigmod_shanbhagpm18_b200 import costmodel as cm

N, W = 1 << 29, 4


def test_bitonic_tg_matches_p341():
    t = cm.bitonic_tg(N, W, cm.TITAN_X, x=8)
    assert t * 1e3 == pytest.approx(8.96, abs=0.01)


def test_bitonic_tk_matches_p341_within_units():
    tk = cm.sortreducer_smem_factor(32) * N * W / cm.TITAN_X.b_s
    assert cm.sortreducer_smem_factor(32) == 17.5
    assert 11.7e-3 < tk < 13.0e-3                           # 12.1 ms printed (TB vs TiB)
    assert tk > cm.bitonic_tg(N, W, cm.TITAN_X)             # smem-bound, as P:341 says


def test_radix_first_kernel_matches_p343():
    hw = cm.Hardware(b_g=251e9, b_s=2.9e12, n_t=cm.TITAN_X.n_t)
    d, _ = cm.radix_passes(N, W)[0]
    t11 = d / hw.b_g + 16 * 4 * hw.n_t / hw.b_g             # T_11
    assert t11 * 1e3 == pytest.approx(8.6, abs=0.06)


def test_radix_passes_structure():
    p = cm.radix_passes(N, W)
    assert len(p) == 4                                      # "4 passes for 32 bit"
    assert p[0][0] == N * W and p[1][0] == pytest.approx(N * W / 256)
    assert len(cm.radix_passes(N, 8)) == 8
    # eta = 1 skips the scatter ("skipped if eta_i = 1")
    hw = cm.TITAN_X
    t_skip = cm.radix_time(N, W, hw, etas=[1.0] * 4)
    assert t_skip < 4 * (N * W / hw.b_g) * 1.01


def test_crossover_direction():
    """The model prefers bitonic for small K and its cost grows with K."""
    hw = cm.TITAN_X
    assert cm.choose(N, W, 32, hw) == "bitonic"
    ts = [cm.bitonic_time(N, W, 1 << j, hw) for j in range(0, 11)]
    assert all(b >= a for a, b in zip(ts, ts[1:]))
    assert cm.choose(N, W, 1024, hw) == "radix"
    hb = cm.b200(6563.0)
    assert hb.b_s == pytest.approx(148 * 128 * 1.965e9)
    assert math.isfinite(cm.radix_time(N, W, hb))


def test_b200_model_prefers_one_pass():
    """One read of the input (the B200 pass) beats radix's >= 2 reads at any k."""
    hb = cm.b200(6563.0)
    assert cm.bitonic_b200_time(N, W, hb) == pytest.approx(N * W / hb.b_g)
    for k in (1, 32, 256, 1024, 2048):
        assert cm.choose_b200(N, W, k, hb) == "bitonic"
