"""Pins for the oracle's sparsity probe, integer estimates, selector (PAPER.md:137-154,
§IV-B Eq. 1-4), LR time model and RAE."""
import itertools

import numpy as np
import pytest

import synth
from oracle import oracle as O


def full_counts(x):
    """numpy: zeros, zero-run starts, adjacent inequalities over the whole array."""
    z = x == 0
    starts = z & np.concatenate([[True], ~z[:-1]])
    return int(z.sum()), int(starts.sum()), int(np.count_nonzero(np.diff(x.astype(np.int64))))


@pytest.mark.parametrize("n", [1, 2, 255, 256, 1000, 1 << 18])
@pytest.mark.parametrize("dtype", [O.F32, O.F16])
def test_probe_is_exact_for_small_tensors(n, dtype):
    x = synth.relu_clustered(n, 0.6, 5, seed=n, dtype=dtype)
    zeros, zr, bnd = full_counts(x)
    assert O.probe(x, dtype) == (zeros, zr, bnd, n, n - 1)


def test_probe_windows_large():
    n = (1 << 18) + 12345
    x = synth.relu_iid(n, 0.3, seed=4)
    tot = np.zeros(3, np.int64)
    for k in range(1024):
        s0 = k * (n - 256) // 1023
        tot += full_counts(x[s0:s0 + 256])
    assert O.probe(x, O.F32) == (int(tot[0]), int(tot[1]), int(tot[2]), 1024 * 256, 1024 * 255)


def test_probe_estimate_accuracy_large():
    """The sampled estimate is within sampling error of the true counts (2^18 samples)."""
    n = 1 << 22
    x = synth.relu_iid(n, 0.55, seed=6)
    est = O.probe_estimates(n, O.probe(x, O.F32))
    zeros, zr, bnd = full_counts(x)
    assert abs(est[0] - zeros) / n < 0.005
    assert abs(est[2] - (bnd + 1)) / n < 0.01
    assert abs(est[3] - zr) / n < 0.01


def test_probe_estimates_integer_rounding():
    # zeros_hat = (zeros*n + samples/2) // samples : round half up, exact when n == samples
    assert O.probe_estimates(1000, (500, 10, 20, 1000, 999)) == (500, 500, 21, 10)
    assert O.probe_estimates(10, (1, 0, 0, 4, 3)) == (3, 7, 1, 0)       # 2.5 -> 3
    assert O.probe_estimates(5, (0, 0, 0, 0, 0))[1] == 0
    assert O.probe_estimates(7, (0, 0, 0, 1, 0)) == (0, 7, 1, 0)         # pairs == 0 -> r = 1


# ---------------------------------------------------------------- selector
def beta_const(tc=0.0, tdc=0.0, per_byte_c=0.0, per_byte_dc=0.0):
    b = np.zeros((4, 2, 6, 3))
    b[:, 0, :, 0], b[:, 1, :, 0] = tc, tdc
    b[:, 0, :, 1], b[:, 1, :, 1] = per_byte_c, per_byte_dc
    return b


def counts_for(n, s):
    """Exact probe counts of an iid tensor with sparsity s (small n => exact window)."""
    x = synth.relu_iid(n, s, seed=17, exact=True)
    return O.probe(x, O.F32)


def test_eq1_t_prime_closed_form():
    """Eq. 1: T' = max(S/BW_d2h - Hf, 0) + max(S/BW_h2d - Hb, 0)."""
    n = 1 << 16
    S = 4 * n
    cal = O.make_calib(bw_d2h=11.7e9, bw_h2d=10.6e9, mode=1)  # the paper's V100 link
    for hf, hb in [(0, 0), (1e-5, 0), (1, 1), (0, 1e-5)]:
        r = O.select(n, O.F32, counts_for(n, 0.5), hf, hb, cal)
        assert r["t_prime"] == pytest.approx(max(S / 11.7e9 - hf, 0) + max(S / 10.6e9 - hb, 0), rel=1e-12)


def test_paper_mode_zero_cost_codecs_compress_iff_sparse():
    """Orac-like case (zero codec time): with Eq. 2-4, T = S(1-s)(1/BWd+1/BWh)
    < T' iff s > 0; all four codecs tie, so the lowest id (ZVC) is chosen."""
    n = 4096
    cal = O.make_calib(bw_d2h=12e9, bw_h2d=12e9, mode=1)
    for s in (0.0, 0.1, 0.5, 0.9):
        c = counts_for(n, s)
        s_hat = c[0] / c[3]
        r = O.select(n, O.F32, c, 0, 0, cal)
        assert r["codec"] == (O.ZVC if s > 0 else O.NONE)
        assert r["t_pred"] == pytest.approx(2 * 4 * n * (1 - s_hat) / 12e9, rel=1e-12)


def test_tie_means_no_compression():
    """compress only if T' > T (strict)."""
    n = 4096
    cal = O.make_calib(bw_d2h=12e9, bw_h2d=12e9, mode=1)
    r = O.select(n, O.F32, counts_for(n, 0.0), 0, 0, cal)
    assert r["t_pred"] == r["t_prime"] and r["codec"] == O.NONE


def test_fully_hidden_transfer_never_compresses():
    n = 1 << 16
    cal = O.make_calib(bw_d2h=12e9, bw_h2d=12e9, beta=beta_const(1e-6, 1e-6), mode=0)
    r = O.select(n, O.F32, counts_for(n, 0.9), 1.0, 1.0, cal)
    assert r["t_prime"] == 0 and r["codec"] == O.NONE


def test_dense_never_zvc_pipelined():
    """s = 0: ZVC's exact size is S + S/32 + header > S, so ZVC can never win."""
    n = 1 << 16
    cal = O.make_calib(bw_d2h=12e9, bw_h2d=12e9, mode=0, margin=0.0)
    x = synth.relu_iid(n, 0.0, seed=1)
    r = O.select(n, O.F32, O.probe(x, O.F32), 0, 0, cal)
    assert r["size"][0] > 4 * n and r["codec"] != O.ZVC


def test_all_zero_prefers_rle_pipelined():
    n = 1 << 16
    # gamma2 = 1: one LZ4 length-extension byte per 255 bytes of zero-run match
    cal = O.make_calib(bw_d2h=12e9, bw_h2d=12e9, mode=0, lz4_gamma2=1.0)
    r = O.select(n, O.F32, O.probe(np.zeros(n, np.uint32), O.F32), 0, 0, cal)
    assert r["codec"] == O.RLE
    # RLE predicted = header(80) + subheader(16) + one length (16) + one value (16)
    assert r["size"][1] == 80 + 16 + 16 + 16


def test_pipelined_sizes_exact_for_single_frame():
    """With one frame and exact counts, the pipelined ZVC/CSR/RLE size predictions equal
    the real container sizes produced by the codecs."""
    n = 5000
    x = synth.relu_clustered(n, 0.6, 8, seed=2)
    cal = O.make_calib(mode=0, frame_elems=8192)
    r = O.select(n, O.F32, O.probe(x, O.F32), 0, 0, cal)
    assert r["size"][0] == len(O.compress(x, O.ZVC, O.F32, F=8192))
    assert r["size"][1] == len(O.compress(x, O.RLE, O.F32, F=8192))
    assert r["size"][2] == len(O.compress(x, O.CSR, O.F32, F=8192))


def test_pipelined_overlap_formula():
    """K frames overlap codec and copy: T_out = max(tc, x) + min(tc, x)/K."""
    n = 1 << 22
    F = 1 << 20
    # group_bytes = 0: one frame per swap-in step, so both directions are K-step pipelines
    cal = O.make_calib(bw_d2h=50e9, bw_h2d=50e9, beta=beta_const(1e-3, 2e-3), frame_elems=F, mode=0,
                       margin=0.0, group_bytes=0.0)
    x = synth.relu_iid(1 << 18, 0.5, seed=1, exact=True)
    counts = O.probe(x, O.F32)
    r = O.select(n, O.F32, counts, 0, 0, cal)
    size = r["size"][0]
    xo = size / 50e9
    assert r["t_codec"][0] == pytest.approx(max(1e-3, xo) + min(1e-3, xo) / 4 + max(2e-3, xo) + min(2e-3, xo) / 4,
                                            rel=1e-12)


def test_selector_brute_force_grid():
    """Exhaustive grid: the returned codec is the lowest-id argmin of the returned per-codec
    times, compression happens iff T(c*) < (1-m) T', and monotonicity in the link speed
    holds (a faster link never turns NONE into a compression)."""
    rng = np.random.default_rng(3)
    beta = rng.uniform(0, 1e-10, size=(4, 2, 6, 3))
    beta[..., 0] = rng.uniform(0, 2e-5, size=(4, 2, 6))
    for n, s, hf, hb, mode, bw in itertools.product([1000, 65536, 1 << 18], [0.0, 0.3, 0.7, 0.99],
                                                    [0, 1e-4], [0, 1e-4], [0, 1], [5e9, 50e9, 500e9]):
        cal = O.make_calib(bw_d2h=bw, bw_h2d=bw, alpha_d2h=2e-6, alpha_h2d=2e-6, beta=beta, mode=mode)
        r = O.select(n, O.F32, counts_for(n, s), hf, hb, cal)
        T = r["t_codec"]
        best = min(range(4), key=lambda i: (T[i], i))
        m = 0.0 if mode == 1 else 0.05
        near_tie = abs(T[best] - (1 - m) * r["t_prime"]) <= 1e-12 * max(r["t_prime"], 1e-30)
        if not near_tie:
            assert r["codec"] == (best + 1 if T[best] < (1 - m) * r["t_prime"] else O.NONE)
        if r["codec"] == O.NONE and bw < 500e9:
            cal2 = O.make_calib(bw_d2h=bw * 10, bw_h2d=bw * 10, alpha_d2h=2e-6, alpha_h2d=2e-6, beta=beta,
                                mode=mode)
            assert O.select(n, O.F32, counts_for(n, s), hf, hb, cal2)["codec"] == O.NONE


# ---------------------------------------------------------------- LR model + RAE
def test_lstsq_recovers_exact_linear_model():
    rng = np.random.default_rng(0)
    S = rng.uniform(20e6, 2000e6, 200)     # 20-2000 MB
    s = rng.uniform(0.2, 0.8, 200)         # 20-80 % sparsity
    beta = np.array([3e-5, 2.5e-13, -1.1e-13])
    t = beta[0] + beta[1] * S + beta[2] * S * s
    assert np.allclose(O.lstsq_fit(S, s, t), beta, rtol=1e-8, atol=1e-15)


def test_rae_hand_value():
    # mean(y) = 7/3; sum|yhat-y| = 1; sum|ybar-y| = 4/3 + 1/3 + 5/3 = 10/3 -> 0.3
    assert O.rae([1, 2, 3], [1, 2, 4]) == pytest.approx(0.3, rel=1e-14)
    assert O.rae([1, 2, 4], [1, 2, 4]) == 0.0
