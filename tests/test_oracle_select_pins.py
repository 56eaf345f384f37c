"""Hand-computed pins for the parts of the oracle's selector (`orc_select`, PAPER.md:137-154
§IV-B Eq. 1-4; :164-168 §IV-C) and of `orc_max_size` that the round-1 tests left unpinned
("What's weak" #1).  Every expected number below was worked out by hand from the
paper's formulas and the DESIGN.md readings, and is written as a literal (the arithmetic is in
the comments), so a dropped term, a wrong band edge, a swapped direction or a misplaced
alignment in the oracle fails here.

Readings used (DESIGN.md §2 / §3.3): R14 bands [0,.2) [.2,.35) [.35,.5) [.5,.65) [.65,.8)
[.8,1]; R10/R11 paper mode = Size*(1-s) and the Eq. 2 sum with alpha = 0; pipelined mode =
exact container sizes and T_out = max(t_c, x) + min(t_c, x)/K; R19 u64 round-half-up estimates.
"""
import numpy as np
import pytest

from oracle import oracle as O

ZVC, RLE, CSR, LZ4 = O.ZVC, O.RLE, O.CSR, O.LZ4


def beta_bands(c0, d0):
    """beta[codec][dir][band] = [b0, 0, 0] with b0 = c0(band) / d0(band)."""
    b = np.zeros((4, 2, 6, 3))
    for band in range(6):
        b[:, 0, band, 0] = c0(band)
        b[:, 1, band, 0] = d0(band)
    return b


# ------------------------------------------------------------------ band edges (R14, :166-168)
@pytest.mark.parametrize("zeros,band", [
    (0, 0), (199, 0),          # s = 0.199 -> [0, .2)
    (200, 1), (349, 1),        # s = 0.2 sits in the second band; 0.349 too
    (350, 2), (499, 2),        # 0.35 -> [.35, .5)
    (500, 3), (649, 3),        # 0.5 -> [.5, .65)
    (650, 4), (799, 4),        # 0.65 -> [.65, .8)
    (800, 5), (1000, 5),       # 0.8 and above -> [.8, 1]
])
def test_band_edges_pick_the_right_sub_model(zeros, band):
    # n = 1000 fp32, exact window: s_hat = zeros / 1000; zeros / 1000 in double is the double
    # nearest the decimal, i.e. the same double as the edge literal, so s_hat == edge exactly
    cal = O.make_calib(beta=beta_bands(lambda b: (b + 1) * 1e-6, lambda b: (b + 1) * 1e-7), mode=0)
    r = O.select(1000, O.F32, (zeros, 1, 2, 1000, 999), 0.0, 0.0, cal)
    assert r["t_c"] == [(band + 1) * 1e-6] * 4
    assert r["t_dc"] == [(band + 1) * 1e-7] * 4


# ------------------------------------------------------------------ t = b0 + b1 S + b2 S s
def test_time_model_size_and_sparsity_terms():
    b = np.zeros((4, 2, 6, 3))
    b[ZVC - 1, 0, 3] = [1e-6, 2e-9, 3e-9]    # band 3 (s = 0.5)
    b[ZVC - 1, 1, 3] = [2e-6, 1e-9, -1e-9]
    b[CSR - 1, 0, 5] = [0.0, 1e-9, 1e-9]     # band 5 (s = 0.8)
    cal = O.make_calib(beta=b, mode=0)
    # n = 1000 fp32: S = 4000 B.  s = 0.5: t_c = 1e-6 + 2e-9*4000 + 3e-9*4000*0.5 = 1e-6 + 8e-6 + 6e-6
    r = O.select(1000, O.F32, (500, 1, 2, 1000, 999), 0.0, 0.0, cal)
    assert r["t_c"][ZVC - 1] == pytest.approx(1.5e-5, rel=1e-12)
    # t_dc = 2e-6 + 1e-9*4000 - 1e-9*2000 = 2e-6 + 4e-6 - 2e-6
    assert r["t_dc"][ZVC - 1] == pytest.approx(4e-6, rel=1e-12)
    # s = 0.8: t_c(CSR) = 1e-9*4000 + 1e-9*4000*0.8 = 4e-6 + 3.2e-6
    r = O.select(1000, O.F32, (800, 1, 2, 1000, 999), 0.0, 0.0, cal)
    assert r["t_c"][CSR - 1] == pytest.approx(7.2e-6, rel=1e-12)
    assert r["t_c"][ZVC - 1] == 0.0  # band 5 of ZVC is all zero


# ------------------------------------------------------------------ predicted sizes, K = 1
def blocks_tensor():
    """2048 fp32: 16 x (64 x 1.0, 64 x 0) -> 1024 zeros, 16 zero runs, 31 value changes."""
    one = np.uint32(0x3F800000)
    x = np.zeros(2048, np.uint32)
    for b in range(16):
        x[128 * b:128 * b + 64] = one
    return x


def test_predicted_sizes_single_frame_by_hand():
    x = blocks_tensor()
    counts = O.probe(x, O.F32)
    assert counts == (1024, 16, 31, 2048, 2047)  # exact window (n <= 2^18)
    cal = O.make_calib(mode=0, lz4_gamma1=3.0, lz4_gamma2=1.0)  # F = 2^22 > n: K = 1
    size = O.select(2048, O.F32, counts, 0.0, 0.0, cal)["size"]
    # header align16(64 + 8) = 80
    # ZVC: 80 + align16(4 * 2048/32 = 256) + align16(4 * 1024) = 80 + 256 + 4096
    assert size[ZVC - 1] == 4432
    # RLE: r_hat = 1 + 31 = 32: 80 + 16 + align16(4 * 32) + align16(4 * 32)
    assert size[RLE - 1] == 352
    # CSR (C = 1024, R = 2): 80 + align16(4 * 3) + 4096 + 4096
    assert size[CSR - 1] == 8288
    # LZ4 (B = 65536, one 8192-byte block): 80 + align16(4) + 4 * 1024 + 3 * 16 + 1 * 4 * 1024 / 255
    assert size[LZ4 - 1] == pytest.approx(96 + 4096 + 48 + 4096 / 255, rel=1e-15)
    assert size[LZ4 - 1] == pytest.approx(4256.062745098039, rel=1e-15)
    # and the three exact-format predictions equal the real containers (codec code, not selector)
    for c in (ZVC, RLE, CSR):
        assert size[c - 1] == len(O.compress(x, c, O.F32))


# ------------------------------------------------------------------ K = 3 ragged frames
def ragged_frames_tensor():
    """n = 2500 fp32 in frames of F = 1024 (1024, 1024, 452 elements).  Every frame has a
    multiple of 4 non-zeros and runs (so per-frame 16-byte alignment adds nothing) and the value
    does not change across frame boundaries (so the runs are 1 + changes + K - 1)."""
    f = lambda v: np.uint32(np.float32(v).view(np.uint32))  # noqa: E731
    z = [np.uint32(0)]
    fr0 = z * 256 + [f(1)] * 256 + [f(2)] * 256 + z * 256            # nnz 512, 4 runs
    fr1 = z * 100 + [f(3)] * 128 + [f(4)] * 128 + z * 668            # nnz 256, 4 runs
    fr2 = z * 52 + [f(5)] * 50 + [f(6)] * 50 + z * 300               # nnz 100, 4 runs
    x = np.array(fr0 + fr1 + fr2, np.uint32)
    assert x.size == 2500
    return x


def test_predicted_sizes_three_ragged_frames_by_hand():
    x = ragged_frames_tensor()
    counts = O.probe(x, O.F32)
    # zeros 1632; zero runs start at 0, 768, 1380, 2200 (frames 1 and 2 continue a zero run);
    # 3 changes per frame, none at the frame boundaries
    assert counts == (1632, 4, 9, 2500, 2499)
    cal = O.make_calib(mode=0, frame_elems=1024, lz4_gamma1=3.0, lz4_gamma2=1.0)
    size = O.select(2500, O.F32, counts, 0.0, 0.0, cal)["size"]
    # header align16(64 + 8*3) = 96; bitmaps align16(4*32) x 2 + align16(4*15) = 128 + 128 + 64;
    # values align16(4 * 868) = 3472
    assert size[ZVC - 1] == 96 + 320 + 3472 == 3888
    # CSR (C = 1024, one row per frame): row_ptr align16(8) x 3 = 48; col + values 2 x 3472
    assert size[CSR - 1] == 96 + 48 + 6944 == 7088
    # RLE: r = r_hat + K - 1 = (1 + 9) + 2 = 12; sub-headers 3 x 16; lengths / values align16(48)
    assert size[RLE - 1] == 96 + 48 + 48 + 48 == 240
    # LZ4: block tables align16(4) x 3 = 48; 4 * 868 + 3 * 4 + 4 * 1632 / 255 (= 25.6 exactly)
    assert size[LZ4 - 1] == pytest.approx(96 + 48 + 3472 + 12 + 25.6, rel=1e-15)
    for c in (ZVC, RLE, CSR):
        assert size[c - 1] == len(O.compress(x, c, O.F32, F=1024))


# ------------------------------------------------------------------ alpha in pipelined T' and T
def test_alpha_enters_t_prime_and_t_pipelined_single_frame():
    b = np.zeros((4, 2, 6, 3))
    b[:, 0, 5, 0] = 4e-6    # t_c  (all-zero tensor: band 5)
    b[:, 1, 5, 0] = 3e-5    # t_dc
    cal = O.make_calib(alpha_d2h=1e-5, bw_d2h=4e8, alpha_h2d=2e-5, bw_h2d=2e8, beta=b, mode=0, margin=0.0)
    r = O.select(1000, O.F32, (1000, 1, 0, 1000, 999), 0.5e-5, 5e-5, cal)
    # T' = max(1e-5 + 4000/4e8 - 0.5e-5, 0) + max(2e-5 + 4000/2e8 - 5e-5, 0) = 1.5e-5 + 0
    assert r["t_prime"] == pytest.approx(1.5e-5, rel=1e-12)
    # ZVC size = 80 + align16(128) + 0 = 208: x_o = 1e-5 + 5.2e-7, x_i = 2e-5 + 1.04e-6
    # K = 1: T_out = 1.052e-5 + 4e-6 = 1.452e-5; T_in = 3e-5 + 2.104e-5 = 5.104e-5
    # T = (1.452e-5 - 0.5e-5) + (5.104e-5 - 5e-5) = 0.952e-5 + 0.104e-5
    assert r["size"][ZVC - 1] == 208
    assert r["t_codec"][ZVC - 1] == pytest.approx(1.056e-5, rel=1e-9)
    # CSR is smaller still (80 + align16(8) = 96 B): x_o = 1.024e-5, x_i = 2.048e-5,
    # T = (1.024e-5 + 4e-6 - 0.5e-5) + (3e-5 + 2.048e-5 - 5e-5) = 0.924e-5 + 0.048e-5, the argmin
    # (RLE 128 B -> 0.996e-5; LZ4 96 + 3 + 4000/255 B -> 0.986e-5)
    assert r["size"][CSR - 1] == 96
    assert r["t_codec"][CSR - 1] == pytest.approx(0.972e-5, rel=1e-9)
    assert r["t_codec"][RLE - 1] == pytest.approx(0.996e-5, rel=1e-9)
    assert r["codec"] == CSR and r["t_pred"] == r["t_codec"][CSR - 1]


@pytest.mark.parametrize("group_bytes,t_zvc", [
    (0.0, 1.4e-5),            # one frame per swap-in step: G = K = 4, T_in = 8e-6 + 3e-6/4
    (256.0, 1.475e-5),        # frames of (608 - 96)/4 = 128 B, q = 2 per step: G = 2, T_in = 8e-6 + 3e-6/2
    (float(32 << 20), 1.625e-5),  # one step: G = 1, T_in = 8e-6 + 3e-6
])
def test_alpha_with_four_frames_and_swap_in_groups(group_bytes, t_zvc):
    b = np.zeros((4, 2, 6, 3))
    b[:, 0, 5, 0] = 1e-6
    b[:, 1, 5, 0] = 8e-6
    cal = O.make_calib(alpha_d2h=4e-6, bw_d2h=6.08e8, alpha_h2d=1e-6, bw_h2d=3.04e8, beta=b, mode=0,
                       frame_elems=1024, group_bytes=group_bytes)
    r = O.select(4096, O.F32, (4096, 1, 0, 4096, 4095), 0.0, 0.0, cal)
    # K = 4; ZVC size = align16(64 + 32) + 4 * align16(128) + 0 = 96 + 512 = 608
    # x_o = 4e-6 + 608/6.08e8 = 5e-6; ZVC swap-out is a K-step pipeline: T_out = 5e-6 + 1e-6/4 = 5.25e-6
    # x_i = 1e-6 + 608/3.04e8 = 3e-6; T_in = 8e-6 + 3e-6/G
    assert r["size"][ZVC - 1] == 608
    assert r["t_codec"][ZVC - 1] == pytest.approx(t_zvc, rel=1e-9)
    # T' = (4e-6 + 16384/6.08e8) + (1e-6 + 16384/3.04e8)
    assert r["t_prime"] == pytest.approx(5e-6 + 16384 / 6.08e8 + 16384 / 3.04e8, rel=1e-12)


def test_multi_pass_codecs_swap_out_is_codec_time_then_transfer():
    """RLE / CSR / LZ4 place a frame only after every frame is counted / parsed (R22),
    so their pipelined T_out is t_c + x_o, not the K-step overlap ZVC gets."""
    b = np.zeros((4, 2, 6, 3))
    b[:, 0, 5, 0] = 2e-6
    b[:, 1, 5, 0] = 1e-6
    cal = O.make_calib(alpha_d2h=4e-6, bw_d2h=6.08e8, alpha_h2d=1e-6, bw_h2d=3.04e8, beta=b, mode=0,
                       frame_elems=1024)
    r = O.select(4096, O.F32, (4096, 1, 0, 4096, 4095), 0.0, 0.0, cal)
    # RLE: r = 1 + (K - 1) = 4 runs: 96 + 4 x 16 + align16(16) + align16(16) = 192 B
    assert r["size"][RLE - 1] == 192
    # T_out = 2e-6 + (4e-6 + 192/6.08e8); T_in (one step) = max(1e-6, x_i) + min(...) = 1e-6 + 1e-6 + 192/3.04e8
    assert r["t_codec"][RLE - 1] == pytest.approx(8e-6 + 192 / 6.08e8 + 192 / 3.04e8, rel=1e-12)
    # ZVC with the same times overlaps its 4 frames: T_out = max(2e-6, 5e-6) + 2e-6/4 = 5.5e-6
    assert r["t_codec"][ZVC - 1] == pytest.approx(5.5e-6 + 1e-6 + 3e-6, rel=1e-12)


# ------------------------------------------------------------------ paper mode, Eq. 2 with codec times
def test_paper_mode_eq2_with_codec_times_and_alpha_ignored():
    b = np.zeros((4, 2, 6, 3))
    b[:, 0, 3, 0] = 3e-6      # Time_c, band 3 (s = 0.6)
    b[:, 1, 3, 0] = 4e-6      # Time_dc
    # alpha is set but paper mode uses alpha = 0 (R10/R11: Eq. 2-4 have no latency term)
    cal = O.make_calib(alpha_d2h=1e-3, bw_d2h=1.6e8, alpha_h2d=1e-3, bw_h2d=8e7, beta=b, mode=1)
    r = O.select(1000, O.F32, (600, 1, 2, 1000, 999), 2e-6, 5e-5, cal)
    # size = S (1 - s) = 4000 * 0.4 = 1600 for every codec (Eq. 3-4)
    assert r["size"] == pytest.approx([1600.0] * 4, rel=1e-15)
    # T = 3e-6 + 4e-6 + max(1600/1.6e8 - 2e-6, 0) + max(1600/8e7 - 5e-5, 0) = 7e-6 + 8e-6 + 0
    assert r["t_codec"] == pytest.approx([1.5e-5] * 4, rel=1e-12)
    # Eq. 1: T' = max(4000/1.6e8 - 2e-6, 0) + max(4000/8e7 - 5e-5, 0) = 2.3e-5 + 0
    assert r["t_prime"] == pytest.approx(2.3e-5, rel=1e-12)
    assert r["codec"] == ZVC  # four-way tie -> lowest id (R12); 1.5e-5 < 2.3e-5 (strict, R13)
    # a cheaper RLE wins the argmin: T(RLE) = 1e-6 + 4e-6 + 8e-6
    b[RLE - 1, 0, 3, 0] = 1e-6
    cal = O.make_calib(alpha_d2h=1e-3, bw_d2h=1.6e8, alpha_h2d=1e-3, bw_h2d=8e7, beta=b, mode=1)
    r = O.select(1000, O.F32, (600, 1, 2, 1000, 999), 2e-6, 5e-5, cal)
    assert r["codec"] == RLE and r["t_pred"] == pytest.approx(1.3e-5, rel=1e-12)
    # codec time alone can cancel the gain: Time_c = 2e-5 gives T = 2e-5 + 4e-6 + 8e-6 = 3.2e-5 > T'
    b[:, 0, 3, 0] = 2e-5
    cal = O.make_calib(bw_d2h=1.6e8, bw_h2d=8e7, beta=b, mode=1)
    r = O.select(1000, O.F32, (600, 1, 2, 1000, 999), 2e-6, 5e-5, cal)
    assert r["t_codec"] == pytest.approx([3.2e-5] * 4, rel=1e-12) and r["codec"] == O.NONE


# ------------------------------------------------------------------ orc_max_size
def _liblz4_bound():
    import ctypes
    try:
        L = ctypes.CDLL("liblz4.so.1")
    except OSError:
        pytest.skip("liblz4.so.1 not available")
    L.LZ4_compressBound.argtypes = [ctypes.c_int]
    return L.LZ4_compressBound


@pytest.mark.parametrize("n,dtype,F,B", [(70000, O.F32, 1 << 22, 65536), (70000, O.F16, 1 << 22, 65536),
                                         (5000, O.F32, 2048, 1024), (300001, O.F32, 1 << 16, 65536)])
def test_lz4_max_size_is_liblz4_compress_bound_per_block(n, dtype, F, B):
    bound = _liblz4_bound()
    w = 4 if dtype == O.F32 else 2
    K = -(-n // F)
    a16 = lambda v: (v + 15) // 16 * 16  # noqa: E731
    total = a16(64 + 8 * K)
    for k in range(K):
        nbytes = min(F, n - k * F) * w
        lens = [min(B, nbytes - b) for b in range(0, nbytes, B)]
        total += a16(4 * len(lens)) + a16(sum(bound(L) for L in lens))
    assert O.max_size(LZ4, dtype, n, F, B) == total


@pytest.mark.parametrize("codec", [O.NONE, ZVC, RLE, CSR])
def test_max_size_is_reached_by_the_worst_case_input(codec):
    """Dense, all-distinct data is the worst case of every exact format: ZVC/CSR store every
    element, RLE makes a run per element, so the real container equals the bound exactly."""
    n, F = 5000, 2048
    x = (np.arange(n, dtype=np.uint32) + 1)  # no zeros, every neighbour differs
    assert len(O.compress(x, codec, O.F32, F=F)) == O.max_size(codec, O.F32, n, F)
