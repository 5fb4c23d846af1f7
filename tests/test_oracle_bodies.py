"""Pins for the oracle's task bodies (CPU only).

Each test checks oracle/ against something other than itself: values from
external standards (golden files, cited), closed forms, mathematical invariants,
library routines in float64 (numpy / scipy / `cryptography`) within the
textbook fp32 error bound.  See DESIGN.md "Oracle pins".
"""
import math

import numpy as np
import pytest

from conftest import golden_facts, read_golden
from paper_conf_ppopp_yehsser17_b200 import inputs

U = 2.0 ** -24            # unit roundoff of fp32


def gamma(n):
    return n * U / (1 - n * U)


# ------------------------------------------------------------------ Mandelbrot
@pytest.fixture(scope="module")
def mb_image(orc):
    img = np.zeros((2048, 2048), np.uint16)
    for ty in range(32):
        for tx in range(32):
            img[ty * 64:(ty + 1) * 64, tx * 64:(tx + 1) * 64] = orc.mandelbrot_tile(tx, ty)
    return img


def test_mb_golden_pixels(mb_image):
    for gx, gy, n in read_golden("mandelbrot_pins.txt"):
        assert mb_image[int(gy), int(gx)] == int(n), (gx, gy)


def test_mb_whole_config_facts(mb_image):
    f = golden_facts("mandelbrot_pins.txt")
    assert int(mb_image.astype(np.int64).sum()) == int(f["sum"])
    tiles = mb_image.reshape(32, 64, 32, 64).transpose(0, 2, 1, 3).reshape(1024, 4096).astype(np.int64)
    sums = tiles.sum(1)
    assert int((tiles == 256).all(1).sum()) == int(f["saturated_tiles"])
    assert sums.min() == f["tile_sum_min"] and sums.max() == f["tile_sum_max"]
    assert float(np.median(sums)) == f["tile_sum_median"]


def test_mb_conjugate_symmetry(mb_image):
    # RN is sign-symmetric, so count(c) == count(conj(c)) exactly; ci(2048-gy) = -ci(gy)
    assert np.array_equal(mb_image[1:1024, :], mb_image[2047:1024:-1, :])


def _mb_point(orc, cr, ci, maxit=256):
    return int(orc.mandelbrot_tile(0, 0, x0=cr, y0=ci, dx=1.0 / 1024, maxit=maxit)[0, 0])


def test_mb_closed_forms(orc):
    # exactly representable real orbits, counted by hand:
    # c=1: 0 -> 1 -> 2 -> 5 : |2|^2 = 4 is not > 4, |5|^2 > 4 -> n = 3
    assert _mb_point(orc, 1.0, 0.0) == 3
    # c=2: 0 -> 2 -> 6 : |2|^2 = 4 not > 4 -> n = 2
    assert _mb_point(orc, 2.0, 0.0) == 2
    # |c| > 2 escapes right after the first step: n = 1
    assert _mb_point(orc, 2.5, 0.0) == 1
    assert _mb_point(orc, 0.0, -3.0) == 1
    # c = 0 and c = -1 (period-2 cycle 0,-1,0,-1) never escape
    assert _mb_point(orc, 0.0, 0.0) == 256
    assert _mb_point(orc, -1.0, 0.0) == 256
    # c = -2: orbit -2, 2, 2, ... has |z|^2 = 4 exactly: strict '>' keeps it (256); '>=' would give 2
    assert _mb_point(orc, -2.0, 0.0) == 256
    # maxit is honoured
    assert _mb_point(orc, 0.0, 0.0, maxit=17) == 17


def test_mb_set_membership_invariants(orc, mb_image):
    # points well inside the main cardioid / period-2 bulb never escape;
    # points with |c| > 2 escape at n = 1.
    g = np.arange(2048)
    cr = (-2.0 + g * (3.0 / 2048))[None, :]
    ci = (-1.5 + g * (3.0 / 2048))[:, None]
    c = cr + 1j * ci
    card = np.abs(1 - np.sqrt(1 - 4 * c)) < 0.95          # interior of main cardioid (margin)
    bulb = np.abs(c + 1) < 0.24
    assert (mb_image[card | bulb] == 256).all()
    assert (mb_image[np.abs(c) > 2.0001] == 1).all()


# ------------------------------------------------------------------ 3DES
def test_tdes_known_answers(orc):
    for key, pt, ct in read_golden("tdes_kat.txt"):
        key, pt = bytes.fromhex(key), bytes.fromhex(pt)
        got = orc.tdes_ecb(pt, key)
        assert got.tobytes().hex() == ct.lower()
        assert orc.tdes_ecb(got.tobytes(), key, decrypt=True).tobytes() == pt


def test_des_single_block_kat(orc):
    # FIPS 46 worked example, single DES
    assert orc.des_block(0x0123456789ABCDEF, bytes.fromhex("133457799BBCDFF1")) == 0x85E813540F0AB405
    assert orc.des_block(0x85E813540F0AB405, bytes.fromhex("133457799BBCDFF1"), decrypt=True) == 0x0123456789ABCDEF


def test_tdes_packets_vs_library(orc):
    from cryptography.hazmat.decrepit.ciphers.algorithms import TripleDES
    from cryptography.hazmat.primitives.ciphers import Cipher, modes
    pk = inputs.tdes_packets(6)
    for i in range(len(pk)):
        enc = Cipher(TripleDES(inputs.TDES_KEYS), modes.ECB()).encryptor()
        ref = enc.update(pk[i].tobytes()) + enc.finalize()
        assert orc.tdes_ecb(pk[i], inputs.TDES_KEYS).tobytes() == ref
    # packet 0 carries the SP 800-67 example in bytes [0,24)
    assert orc.tdes_ecb(pk[0], inputs.TDES_KEYS)[:24].tobytes().hex() == read_golden("tdes_kat.txt")[0][2]


def test_tdes_round_trip_random_keys(orc):
    rng = np.random.default_rng(7)
    for _ in range(4):
        key = rng.integers(0, 256, 24, dtype=np.uint8).tobytes()
        data = rng.integers(0, 256, 512, dtype=np.uint8)
        ct = orc.tdes_ecb(data, key)
        assert orc.tdes_ecb(ct, key, decrypt=True).tobytes() == data.tobytes()


# ------------------------------------------------------------------ MM
def test_mm_identity(orc):
    A, B = inputs.mm_inputs(2)
    assert np.array_equal(orc.mm32(A[0], np.eye(32, dtype=np.float32)), A[0])
    assert np.array_equal(orc.mm32(np.eye(32, dtype=np.float32), B[1]), B[1])


def test_mm_integer_exact(orc):
    A, B = inputs.mm_inputs(4, integer=True)
    for i in range(4):
        ref = A[i].astype(np.int64) @ B[i].astype(np.int64)
        assert np.array_equal(orc.mm32(A[i], B[i]).astype(np.int64), ref)


def test_mm_within_error_bound(orc):
    A, B = inputs.mm_inputs(8)
    for i in range(8):
        got = orc.mm32(A[i], B[i]).astype(np.float64)
        a, b = A[i].astype(np.float64), B[i].astype(np.float64)
        ref = a @ b
        bound = gamma(32) * (np.abs(a) @ np.abs(b))
        assert (np.abs(got - ref) <= bound).all()
    # a transposed operand is caught
    assert not np.allclose(orc.mm32(A[0], B[0]), (A[0].astype(np.float64) @ B[0].T), atol=1e-3)


def test_mm64_pins(orc):
    """Table 4's 64x64 size: identity both sides, integer inputs exact (every partial sum
    is an integer below 2^24), random inputs within the fma chain's bound gamma_64 |A||B|,
    a transposed operand and a dropped last k term are caught."""
    A, B = inputs.mm64_inputs(2)
    I64 = np.eye(64, dtype=np.float32)
    assert np.array_equal(orc.mm64(A[0], I64), A[0])
    assert np.array_equal(orc.mm64(I64, B[1]), B[1])
    Ai, Bi = inputs.mm64_inputs(3, integer=True)
    for i in range(3):
        assert np.array_equal(orc.mm64(Ai[i], Bi[i]).astype(np.int64), Ai[i].astype(np.int64) @ Bi[i].astype(np.int64))
    for i in range(2):
        a, b = A[i].astype(np.float64), B[i].astype(np.float64)
        got = orc.mm64(A[i], B[i]).astype(np.float64)
        assert (np.abs(got - a @ b) <= gamma(64) * (np.abs(a) @ np.abs(b))).all()
    assert not np.allclose(orc.mm64(A[0], B[0]), A[0].astype(np.float64) @ B[0].T, atol=1e-3)
    got = orc.mm64(Ai[0], Bi[0]).astype(np.int64)
    assert not np.array_equal(got, Ai[0][:, :63].astype(np.int64) @ Bi[0][:63].astype(np.int64))


def test_mm_exact_variant(orc):
    """mm32_exact (NEXT-4's definition): integer inputs exact; random inputs
    equal the exactly rounded product (exact rational sum via fractions,
    rounded once to fp32; 32 products of 24-bit values fit a double
    exactly, their sum may not); a transposed operand is caught."""
    from fractions import Fraction
    A, B = inputs.mm_inputs(3, integer=True)
    for i in range(3):
        ref = A[i].astype(np.int64) @ B[i].astype(np.int64)
        assert np.array_equal(orc.mm32_exact(A[i], B[i]).astype(np.int64), ref)
    A, B = inputs.mm_inputs(2)
    got = orc.mm32_exact(A[0], B[0])
    for i, j in [(0, 0), (3, 17), (31, 31), (12, 5), (20, 30)]:
        exact = sum(Fraction(float(A[0][i, k])) * Fraction(float(B[0][k, j])) for k in range(32))
        near = np.float32(float(exact))            # exact -> double -> fp32: one ulp of slack for double rounding
        assert abs(float(got[i, j]) - float(exact)) <= abs(float(near) - float(exact)) + 1e-12, (i, j)
    assert np.array_equal(orc.mm32_exact(A[1], np.eye(32, dtype=np.float32)), A[1])
    assert not np.allclose(got, A[0].astype(np.float64) @ B[0].T, atol=1e-3)


# ------------------------------------------------------------------ FB
def _fb_fp64(r, H, F):
    r, H, F = (np.asarray(v, np.float64) for v in (r, H, F))
    vh = np.convolve(r, H)[:2048]
    vu = np.zeros(2048)
    vu[::8] = vh[::8]
    return np.convolve(vu, F)[:2048], vh, vu


def test_fb_impulse_closed_form(orc):
    _, H, F = inputs.fb_inputs(1)
    r = np.zeros(2048, np.float32); r[0] = 1.0
    y = orc.filterbank(r, H[0], F[0])
    # y[j] = sum_{m: 0 <= 8m <= j, j-8m < 32, 8m < 32} H[8m] F[j-8m]  (each term exact, one rounding per add)
    for j in range(2048):
        terms = [np.float32(H[0][8 * m]) * np.float32(F[0][j - 8 * m])
                 for m in range(4) if 8 * m <= j and j - 8 * m < 32]
        ref = math.fsum(float(t) for t in terms)
        assert abs(float(y[j]) - ref) <= 4 * U * sum(abs(float(t)) for t in terms), j
    assert (y[64:] == 0).all()


def test_fb_shift_invariance(orc):
    _, H, F = inputs.fb_inputs(1)
    r0 = np.zeros(2048, np.float32); r0[0] = 1.0
    y0 = orc.filterbank(r0, H[0], F[0])
    for s in (8, 16, 800):   # shifts by multiples of N_samp commute with the down/up-sampling
        rs = np.zeros(2048, np.float32); rs[s] = 1.0
        ys = orc.filterbank(rs, H[0], F[0])
        assert np.array_equal(ys[s:], y0[:2048 - s]) and (ys[:s] == 0).all()


def test_fb_vs_fp64(orc):
    r, H, F = inputs.fb_inputs(3)
    for i in range(3):
        got = orc.filterbank(r[i], H[i], F[i]).astype(np.float64)
        ref, vh, vu = _fb_fp64(r[i], H[i], F[i])
        # error: the VH stage (gamma_32 * |H|*|r|) propagates through F, plus the F stage itself
        vh_abs = np.convolve(np.abs(r[i]).astype(np.float64), np.abs(H[i]).astype(np.float64))[:2048]
        vu_abs = np.zeros(2048); vu_abs[::8] = vh_abs[::8]
        bound = (gamma(32) * 2 + gamma(32) ** 2) * np.convolve(vu_abs, np.abs(F[i]).astype(np.float64))[:2048]
        assert (np.abs(got - ref) <= bound + 1e-30).all()


# ------------------------------------------------------------------ BF
def test_bf_delta_onehot(orc):
    x, h, w = inputs.bf_inputs(1)
    h = np.zeros_like(h); h[0, :, 0, 0] = 1.0            # h[c] = delta
    for c in range(4):
        wc = np.zeros_like(w); wc[0, :, c, 0] = 1.0       # every beam selects channel c
        out = orc.beamformer(x[0], h[0], wc[0])
        xr, xi = x[0, c, :, 0], x[0, c, :, 1]
        ref = (xr.astype(np.float64) ** 2 + xi.astype(np.float64) ** 2)
        assert np.allclose(out, ref[None, :], rtol=3 * U, atol=0)


def test_bf_vs_complex128(orc):
    x, h, w = inputs.bf_inputs(3)
    for i in range(3):
        xc = x[i, ..., 0].astype(np.float64) + 1j * x[i, ..., 1]
        hc = h[i, ..., 0].astype(np.float64) + 1j * h[i, ..., 1]
        wc = w[i, ..., 0].astype(np.float64) + 1j * w[i, ..., 1]
        v = np.stack([np.convolve(xc[c], hc[c])[:512] for c in range(4)])
        y = wc @ v
        ref = np.abs(y) ** 2
        got = orc.beamformer(x[i], h[i], w[i]).astype(np.float64)
        # |y| bound: sum |w||h||x| ; relative error of |y|^2 ~ 2*err(|y|)/|y| : use absolute bound
        va = np.stack([np.convolve(np.abs(xc[c]), np.abs(hc[c]))[:512] for c in range(4)])
        ya = np.abs(wc) @ va
        bound = 2 * ya * (gamma(64) * 2 * ya) + gamma(3) * ya ** 2
        assert (np.abs(got - ref) <= bound).all()
        assert np.max(np.abs(got - ref) / np.maximum(ref, 1e-3)) < 1e-4


# ------------------------------------------------------------------ CONV
def test_conv_delta(orc):
    _, krow, kcol = inputs.conv_inputs(1)
    img = np.zeros((128, 128), np.float32)
    y0, x0 = 60, 70
    img[y0, x0] = 1.0
    out = orc.conv(img, krow[0], kcol[0])
    ref = np.zeros((128, 128), np.float32)
    for a in range(-8, 9):
        for b in range(-8, 9):
            # out[y0+a][x0+b] = kcol[8+a]*krow[8+b] (one nonzero term, rounded once)
            ref[y0 + a, x0 + b] = np.float32(kcol[0][8 + a]) * np.float32(krow[0][8 + b])
    assert np.array_equal(out, ref)


def test_conv_constant_interior(orc):
    _, krow, kcol = inputs.conv_inputs(1)
    img = np.full((128, 128), 0.75, np.float32)
    out = orc.conv(img, krow[0], kcol[0]).astype(np.float64)
    ref = 0.75 * krow[0].astype(np.float64).sum() * kcol[0].astype(np.float64).sum()
    inner = out[8:120, 8:120]
    bound = gamma(17) * 2 * 0.75 * np.abs(krow[0]).sum() * np.abs(kcol[0]).sum()
    assert np.all(np.abs(inner - ref) <= bound)


def test_conv_vs_scipy(orc):
    from scipy.ndimage import convolve1d
    img, krow, kcol = inputs.conv_inputs(2)
    for i in range(2):
        a = img[i].astype(np.float64)
        # convolve1d(weights=k) computes sum_j in[x + 8 - j] * k[j]  (true convolution, centred)
        tmp = convolve1d(a, krow[i].astype(np.float64), axis=1, mode="constant")
        ref = convolve1d(tmp, kcol[i].astype(np.float64), axis=0, mode="constant")
        tabs = convolve1d(np.abs(a), np.abs(krow[i]).astype(np.float64), axis=1, mode="constant")
        babs = convolve1d(tabs, np.abs(kcol[i]).astype(np.float64), axis=0, mode="constant")
        got = orc.conv(img[i], krow[i], kcol[i]).astype(np.float64)
        assert np.all(np.abs(got - ref) <= (2 * gamma(17) + gamma(17) ** 2) * babs)


# ------------------------------------------------------------------ DCT
def test_dct_constant_block(orc):
    C = inputs.dct_coef()
    img = np.full((128, 128), 3.0, np.float32)
    out = orc.dct(img, C).astype(np.float64)
    blocks = out.reshape(16, 8, 16, 8).transpose(0, 2, 1, 3)
    assert np.allclose(blocks[:, :, 0, 0], 24.0, rtol=1e-6)
    ac = blocks.copy(); ac[:, :, 0, 0] = 0
    assert np.abs(ac).max() < 1e-5


def test_dct_vs_scipy_and_parseval(orc):
    from scipy.fft import dctn
    C = inputs.dct_coef()
    img = inputs.dct_inputs(2)
    for i in range(2):
        got = orc.dct(img[i], C).astype(np.float64)
        b_in = img[i].astype(np.float64).reshape(16, 8, 16, 8).transpose(0, 2, 1, 3)
        ref = dctn(b_in, type=2, norm="ortho", axes=(2, 3))
        g = got.reshape(16, 8, 16, 8).transpose(0, 2, 1, 3)
        # C rounded to fp32 (rel err U per entry) + two 8-term dot products
        absb = np.abs(C.astype(np.float64)) @ np.abs(b_in) @ np.abs(C.astype(np.float64)).T
        assert np.all(np.abs(g - ref) <= (2 * gamma(8) + 4 * U) * absb + 1e-12)
        # Parseval (orthonormal transform): energies agree to fp32 accuracy
        assert np.allclose((g ** 2).sum((2, 3)), (b_in ** 2).sum((2, 3)), rtol=1e-5)


def test_dct_coef_is_orthonormal():
    C = inputs.dct_coef().astype(np.float64)
    assert np.allclose(C @ C.T, np.eye(8), atol=1e-6)


# ------------------------------------------------------------------ occupancy
def test_occupancy_paper_examples(orc):
    # one 256-thread task on 24 SMMs = 0.52 %, 32 HyperQ tasks = 16.67 %
    assert round(orc.occupancy_pct(8, 24), 2) == 0.52
    assert round(orc.occupancy_pct(8 * 32, 24), 2) == 16.67


# ---------------------------------------------------------------- NEXT-1 / config 5 input recipes (host logic)
def test_tdes_var_sizes_log_uniform():
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    s = I.tdes_var_sizes(32768)
    assert s.min() >= 2048 and s.max() <= 65536 and np.all(s % 8 == 0)
    # log-uniform: log2(size/2048) is uniform on [0, 5): each octave holds ~1/5 of the packets
    oct_ = np.floor(np.log2(s / 2048)).astype(int)
    frac = np.bincount(oct_, minlength=5)[:5] / len(s)
    assert np.all(np.abs(frac - 0.2) < 0.02), frac
    assert abs(s.mean() - (65536 - 2048) / np.log(32)) / s.mean() < 0.03   # E[size] of log-uniform


def test_tdes_var_packets_are_the_tdes_streams():
    """Equal sizes reproduce tdes_packets(); a ragged packet is the prefix of
    its task's stream; the oracle encrypts it like the library does."""
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    flat, off = I.tdes_var_packets(np.array([4096, 2048, 16], np.int64))
    full = I.tdes_packets(3, 4096)
    assert np.array_equal(flat[off[0]:off[1]], full[0])
    assert np.array_equal(flat[off[1]:off[2]], full[1, :2048])
    assert np.array_equal(flat[off[2]:off[3]], full[2, :16])


def test_schedules_mpe_and_c5():
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    k = I.mpe_schedule(32768)
    assert np.array_equal(np.bincount(k), [8192] * 4)           # 8K of each
    assert not np.array_equal(k[:8], np.arange(8) % 4)          # shuffled
    kinds, thr, shm = I.c5_schedule(1_000_000)
    c = np.bincount(kinds, minlength=7)
    assert np.all(np.abs(c / 1e6 - 1 / 7) < 0.002), c           # seeded uniform draw over 7 bodies
    assert set(np.unique(thr)) == set(I.MIX_THREADS)
    assert set(np.unique(shm // 1024)) == set(I.MIX_SHMEM_KB)
    k2 = I.c5_schedule(1000)[0]
    assert np.array_equal(k2, kinds[:1000])                     # prefix-stable: shards agree with the whole


# ------------------------------------------------------------------ fma / order pins
# Error bounds cannot tell fmaf from mul+add, nor one summation order from another.
# These closed forms can: with P = 1 + 2^-12 and Q = 1 + 2^-11 (both fp32),
# P*P = 1 + 2^-11 + 2^-24 exactly, whose fp32 rounding is Q (a tie, to even).
# So the step "acc = -Q; acc = fmaf(P, P, acc)" gives exactly 2^-24 when it is
# fused and taken in the defined (ascending) order; rounding the product first
# (mul+add) or taking the P*P term first (descending order) gives 0.  Each body
# gets one such step at a place its definition fixes.
P32 = 1.0 + 2.0 ** -12
Q32 = 1.0 + 2.0 ** -11


def test_fma_order_pin_mm(orc):
    """C[i][j] = fma chain over k ascending (DESIGN.md MM): A[:,0] = 1, B[0,:] = -Q,
    A[:,1] = B[1,:] = P -> every C[i][j] = 2^-24 exactly."""
    for n, f in ((32, orc.mm32), (64, orc.mm64)):
        A = np.zeros((n, n), np.float32)
        B = np.zeros((n, n), np.float32)
        A[:, 0], B[0, :] = 1.0, -Q32
        A[:, 1], B[1, :] = P32, P32
        C = f(A, B)
        assert (C == np.float32(2.0 ** -24)).all(), (n, np.unique(C))


def test_fma_order_pin_filterbank(orc):
    """VH[8] = fma chain k = 0..8 of H[k] r[8-k] with H[0] r[8] = -Q, H[8] r[0] = P*P -> 2^-24;
    with F = delta, y[8] = VU[8] = VD[1] = VH[8] and y[0] = VH[0] = P."""
    r = np.zeros(2048, np.float32)
    H = np.zeros(32, np.float32)
    F = np.zeros(32, np.float32)
    r[0], r[8] = P32, -Q32
    H[0], H[8] = 1.0, P32
    F[0] = 1.0
    y = orc.filterbank(r, H, F)
    assert y[8] == np.float32(2.0 ** -24) and y[0] == np.float32(P32)


def test_fma_order_pin_beamformer(orc):
    """out = fmaf(y.re, y.re, y.im*y.im) with y = (P, 2^-12): fused = RN(1 + 2^-11 + 2^-23)
    = 1 + 2^-11 + 2^-23; mul+add (or the other operand fused) = Q."""
    x = np.zeros((4, 512, 2), np.float32)
    h = np.zeros((4, 16, 2), np.float32)
    w = np.zeros((4, 4, 2), np.float32)
    x[0, 0] = (P32, 2.0 ** -12)
    h[0, 0] = (1.0, 0.0)
    w[0, 0] = (1.0, 0.0)
    out = orc.beamformer(x, h, w)
    assert out[0, 0] == np.float32(1.0 + 2.0 ** -11 + 2.0 ** -23)
    assert (out[1:] == 0).all()


def test_fma_order_pin_conv(orc):
    """Row pass d ascending: img[64][64] krow[8] = -Q, then img[64][65] krow[7] = P*P ->
    tmp[64][64] = 2^-24; kcol = delta -> out[64][64] = 2^-24."""
    img = np.zeros((128, 128), np.float32)
    krow = np.zeros(17, np.float32)
    kcol = np.zeros(17, np.float32)
    img[64, 64], img[64, 65] = 1.0, P32
    krow[8], krow[7] = -Q32, P32
    kcol[8] = 1.0
    out = orc.conv(img, krow, kcol)
    assert out[64, 64] == np.float32(2.0 ** -24)


def test_fma_order_pin_dct(orc):
    """T[0][0] = fma chain over x ascending: C[0][0] X[0][0] = -Q, then C[0][1] X[1][0] = P*P ->
    2^-24; Y[0][0] = T[0][0] C[0][0] = -(2^-24 + 2^-35) (exact)."""
    img = np.zeros((128, 128), np.float32)
    coef = np.zeros((8, 8), np.float32)
    img[0, 0], img[1, 0] = 1.0, P32
    coef[0, 0], coef[0, 1] = -Q32, P32
    out = orc.dct(img, coef)
    assert out[0, 0] == np.float32(-(2.0 ** -24 + 2.0 ** -35))
    assert (out[8:, :] == 0).all() and (out[:, 8:] == 0).all()


# ------------------------------------------------------------------ Mandelbrot pin provenance
def test_mb_golden_file_regenerates():
    """tests/golden/mandelbrot_pins.txt is exactly what scripts/gen_mandelbrot_pins.py (an
    independent numpy float32 emulation, no oracle code) writes; and a contracted (fma)
    evaluation of the same iteration changes the whole-config sum, so that pin catches it."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "gen_mb", os.path.join(os.path.dirname(__file__), "..", "scripts", "gen_mandelbrot_pins.py"))
    gen = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(gen)
    counts = gen.iteration_counts()
    with open(gen.GOLDEN) as f:
        assert f.read() == gen.render(counts)
    fused = gen.iteration_counts(fused=True)
    assert int(fused.sum(dtype=np.int64)) != int(counts.sum(dtype=np.int64))


# ------------------------------------------------------------------ the timed oracle build
def test_fast_build_outputs_equal_parity_build():
    """bench.py times the oracle built -O3 -march=native -ffp-contract=off; with
    contraction still off its outputs must equal the parity build's, body by body."""
    import oracle as O
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    F = O.lib(fast=True)
    assert np.array_equal(O.mandelbrot_tile(24, 16), O.mandelbrot_tile(24, 16, L=F))
    pk = I.tdes_packets(2, 4096, 0)
    assert np.array_equal(O.tdes_ecb(pk[1], I.TDES_KEYS), O.tdes_ecb(pk[1], I.TDES_KEYS, L=F))
    A, B = I.mm_inputs(2)
    assert np.array_equal(O.mm32(A[1], B[1]), O.mm32(A[1], B[1], L=F))
    A, B = I.mm64_inputs(1)
    assert np.array_equal(O.mm64(A[0], B[0]), O.mm64(A[0], B[0], L=F))
    r, H, Fi = I.fb_inputs(1)
    assert np.array_equal(O.filterbank(r[0], H[0], Fi[0]), O.filterbank(r[0], H[0], Fi[0], L=F))
    x, h, w = I.bf_inputs(1)
    assert np.array_equal(O.beamformer(x[0], h[0], w[0]), O.beamformer(x[0], h[0], w[0], L=F))
    img, kr, kc = I.conv_inputs(1)
    assert np.array_equal(O.conv(img[0], kr[0], kc[0]), O.conv(img[0], kr[0], kc[0], L=F))
    im = I.dct_inputs(1)
    assert np.array_equal(O.dct(im[0], I.dct_coef()), O.dct(im[0], I.dct_coef(), L=F))
