"""Pins of the CPU oracle against things other than itself (task rule 3).

Each test names the PAPER.md passage / DESIGN.md reading it pins.  Sources of
truth: closed forms (ramps, constants, impulses), brute force on tiny inputs,
textbook routines (numpy/scipy), statements of the paper (L142), and an
independent float64 evaluation (tests/exact_ref.py).
"""
import itertools

import numpy as np
import pytest
from scipy import ndimage, signal

import exact_ref
import oracle
import synth

RNG = np.random.default_rng(20150901)
SIZES = [(8, 8), (12, 8), (8, 12), (16, 24), (32, 20), (48, 36), (64, 64)]


def rand_img(W, H, lo=0, hi=256):
    return RNG.integers(lo, hi, size=(H, W), dtype=np.int64).astype(np.uint8)


def ramp(W, H, a, b, c):
    """O[r][c] = a + b*col + c*row (no clamping: caller keeps it in range)."""
    rr, cc = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    v = a + b * cc + c * rr
    assert v.min() >= 0 and v.max() <= 255
    return v.astype(np.uint8)


# --------------------------------------------------------------------------
# Downscale (L130, L136, L218; R2)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", SIZES)
def test_downscale_bruteforce_block_mean(W, H):
    O = rand_img(W, H)
    D = oracle.downscale(O)
    for i in range(H // 4):
        for j in range(W // 4):
            assert D[i, j] == np.mean(O[4 * i:4 * i + 4, 4 * j:4 * j + 4].astype(np.float64))


def test_downscale_ramp_closed_form():
    # f = a + b x + c y  =>  D[i][j] = f(4j+1.5, 4i+1.5)
    O = ramp(64, 40, 7, 2, 3)
    D = oracle.downscale(O)
    i, j = np.meshgrid(np.arange(10), np.arange(16), indexing="ij")
    np.testing.assert_array_equal(D, 7 + 2 * (4 * j + 1.5) + 3 * (4 * i + 1.5))


# --------------------------------------------------------------------------
# Upscale: body (L146, Fig. 4-5; R3) and border (L140-L142; R4, R5)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", SIZES)
def test_upscale_body_is_halfpixel_bilinear(W, H):
    O = rand_img(W, H)
    U = oracle.upscale(oracle.downscale(O), W, H)
    ref = exact_ref.body_bilinear(exact_ref.downscale(O), H, W)
    np.testing.assert_array_equal(U[2:H - 2, 2:W - 2].astype(np.float64), ref)


@pytest.mark.parametrize("W,H", SIZES)
def test_upscale_border_final_state_rule(W, H):
    O = rand_img(W, H)
    U = oracle.upscale(oracle.downscale(O), W, H)
    ref = exact_ref.border_rule(exact_ref.downscale(O), H, W)
    ring = ~np.isnan(ref)
    np.testing.assert_array_equal(U[ring].astype(np.float64), ref[ring])
    assert not np.isnan(U).any()  # every pixel is written by some step


@pytest.mark.parametrize("W,H", SIZES)
def test_upscale_L142_only_bottom_right_2x2_missing_after_vi(W, H):
    # L142: "After all the caculations above, the four elements of the bottom
    # right corner are still missing."
    D = oracle.downscale(rand_img(W, H))
    U6 = oracle.upscale_steps(D, W, H, 6)
    ring = np.zeros((H, W), bool)
    ring[:2, :] = ring[-2:, :] = ring[:, :2] = ring[:, -2:] = True
    missing = np.argwhere(np.isnan(U6) & ring)
    assert sorted(map(tuple, missing)) == [(H - 2, W - 2), (H - 2, W - 1), (H - 1, W - 2), (H - 1, W - 1)]
    # and the fill value is the third last element of the last column
    U7 = oracle.upscale_steps(D, W, H, 7)
    assert np.all(U7[H - 2:, W - 2:] == U6[H - 3, W - 1])


def test_upscale_affine_ramp_body_exact():
    # Bilinear reproduces affine functions: U == O on rows/cols 2..H-3.
    O = ramp(64, 48, 3, 2, 1)
    U = oracle.upscale(oracle.downscale(O), 64, 48)
    np.testing.assert_array_equal(U[2:-2, 2:-2], O[2:-2, 2:-2].astype(np.float32))


def test_upscale_border_ramp_offsets():
    # Ramp O = 3x + 2y, row 0: U - O = 7.5 on {0} u [2, W-4], 4.5 at 1 and W-3,
    # 1.5 at W-2, -1.5 at W-1 (hand-derived from L140-L142).
    W, H = 40, 24
    O = ramp(W, H, 0, 3, 2)
    U = oracle.upscale(oracle.downscale(O), W, H)
    d = U[0].astype(np.float64) - O[0]
    exp = np.full(W, 7.5)
    exp[1] = exp[W - 3] = 4.5
    exp[W - 2] = 1.5
    exp[W - 1] = -1.5
    np.testing.assert_array_equal(d, exp)


@pytest.mark.parametrize("c", [0, 1, 77, 128, 254, 255])
def test_upscale_constant(c):
    O = np.full((20, 28), c, np.uint8)
    U = oracle.upscale(oracle.downscale(O), 28, 20)
    assert np.all(U == c)


@pytest.mark.parametrize("W,H", SIZES)
def test_upscale_dyadic_exact(W, H):
    # D*16 and U*1024 are integers (< 2^18): the stages are exact in float.
    O = rand_img(W, H)
    D = oracle.downscale(O)
    U = oracle.upscale(D, W, H)
    assert np.all(np.mod(D.astype(np.float64) * 16, 1) == 0)
    n = U.astype(np.float64) * 1024
    assert np.all(np.mod(n, 1) == 0) and n.max() < 2 ** 18


@pytest.mark.parametrize("W,H", [(16, 24), (32, 20), (8, 12)])
def test_upscale_transpose_invariance(W, H):
    O = rand_img(W, H)
    U = oracle.upscale(oracle.downscale(O), W, H)
    Ut = oracle.upscale(oracle.downscale(O.T.copy()), H, W)
    np.testing.assert_array_equal(Ut, U.T)


# --------------------------------------------------------------------------
# pError (L148; R6)
# --------------------------------------------------------------------------
def test_perror_sign_and_exactness():
    O = rand_img(16, 16)
    U = oracle.upscale(oracle.downscale(O), 16, 16)
    E = oracle.perror(O, U)
    np.testing.assert_array_equal(E.astype(np.float64), O.astype(np.float64) - U.astype(np.float64))
    assert np.all(E + U == O)  # exact: U + (O - U) == O


# --------------------------------------------------------------------------
# Sobel (L158-L172; R7)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", SIZES)
def test_sobel_matches_scipy(W, H):
    O = rand_img(W, H)
    np.testing.assert_array_equal(oracle.sobel(O), exact_ref.sobel(O))


def test_sobel_constant_checker_zero():
    assert np.all(oracle.sobel(np.full((16, 16), 93, np.uint8)) == 0)
    ck = synth.image(24, 16, "checker", param=10)
    assert np.all(oracle.sobel(ck) == 0)  # 1-px checkerboard is in the Sobel null space


def test_sobel_ramp_and_frame():
    O = ramp(32, 24, 5, 3, 2)
    pE = oracle.sobel(O)
    assert np.all(pE[1:-1, 1:-1] == 8 * (3 + 2))
    assert np.all(pE[0] == 0) and np.all(pE[-1] == 0) and np.all(pE[:, 0] == 0) and np.all(pE[:, -1] == 0)
    O2 = ramp(32, 24, 200, -3, -2)
    assert np.all(oracle.sobel(O2)[1:-1, 1:-1] == 8 * (3 + 2))


def test_sobel_impulse_ring():
    v = 200
    O = np.zeros((16, 16), np.uint8)
    O[7, 8] = v
    pE = oracle.sobel(O)
    ring = [(7 + a, 8 + b) for a in (-1, 0, 1) for b in (-1, 0, 1) if (a, b) != (0, 0)]
    for p in ring:
        assert pE[p] == 2 * v
    assert pE[7, 8] == 0
    assert pE.sum() == 16 * v


def test_sobel_max_1530_bruteforce():
    best = 0
    Mx = np.array([[-1, 0, 1], [-2, 0, 2], [-1, 0, 1]])
    for bits in itertools.product([0, 255], repeat=9):
        win = np.array(bits).reshape(3, 3)
        gx = signal.correlate2d(win, Mx, mode="valid")[0, 0]
        gy = signal.correlate2d(win, Mx.T, mode="valid")[0, 0]
        best = max(best, abs(gx) + abs(gy))
        O = np.zeros((8, 8), np.uint8)
        O[2:5, 2:5] = win
        assert oracle.sobel(O)[3, 3] == abs(gx) + abs(gy)
    assert best == 1530


# --------------------------------------------------------------------------
# Reduction (L174, L284; R8)
# --------------------------------------------------------------------------
def test_reduce_matches_naive_double_sum():
    pE = RNG.integers(0, 1531, size=(300, 200)).astype(np.int32)
    S, mean = oracle.reduce(pE)
    assert S == int(np.sum(pE.astype(np.float64)))
    assert mean == S / (300 * 200)


def test_reduce_closed_forms():
    W, H = 40, 28
    S, _ = oracle.reduce(oracle.sobel(np.full((H, W), 9, np.uint8)))
    assert S == 0
    S, mean = oracle.reduce(oracle.sobel(ramp(W, H, 10, 2, 3)))
    assert S == 8 * (2 + 3) * (W - 2) * (H - 2)
    assert mean == S / (W * H)
    imp = synth.image(W, H, "impulse", seed=5, param=77)
    S, _ = oracle.reduce(oracle.sobel(imp))
    assert S == 16 * 77 * int((imp > 0).sum())


# --------------------------------------------------------------------------
# Strength (L178, L232; R9) -- the curve's shape is "parity unpinned"; these
# pin its special cases and its orientation (p/m, multiplied by A).
# --------------------------------------------------------------------------
def test_strength_special_cases():
    pE = np.arange(0, 1531, dtype=np.int32).reshape(1, -1)
    assert np.all(oracle.strength(pE, 37.25, 1.5, 0.0) == np.float32(1.5))  # gamma 0 (pow(0,0)=1)
    assert np.all(oracle.strength(pE, 37.25, 0.0, 0.7) == 0)  # A = 0
    # gamma = 1: A * p / m rounded once
    a1 = oracle.strength(pE, 40.0, 2.0, 1.0)
    np.testing.assert_array_equal(a1, (2.0 * pE / 40.0).astype(np.float32))
    # gamma = 0.5 on perfect squares of m: p = m k^2 -> A k exactly
    m = 4.0
    ks = np.arange(0, 19)
    p = (m * ks * ks).astype(np.int32).reshape(1, -1)
    np.testing.assert_array_equal(oracle.strength(p, m, 3.0, 0.5)[0], (3.0 * ks).astype(np.float32))
    # gamma = 2: (p/m)^2 with m = 2 -> p^2/4 exactly
    np.testing.assert_array_equal(oracle.strength(pE[:, :100], 2.0, 1.0, 2.0),
                                  ((pE[:, :100] / 2.0) ** 2).astype(np.float32))


def test_strength_mean_guard():
    # R8/R9: m = max(mean, 1): a mean below 1 behaves like 1
    pE = np.arange(0, 50, dtype=np.int32).reshape(1, -1)
    np.testing.assert_array_equal(oracle.strength(pE, 0.25, 1.0, 1.0), pE.astype(np.float32))
    np.testing.assert_array_equal(oracle.strength(pE, 0.0, 1.0, 1.0), pE.astype(np.float32))


# --------------------------------------------------------------------------
# Preliminary (L178; R10) and overshoot (L180-L212, Fig. 8; R11-R13)
# --------------------------------------------------------------------------
def test_preliminary_unit_strength_is_identity():
    O = rand_img(24, 16)
    U = oracle.upscale(oracle.downscale(O), 24, 16)
    E = oracle.perror(O, U)
    P = oracle.preliminary(np.ones_like(E), E, U)
    np.testing.assert_array_equal(P, O.astype(np.float32))


def test_preliminary_single_rounding():
    # fmaf rounds once: pick adj, E, U where a*E+U rounded twice differs.
    adj = np.array([[1.0 + 2.0 ** -23]], np.float32)
    E = np.array([[1.0 + 2.0 ** -23]], np.float32)
    U = np.array([[-1.0]], np.float32)
    P = oracle.preliminary(adj, E, U)
    # exact: (1+e)^2 - 1 = 2e + e^2, e = 2^-23  -> fma keeps the e^2 term
    assert P[0, 0] == np.float32(2.0 ** -22 + 2.0 ** -46)


def _window_minmax(O):
    o = O.astype(np.float32)
    return (ndimage.maximum_filter(o, size=3, mode="nearest"),
            ndimage.minimum_filter(o, size=3, mode="nearest"))


def test_overshoot_gain0_clamps_to_window():
    O = rand_img(24, 20)
    P = RNG.uniform(-80, 330, size=O.shape).astype(np.float32)
    pE = oracle.sobel(O)
    F = oracle.overshoot(O, P, pE, 50.0, 0.0, 2.0)
    mx, mn = _window_minmax(O)
    inner = np.s_[1:-1, 1:-1]
    np.testing.assert_array_equal(F[inner], np.clip(P, mn, mx)[inner])
    frame = np.ones(O.shape, bool)
    frame[inner] = False
    np.testing.assert_array_equal(F[frame], np.clip(P, 0, 255)[frame])


def test_overshoot_unit_osc_is_plain_clamp():
    # pE = 0 and G = 1 -> osc = 1 -> osc max = P -> Final = min(max(P,0),255)
    # (P on a 1/1024 grid so that P - max is exact in f32)
    O = rand_img(16, 16)
    P = (RNG.integers(-80 * 1024, 330 * 1024, size=O.shape) / 1024).astype(np.float32)
    F = oracle.overshoot(O, P, np.zeros(O.shape, np.int32), 10.0, 1.0, 2.0)
    np.testing.assert_array_equal(F, np.clip(P, 0, 255))


def test_overshoot_half_osc_branches():
    # G = 0.5, pE = 0 -> osc = 0.5: P > max -> (max + P)/2, P < min -> (min + P)/2
    O = np.full((8, 8), 100, np.uint8)
    O[3, 3] = 140  # window of (4,4) has max 140, min 100
    P = np.full((8, 8), 120.0, np.float32)
    P[4, 4] = 200.0
    P[4, 5] = 60.0
    P[4, 3] = 101.5
    F = oracle.overshoot(O, P, np.zeros((8, 8), np.int32), 10.0, 0.5, 2.0)
    assert F[4, 4] == (140 + 200) / 2  # above max
    assert F[4, 5] == (100 + 60) / 2   # below min
    assert F[4, 3] == np.float32(101.5)  # inside: unchanged
    # oscStrength decreases with edge strength (R11): larger pE -> closer to max
    F2 = oracle.overshoot(O, P, np.full((8, 8), 500, np.int32), 10.0, 0.5, 2.0)
    assert 140 <= F2[4, 4] < F[4, 4]


def test_output_round_half_even():
    F = np.array([[0.5, 1.5, 2.5, 3.49999, 254.5, 253.5, 0.0, 255.0]], np.float32)
    np.testing.assert_array_equal(oracle.output(F), [[0, 2, 2, 3, 254, 254, 0, 255]])


# --------------------------------------------------------------------------
# Whole pipeline
# --------------------------------------------------------------------------
KINDS = ["natural", "noise", "ramp", "checker", "impulse"]


@pytest.mark.parametrize("kind", KINDS)
@pytest.mark.parametrize("W,H", [(8, 8), (12, 8), (32, 20), (64, 48)])
def test_identity_params_reproduce_input(kind, W, H):
    # A = 1, gamma = 0: adj = 1, P = fma(1, O-U, U) = O, and O lies in its own
    # 3x3 [min, max] -> out == O bit for bit.
    O = synth.image(W, H, kind, seed=W * 131 + H, param=200)
    for G in (0.0, 0.5, 1.0):
        out, _, _ = oracle.sharpen(O, 1.0, 0.0, G, 2.0)
        np.testing.assert_array_equal(out, O)


@pytest.mark.parametrize("c", [0, 1, 128, 254, 255])
def test_constant_is_fixed_point(c):
    O = np.full((24, 32), c, np.uint8)
    for prm in [(1.0, 0.5, 0.5, 2.0), (16.0, 4.0, 1.0, 1e6), (0.0, 0.0, 0.0, 0.5)]:
        out, S, mean = oracle.sharpen(O, *prm)
        assert S == 0 and mean == 0.0
        assert np.all(out == c)


def test_zero_amount_zero_gain_closed_form():
    # A = 0, G = 0: P = U; interior -> rne(clamp(U, mn, mx)); frame -> rne(U)
    O = rand_img(40, 24)
    out, _, _ = oracle.sharpen(O, 0.0, 0.5, 0.0, 2.0)
    U = exact_ref.upscale(O)
    mx, mn = _window_minmax(O)
    exp = np.rint(np.clip(U, 0, 255))
    exp[1:-1, 1:-1] = np.rint(np.clip(U, mn, mx))[1:-1, 1:-1]
    np.testing.assert_array_equal(out, exp.astype(np.uint8))


@pytest.mark.parametrize("kind", ["natural", "noise"])
@pytest.mark.parametrize("W,H", [(16, 24), (40, 28)])
def test_transpose_invariance(kind, W, H):
    O = synth.image(W, H, kind, seed=3)
    out, S, _ = oracle.sharpen(O)
    outT, ST, _ = oracle.sharpen(O.T.copy())
    assert S == ST
    np.testing.assert_array_equal(outT, out.T)


PARAMS = [(1.0, 0.5, 0.5, 2.0), (2.5, 1.0, 0.25, 1.0), (6.0, 0.3, 0.9, 8.0),
          (0.5, 2.0, 0.0, 0.5), (16.0, 4.0, 1.0, 1e6)]


@pytest.mark.parametrize("prm", PARAMS)
@pytest.mark.parametrize("kind", ["natural", "noise", "ramp"])
def test_pipeline_agrees_with_real_number_evaluation(prm, kind):
    # The f32 chain may only differ from the float64 real-number result by
    # the final rounding of values within a hair of a .5 tie.
    O = synth.image(48, 32, kind, seed=11)
    out, S, mean = oracle.sharpen(O, *prm)
    F, S_ref = exact_ref.sharpen_f64(O, *prm)
    assert S == S_ref and mean == S_ref / O.size
    d = np.abs(out.astype(np.int64) - np.rint(F).astype(np.int64))
    assert d.max() <= 1
    far = np.abs(F - np.floor(F) - 0.5) > 1e-3
    np.testing.assert_array_equal(out[far], np.rint(F[far]).astype(np.uint8))


def test_batch_equals_single_and_thread_count_independent():
    imgs = synth.frames(6, 32, 24, "natural", seed=99)
    o1, s1 = oracle.sharpen_batch(imgs, threads=1)
    o4, s4 = oracle.sharpen_batch(imgs, threads=4)
    np.testing.assert_array_equal(o1, o4)
    np.testing.assert_array_equal(s1, s4)
    for f in range(6):
        out, S, _ = oracle.sharpen(imgs[f])
        np.testing.assert_array_equal(out, o1[f])
        assert S == s1[f]


@pytest.mark.parametrize("W,H", [(6, 8), (8, 6), (10, 8), (8, 10), (4, 4), (0, 8)])
def test_geometry_rejected(W, H):
    # R1
    import ctypes
    lib = oracle._load()
    assert lib.oracle_check_geometry(W, H) == -1
    if W > 0 and H > 0:
        with pytest.raises(ValueError):
            oracle.sharpen(np.zeros((H, W), np.uint8))


@pytest.mark.parametrize("prm", [(-1, 0.5, 0.5, 2), (1, 5, 0.5, 2), (1, 0.5, 1.5, 2),
                                 (1, 0.5, 0.5, 0), (float("nan"), 0.5, 0.5, 2)])
def test_params_rejected(prm):
    with pytest.raises(ValueError):
        oracle.sharpen(np.zeros((8, 8), np.uint8), *prm)
