"""Pins of the oracle's general geometry (reading R1', SURVEY.md sec. 8(f)
NEXT 3) and of its reading switches (R2, R5, R8, R9, R11, R14 alternatives,
NEXT 4) against things other than the oracle itself: numpy / brute-force
formulations of the extension and the integer downscale, hand-derived corner
values of the border step order, closed forms, special cases that reduce to a
library routine (np.floor, np.clip), and metamorphic invariants (identity
parameters, constants, transposition, pitch).
"""
import numpy as np
import pytest

import oracle
import synth

RNG = np.random.default_rng(20151017)
ODD_SIZES = [(5, 5), (9, 7), (13, 9), (17, 22), (30, 31), (33, 18), (64, 61)]
FLAG_SETS = [0, oracle.READ_INT_DOWNSCALE, oracle.READ_COLUMN_WINS, oracle.READ_INTERIOR_MEAN,
             oracle.READ_STRENGTH_EXP, oracle.READ_OSC_CONST, oracle.READ_TRUNCATE, oracle.READ_ALL]


def rand_img(W, H):
    return RNG.integers(0, 256, size=(H, W), dtype=np.int64).astype(np.uint8)


def natural(W, H, seed):
    """A `natural` synthetic frame of any size (cropped from one >= 16 x 16)."""
    return np.ascontiguousarray(synth.image(max(W, 16), max(H, 16), "natural", seed=seed)[:H, :W])


# --------------------------------------------------------------------------
# R1': general geometry (replicate-extend to multiples of 4, crop)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", [(8, 8), (16, 12), (32, 20), (64, 48)])
@pytest.mark.parametrize("flags", [0, oracle.READ_TRUNCATE])
def test_general_reduces_to_r1_for_multiples_of_4(W, H, flags):
    O = synth.image(W, H, "natural", seed=synth.BASE_SEED + W + H)
    a, Sa, ma = oracle.sharpen_ex(O, flags=0)
    b, Sb, mb = oracle.sharpen(O)
    assert np.array_equal(a, b) and Sa == Sb and ma == mb


@pytest.mark.parametrize("W,H", ODD_SIZES)
def test_general_equals_numpy_edge_pad_then_crop(W, H):
    """R1': the extension is np.pad(mode='edge') to the right and bottom."""
    O = rand_img(W, H)
    W4, H4 = -(-W // 4) * 4, -(-H // 4) * 4
    X = np.pad(O, ((0, H4 - H), (0, W4 - W)), mode="edge")
    ref, S, mean = oracle.sharpen(X)
    out, S2, mean2 = oracle.sharpen_ex(O)
    assert np.array_equal(out, ref[:H, :W]) and S == S2 and mean == mean2


@pytest.mark.parametrize("W,H", ODD_SIZES)
@pytest.mark.parametrize("flags", [0, oracle.READ_INT_DOWNSCALE, oracle.READ_TRUNCATE, oracle.READ_OSC_CONST])
def test_general_identity_params_reproduce_input(W, H, flags):
    """A = 1, gamma = 0: adj = 1, P = U + (O - U) = O exactly, O is inside its
    own 3x3 window -> the output is the input, at every size (pins the crop
    alignment of R1').  (Not with R9-exp, whose strength is not 1.)"""
    O = rand_img(W, H)
    out, _, _ = oracle.sharpen_ex(O, amount=1.0, gamma=0.0, flags=flags)
    assert np.array_equal(out, O)


@pytest.mark.parametrize("W,H", ODD_SIZES)
@pytest.mark.parametrize("flags", FLAG_SETS)
def test_general_constant_is_fixed_point(W, H, flags):
    O = np.full((H, W), 77, np.uint8)
    out, S, _ = oracle.sharpen_ex(O, flags=flags)
    assert S == 0 and np.all(out == 77)


@pytest.mark.parametrize("W,H", ODD_SIZES)
@pytest.mark.parametrize("flags", [f for f in FLAG_SETS if not f & oracle.READ_COLUMN_WINS])
def test_general_transpose_invariance(W, H, flags):
    O = natural(W, H, synth.BASE_SEED + 7 * W + H)
    a, Sa, _ = oracle.sharpen_ex(O, flags=flags)
    b, Sb, _ = oracle.sharpen_ex(np.ascontiguousarray(O.T), flags=flags)
    assert Sa == Sb and np.array_equal(a, b.T)


@pytest.mark.parametrize("W,H", [(13, 9), (30, 31)])
def test_general_pitch_view(W, H):
    big = rand_img(W + 37, H + 5)
    view = big[3:3 + H, 11:11 + W]
    a, Sa, _ = oracle.sharpen_ex(view)
    b, Sb, _ = oracle.sharpen_ex(np.ascontiguousarray(view))
    assert Sa == Sb and np.array_equal(a, b)


def test_general_rejects_bad_geometry():
    for W, H in [(4, 8), (8, 4), (3, 3)]:
        with pytest.raises(ValueError):
            oracle.sharpen_ex(np.zeros((H, W), np.uint8))
    with pytest.raises(ValueError):
        oracle.sharpen_ex(np.zeros((8, 8), np.uint8), flags=64)


# --------------------------------------------------------------------------
# R2 alternative: integer downscale (L374: shifts replace division)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", [(8, 8), (16, 12), (36, 20)])
def test_int_downscale_bruteforce(W, H):
    O = rand_img(W, H)
    D = oracle.downscale_ex(O, oracle.READ_INT_DOWNSCALE)
    sums = O.reshape(H // 4, 4, W // 4, 4).astype(np.int64).sum(axis=(1, 3))
    assert np.array_equal(D, (sums // 16).astype(np.float32))
    # and it is never above the exact mean, by less than one grey level
    Dx = oracle.downscale(O)
    assert np.all(D <= Dx) and np.all(Dx - D < 1.0)


def test_int_downscale_equals_exact_for_multiples_of_16():
    O = np.kron(rand_img(5, 4), np.ones((4, 4), np.uint8))  # constant 4x4 blocks: sums = 16 v
    assert np.array_equal(oracle.downscale_ex(O, oracle.READ_INT_DOWNSCALE), oracle.downscale(O))


# --------------------------------------------------------------------------
# R5 alternative: column work after row work in the border steps (L140)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", [(8, 8), (16, 12), (20, 28)])
def test_column_wins_only_changes_top_left_2x2(W, H):
    D = oracle.downscale(rand_img(W, H))
    U0 = oracle.upscale(D, W, H)
    U1 = oracle.upscale_ex(D, W, H, oracle.READ_COLUMN_WINS)
    diff = U0 != U1
    diff[:2, :2] = False
    assert not diff.any()
    # hand-derived: (ii) writes column 0 = line of D column 0, (vi) copies it to column 1
    d00, d10 = float(D[0, 0]), float(D[1, 0])
    lerp = (3 * d00 + d10) / 4
    assert U1[0, 0] == d00 and U1[0, 1] == d00
    assert U1[1, 0] == np.float32(lerp) and U1[1, 1] == np.float32(lerp)
    # default (R5): the whole 2x2 is D[0][0]
    assert np.all(U0[:2, :2] == d00)


@pytest.mark.parametrize("W,H", [(8, 8), (24, 16)])
def test_column_wins_leaves_only_bottom_right_after_six_steps(W, H):
    """L142: "the four elements of the bottom right corner are still missing"
    holds in the alternative order too."""
    D = oracle.downscale(rand_img(W, H))
    U = oracle.upscale_ex(D, W, H, oracle.READ_COLUMN_WINS, last_step=6)
    ring = np.zeros((H, W), bool)
    ring[:2, :] = ring[-2:, :] = ring[:, :2] = ring[:, -2:] = True
    missing = np.isnan(U) & ring
    assert np.array_equal(np.argwhere(missing), np.argwhere(np.pad(np.ones((2, 2), bool), ((H - 2, 0), (W - 2, 0)))))


def test_column_wins_breaks_transpose_invariance():
    """the alternative is not transpose-symmetric (the default is)."""
    O = synth.image(32, 32, "natural", seed=synth.BASE_SEED + 3)
    D = oracle.downscale(O)
    Dt = oracle.downscale(np.ascontiguousarray(O.T))
    U = oracle.upscale_ex(D, 32, 32, oracle.READ_COLUMN_WINS)
    Ut = oracle.upscale_ex(Dt, 32, 32, oracle.READ_COLUMN_WINS)
    if D[0, 0] != D[1, 0] or D[0, 0] != D[0, 1]:
        assert not np.array_equal(U, Ut.T)


# --------------------------------------------------------------------------
# R8 alternative: interior-only mean
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H,b,c", [(16, 12, 2, 3), (40, 24, 1, -2), (64, 32, -3, 1)])
def test_interior_mean_ramp_closed_form(W, H, b, c):
    a = 20 - min(0, b * (W - 1)) - min(0, c * (H - 1))
    rr, cc = np.meshgrid(np.arange(H), np.arange(W), indexing="ij")
    O = (a + b * cc + c * rr).astype(np.uint8)
    pE = oracle.sobel(O)
    S, mean = oracle.reduce_ex(pE, oracle.READ_INTERIOR_MEAN)
    S0, mean0 = oracle.reduce(pE)
    assert S == S0 == 8 * (abs(b) + abs(c)) * (W - 2) * (H - 2)
    assert mean == 8 * (abs(b) + abs(c))  # the interior is the ramp's exact gradient
    assert mean0 == pytest.approx(mean * (W - 2) * (H - 2) / (W * H), rel=1e-15)


# --------------------------------------------------------------------------
# R9 alternative: saturating strength (shape parity unpinned; special cases)
# --------------------------------------------------------------------------
def test_strength_exp_special_cases():
    pE = np.arange(0, 1531, 2, dtype=np.int32).reshape(1, -1)
    adj = oracle.strength_ex(pE, 40.0, 2.5, 0.5, 2.0, oracle.READ_STRENGTH_EXP)
    assert adj[0, 0] == 0.0                      # no edge, no sharpening
    assert np.all(np.diff(adj[0]) >= 0)          # monotone in pEdge
    assert np.all(adj <= 2.5) and adj[0, -1] > 2.5 * (1 - np.exp(-1530 / 80.0)) * (1 - 1e-6)
    assert np.all(oracle.strength_ex(pE, 40.0, 0.0, 0.5, 2.0, oracle.READ_STRENGTH_EXP) == 0)
    # the default curve is untouched by the unrelated K
    assert np.array_equal(oracle.strength_ex(pE, 40.0, 1.5, 0.5, 7.0, 0), oracle.strength(pE, 40.0, 1.5, 0.5))


# --------------------------------------------------------------------------
# R11 alternative: constant oscStrength
# --------------------------------------------------------------------------
@pytest.mark.parametrize("W,H", [(16, 16), (24, 20)])
def test_osc_const_one_disables_overshoot_control(W, H):
    """osc = G = 1: osc max = max + (P - max) = P, so Final = clamp(P, 0, 255)
    for every pixel (np.clip)."""
    O = synth.image(W, H, "natural", seed=synth.BASE_SEED + 11)
    D = oracle.downscale(O)
    U = oracle.upscale(D, W, H)
    pE = oracle.sobel(O)
    S, mean = oracle.reduce(pE)
    adj = oracle.strength(pE, mean, 3.0, 0.5)
    P = oracle.preliminary(adj, oracle.perror(O, U), U)
    F = oracle.overshoot_ex(O, P, pE, mean, 1.0, 2.0, oracle.READ_OSC_CONST)
    # exact wherever P >= window min (P - max is exact for P > max); below the
    # min, P - min is one f32 rounding, so within an ulp of 255
    from scipy import ndimage
    mn = ndimage.minimum_filter(O, size=3).astype(np.float32)
    exact = P >= mn
    exact[0, :] = exact[-1, :] = exact[:, 0] = exact[:, -1] = True  # frame: clamp(P) (R13)
    assert np.array_equal(F[exact], np.clip(P, 0, 255)[exact])
    assert np.all(np.abs(F - np.clip(P, 0, 255)) <= 2.0 ** -15)


@pytest.mark.parametrize("G", [0.0, 0.25, 0.5])
def test_osc_const_is_pedge_independent(G):
    """Two images with the same O window / P but different pEdge get the same
    Final under R11-const."""
    W = H = 16
    O = synth.image(W, H, "natural", seed=synth.BASE_SEED + 12)
    P = (O.astype(np.float32) * 1.3 - 20.0).astype(np.float32)
    pE1 = oracle.sobel(O)
    pE2 = (pE1[::-1, ::-1] + 4).astype(np.int32)
    a = oracle.overshoot_ex(O, P, pE1, 30.0, G, 2.0, oracle.READ_OSC_CONST)
    b = oracle.overshoot_ex(O, P, pE2, 30.0, G, 2.0, oracle.READ_OSC_CONST)
    assert np.array_equal(a, b)


# --------------------------------------------------------------------------
# R14 alternative: truncation
# --------------------------------------------------------------------------
def test_truncate_is_floor_on_the_output_range():
    F = np.concatenate([RNG.uniform(0, 255, 5000), np.arange(0, 255) + 0.5, np.arange(0, 256)]).astype(np.float32)
    assert np.array_equal(oracle.output_ex(F, oracle.READ_TRUNCATE), np.floor(F).astype(np.uint8))
    ties = (np.arange(0, 255) + 0.5).astype(np.float32)
    rne = oracle.output_ex(ties, 0)
    assert np.array_equal(rne, np.round(ties).astype(np.uint8))  # numpy rounds half to even
    assert np.array_equal(oracle.output_ex(ties, oracle.READ_TRUNCATE), (ties - 0.5).astype(np.uint8))


@pytest.mark.parametrize("flags", FLAG_SETS)
def test_flags_whole_pipeline_range_and_determinism(flags):
    O = synth.image(20, 13, "natural", seed=synth.BASE_SEED + 5)
    a = oracle.sharpen_ex(O, amount=2.0, flags=flags)
    b = oracle.sharpen_ex(O, amount=2.0, flags=flags)
    assert np.array_equal(a[0], b[0]) and a[1] == b[1]
