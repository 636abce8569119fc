"""GPU <-> oracle parity through the C ABI (task rule 3).

Every output pixel must be bit-identical to the oracle (the oracle fixes the
f32 evaluation order everywhere, R15), the pEdge sum S exact and
the mean exact.  Inputs: tests/../synth (seeded), the same bytes on both sides.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EINVAL, SHARP_EUNSUPPORTED, SHARP_PATH_FUSED, SHARP_PATH_FUSED_EXP,
                                            SHARP_PATH_RES, SHARP_PATH_STAGED,
                                            SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, STAGE_NAMES, SharpError, Sharpener)

pytestmark = pytest.mark.gpu

DEFAULT = (1.0, 0.5, 0.5, 2.0)
PARAMS = [
    DEFAULT,
    (1.0, 0.0, 0.5, 2.0),     # identity: adj == 1
    (0.0, 0.5, 0.0, 2.0),     # A = 0, G = 0
    (2.5, 1.0, 0.25, 1.0),
    (16.0, 4.0, 1.0, 1e6),    # extremes
    (0.5, 2.0, 0.0, 0.5),
    (6.0, 0.3, 0.9, 8.0),
]


@pytest.fixture(scope="module", params=["auto", "res", "step", "generic", "fused", "fused_exp", "staged"])
def sh(request):
    """A context on the automatic kernel path (the TMEM-resident kernel, else
    the step kernel, when W % 16 == 0), one forced onto the step kernel, one
    forced onto the generic two-pass LDG kernels, and one on the paper's
    staged base design (one kernel per stage)."""
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import os
    old = os.environ.get("SHARP_FORCE_GENERIC")
    os.environ["SHARP_FORCE_GENERIC"] = "1" if request.param == "generic" else "0"
    s = Sharpener()
    if request.param == "staged":
        s.set_path(SHARP_PATH_STAGED)
    if request.param == "step":
        s.set_path(SHARP_PATH_STEP)
        s._force_step = True
    if request.param == "res":
        s.set_path(SHARP_PATH_RES)
        s._force_step = True  # same geometry rules
    if request.param == "fused":
        s.set_path(SHARP_PATH_FUSED)
    if request.param == "fused_exp":
        s.set_path(SHARP_PATH_FUSED_EXP)
    if old is None:
        del os.environ["SHARP_FORCE_GENERIC"]
    else:
        os.environ["SHARP_FORCE_GENERIC"] = old
    yield s
    s.close()


def gpu_run(sh, img, prm=DEFAULT):
    d = torch.from_numpy(img).cuda()
    o = torch.empty_like(d)
    sh.run(d, prm, o)
    torch.cuda.synchronize()
    st = sh.stats()
    return o.cpu().numpy(), st.edge_sum, st.edge_mean


def assert_parity(sh, img, prm=DEFAULT):
    if getattr(sh, "_force_step", False) and (img.shape[-1] % 16 or img.shape[-1] < 16):
        pytest.skip("SHARP_PATH_STEP needs W % 16 == 0 (the other fixtures cover this size)")
    try:
        out, S, mean = gpu_run(sh, img, prm)
    except SharpError as e:
        if getattr(sh, "_force_step", False) and e.code == SHARP_EUNSUPPORTED:
            pytest.skip(f"forced path does not take this size: {e}")
        raise
    ref, S_ref, mean_ref = oracle.sharpen(img, *prm)
    bad = np.argwhere(out != ref)
    assert S == S_ref, f"edge sum {S} != {S_ref}"
    assert mean == mean_ref
    assert bad.size == 0, (f"{len(bad)} mismatches of {out.size}, first at {bad[:5].tolist()}: "
                           f"gpu {out[tuple(bad[0])]} oracle {ref[tuple(bad[0])]}")


SIZES = [(8, 8), (12, 8), (8, 12), (16, 16), (20, 12), (64, 48), (100, 36), (252, 20), (260, 36),
         (300, 68), (516, 44), (1028, 40),
         # W % 16 == 0 (TMA path): one warp tile, tile + 16, CTA tile edges, ragged rows
         (16, 8), (32, 12), (240, 36), (256, 40), (480, 68), (960, 36), (976, 44), (1920, 36)]


@pytest.mark.parametrize("W,H", SIZES)
@pytest.mark.parametrize("kind", ["natural", "noise"])
def test_small_sizes_tiles_and_ragged_tails(W, H, kind, sh):
    img = synth.image(W, H, kind, seed=W * 1000 + H)
    assert_parity(sh, img)


@pytest.mark.parametrize("kind,param", [("natural", 0), ("noise", 0), ("ramp", 0), ("const", 0),
                                        ("const", 255), ("const", 131), ("checker", 30),
                                        ("impulse", 255)])
@pytest.mark.parametrize("prm", PARAMS)
def test_kinds_and_params_512(kind, param, prm, sh):
    img = synth.image(512, 512, kind, seed=synth.BASE_SEED, param=param)
    assert_parity(sh, img, prm)


@pytest.mark.parametrize("W,H,seed", [(1920, 1080, 1), (3840, 2160, 2)])
def test_full_frames_1080p_4k(W, H, seed, sh):
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + seed)
    assert_parity(sh, img)


def test_full_frame_8k(sh):
    img = synth.image(7680, 4320, "natural", seed=synth.BASE_SEED + 3)
    assert_parity(sh, img)


def test_identity_params_reproduce_input_on_gpu(sh):
    img = synth.image(1920, 1080, "noise", seed=7)
    out, _, _ = gpu_run(sh, img, (1.0, 0.0, 0.3, 2.0))
    np.testing.assert_array_equal(out, img)


def test_batch_frames_independent_and_equal_to_oracle(sh):
    imgs = synth.frames(6, 264, 40, "natural", seed=123)
    imgs[2] = 77  # a constant frame in the middle: S = 0
    d = torch.from_numpy(imgs).cuda()
    o = torch.empty_like(d)
    sh.run_batch(d, DEFAULT, o)
    sums = sh.batch_sums(6)
    out = o.cpu().numpy()
    ref, ref_sums = oracle.sharpen_batch(imgs, *DEFAULT)
    np.testing.assert_array_equal(out, ref)
    assert sums == [int(s) for s in ref_sums]


@pytest.mark.parametrize("n,W,H", [(1, 16, 8), (3, 16, 16), (40, 256, 40), (9, 976, 44), (2, 3840, 2160),
                                   (20, 976, 100), (80, 480, 260)])
def test_batch_single_launch_dependencies(n, W, H):
    """TMA batch kernel: pass 1 -> LUT -> pass 2 dependencies resolved inside
    one launch (rounds with lags; empty tasks at the ends).  (20, 976, 100):
    the compact order of a mid-size batch; (80, 480, 260): the lagged order
    with 2-sub-tile pass-1 and 4-sub-tile pass-2 tasks and ragged last tasks
    (260 = 7 x 36 + 8 = 5 x 48 + 20 rows)."""
    imgs = synth.frames(n, W, H, "natural", seed=n * 7 + W)
    with Sharpener() as s:
        d = torch.from_numpy(imgs).cuda()
        o = torch.empty_like(d)
        s.run_batch(d, DEFAULT, o)
        sums = s.batch_sums(n)
        st = s.stats()
    ref, ref_sums = oracle.sharpen_batch(imgs, *DEFAULT)
    np.testing.assert_array_equal(o.cpu().numpy(), ref)
    assert sums == [int(x) for x in ref_sums]
    assert st.edge_sum == int(ref_sums[0])


def test_batch_chunking_many_chunks():
    # chunk_frames=3 forces several pass-1/pass-2 chunk pairs on one stream
    imgs = synth.frames(10, 128, 64, "natural", seed=9)
    with Sharpener(chunk_frames=3) as s:
        d = torch.from_numpy(imgs).cuda()
        o = torch.empty_like(d)
        s.run_batch(d, DEFAULT, o)
        sums = s.batch_sums(10)
    ref, ref_sums = oracle.sharpen_batch(imgs, *DEFAULT)
    np.testing.assert_array_equal(o.cpu().numpy(), ref)
    assert sums == [int(x) for x in ref_sums]


@pytest.mark.parametrize("mode", ["pageable", "pinned", "dev_in_host_out", "host_in_dev_out"])
def test_host_memory_paths(mode):
    imgs = synth.frames(7, 1920, 1080, "natural", seed=44)
    ref, ref_sums = oracle.sharpen_batch(imgs, *DEFAULT)
    with Sharpener(chunk_frames=2, streams=3) as s:
        if mode == "pageable":
            out = np.empty_like(imgs)
            s.run_batch(imgs, DEFAULT, out)
        elif mode == "pinned":
            src = torch.from_numpy(imgs).pin_memory()
            dst = torch.empty_like(src).pin_memory()
            s.run_batch(src, DEFAULT, dst)
            out = dst.numpy()
        elif mode == "dev_in_host_out":
            src = torch.from_numpy(imgs).cuda()
            out = np.empty_like(imgs)
            s.run_batch(src, DEFAULT, out)
        else:
            dst = torch.empty(imgs.shape, dtype=torch.uint8, device="cuda")
            s.run_batch(imgs, DEFAULT, dst)
            out = dst.cpu().numpy()
        sums = s.batch_sums(7)
    np.testing.assert_array_equal(out, ref)
    assert sums == [int(x) for x in ref_sums]


def test_bench_configuration_sampled_frames():
    """The bench's launch configuration (1024 x 1080p, device-resident,
    automatic chunking) compared on sampled frames against the oracle."""
    n, W, H = 1024, 1920, 1080
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 5)
    with Sharpener() as s:
        d = torch.from_numpy(imgs).cuda()
        o = torch.empty_like(d)
        s.enqueue_batch(d, o, DEFAULT)
        torch.cuda.synchronize()
        sums = s.batch_sums(n)
    sample = list(range(0, n, 33))[:32]
    ref, ref_sums = oracle.sharpen_batch(imgs[sample], *DEFAULT)
    out = o[sample].cpu().numpy()
    np.testing.assert_array_equal(out, ref)
    assert [sums[i] for i in sample] == [int(x) for x in ref_sums]


@pytest.mark.parametrize("W,H", [(6, 8), (8, 6), (10, 8), (8, 10)])
def test_invalid_geometry_rejected_out_untouched(W, H, sh):
    d = torch.zeros((H, W), dtype=torch.uint8, device="cuda")
    o = torch.full((H, W), 7, dtype=torch.uint8, device="cuda")
    with pytest.raises(SharpError) as e:
        sh.run(d, DEFAULT, o)
    assert e.value.code == SHARP_EINVAL
    assert bool((o == 7).all())


def test_invalid_params_and_overlap_rejected(sh):
    d = torch.zeros((64, 64), dtype=torch.uint8, device="cuda")
    o = torch.full((64, 64), 7, dtype=torch.uint8, device="cuda")
    for bad in [(float("nan"), 0.5, 0.5, 2.0), (1.0, 5.0, 0.5, 2.0), (1.0, 0.5, -0.1, 2.0),
                (1.0, 0.5, 0.5, 0.0), (17.0, 0.5, 0.5, 2.0)]:
        with pytest.raises(SharpError) as e:
            sh.run(d, bad, o)
        assert e.value.code == SHARP_EINVAL
    assert bool((o == 7).all())
    big = torch.zeros((2, 64, 64), dtype=torch.uint8, device="cuda")
    with pytest.raises(SharpError) as e:
        sh.run(big[0], DEFAULT, big[0])  # in place
    assert e.value.code == SHARP_EINVAL


def test_ladder_paths_identical_and_stage_times():
    """The optimisation ladder (staged base -> scalar fused with per-pixel
    exponentiation -> + strength table -> vectorised two-pass -> step kernel
    -> TMEM-resident kernel) gives the same bytes; the staged path reports a
    time for every stage."""
    imgs = synth.frames(2, 3840, 2160, "natural", seed=synth.BASE_SEED + 2)
    ref, ref_sums = oracle.sharpen_batch(imgs, *DEFAULT)
    d = torch.from_numpy(imgs).cuda()
    for path in [SHARP_PATH_STAGED, SHARP_PATH_FUSED_EXP, SHARP_PATH_FUSED, SHARP_PATH_TWO_PASS, SHARP_PATH_STEP,
                 SHARP_PATH_RES]:
        with Sharpener() as s:
            s.set_path(path)
            s.set_profiling(True)
            o = torch.empty_like(d)
            s.run_batch(d, DEFAULT, o)
            np.testing.assert_array_equal(o.cpu().numpy(), ref)
            assert s.batch_sums(2) == [int(x) for x in ref_sums]
            if path == SHARP_PATH_STAGED:
                t = s.stage_times()
                assert list(t) == list(STAGE_NAMES)
                assert all(v > 0 for v in t.values()), t
                assert s.stats().kernels == 2 * 7


def test_step_path_rejects_unsupported_geometry():
    with Sharpener() as s:
        s.set_path(SHARP_PATH_STEP)
        d = torch.zeros((16, 20), dtype=torch.uint8, device="cuda")  # W % 16 != 0
        o = torch.empty_like(d)
        with pytest.raises(SharpError) as e:
            s.run(d, DEFAULT, o)
        assert e.value.code == SHARP_EUNSUPPORTED



def oracle_rows(img, mean, r0, r1, prm=DEFAULT):
    """Oracle output rows [r0, r1) of a big image from its stages on the row
    window [max(r0 - 8, 0), min(r1 + 8, H)) (4-aligned r0, r1) with the WHOLE
    image's mean: an output row reads D, U (body formula, L146), pEdge and the
    3x3 window only within 5 rows, so rows more than 5 away
    from a window edge that is not an image edge equal the whole-image stages."""
    A, g, G, K = prm
    lo, hi = max(r0 - 8, 0), min(r1 + 8, img.shape[0])
    sub = np.ascontiguousarray(img[lo:hi])
    Hs, Ws = sub.shape
    U = oracle.upscale(oracle.downscale(sub), Ws, Hs)
    pE = oracle.sobel(sub)
    adj = oracle.strength(pE, mean, A, g)
    P = oracle.preliminary(adj, oracle.perror(sub, U), U)
    return oracle.output(oracle.overshoot(sub, P, pE, mean, G, K))[r0 - lo:r1 - lo]


def test_oracle_rows_helper_matches_whole_image():
    img = synth.image(512, 256, "natural", seed=5)
    ref, S, mean = oracle.sharpen(img)
    for r0 in (0, 8, 100, 192):
        np.testing.assert_array_equal(oracle_rows(img, mean, r0, r0 + 64), ref[r0:r0 + 64])


def test_full_size_16384_sampled_rows():
    """BASELINE configs[3] C4b (16384^2, 268 Mpx) on one GPU: S exact against
    the oracle's full-image Sobel + reduction, and 64-row bands at the top
    (ring rows), middle and bottom (ring rows) bit-exact."""
    W = H = 16384
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 4)
    s = Sharpener()
    d = torch.from_numpy(img).cuda()
    o = torch.empty_like(d)
    s.run(d, DEFAULT, o)
    torch.cuda.synchronize()
    st = s.stats()
    S_ref, mean_ref = oracle.reduce(oracle.sobel(img))
    assert st.edge_sum == S_ref and st.edge_mean == mean_ref
    out = o.cpu().numpy()
    for r0 in (0, 8192 - 32, H - 64):
        np.testing.assert_array_equal(out[r0:r0 + 64], oracle_rows(img, mean_ref, r0, r0 + 64))
    s.close()


@pytest.mark.parametrize("W,H,path", [(32768, 16384, "step"), (32768, 16392, "two-pass")])
def test_maximum_sizes_at_the_step_kernel_limit(W, H, path):
    """Edge of the step kernel's domain (W*H <= 2^29: the packed arrival count
    + 40-bit sum of `acc`) with worst-case content (uniform
    noise, large pEdge everywhere), and just past it (the two-pass path takes
    over).  S exact against the oracle's full-image Sobel + reduction; top,
    middle and bottom row bands bit-exact."""
    img = synth.image(W, H, "noise", seed=synth.BASE_SEED + 6)
    s = Sharpener()
    d = torch.from_numpy(img).cuda()
    o = torch.empty_like(d)
    s.set_profiling(True)
    s.run(d, DEFAULT, o)
    torch.cuda.synchronize()
    kt = s.kernel_times()
    assert (kt.step_launches > 0) == (path == "step")
    st = s.stats()
    S_ref, mean_ref = oracle.reduce(oracle.sobel(img))
    assert st.edge_sum == S_ref and st.edge_mean == mean_ref
    out = o.cpu().numpy()
    for r0 in (0, (H // 2) & ~3, H - 32):
        np.testing.assert_array_equal(out[r0:r0 + 32], oracle_rows(img, mean_ref, r0, r0 + 32))
    s.close()


def test_randomised_parameters_bit_exact():
    """300 seeded random parameter sets (A, gamma, G, K over their ranges) x
    random natural / noise frames: every output bit-exact, S exact.  Stresses
    the f64 pow / exp of the tables (CUDA libm vs glibc, R19) and
    the f32 overshoot chain far from the default parameters."""
    rng = np.random.default_rng(20151016)
    s = Sharpener()
    kinds = ["natural", "noise"]
    imgs = [synth.image(96, 64, kinds[i % 2], seed=synth.BASE_SEED + 900 + i) for i in range(12)]
    d = [torch.from_numpy(im).cuda() for im in imgs]
    o = torch.empty_like(d[0])
    for case in range(300):
        prm = (float(rng.uniform(0, 16)), float(rng.uniform(0, 4)), float(rng.uniform(0, 1)),
               float(np.exp(rng.uniform(np.log(1e-3), np.log(1e3)))))
        prm = tuple(float(np.float32(v)) for v in prm)
        k = case % len(imgs)
        s.run(d[k], prm, o)
        torch.cuda.synchronize()
        ref, S_ref, _ = oracle.sharpen(imgs[k], *prm)
        got = o.cpu().numpy()
        assert s.stats().edge_sum == S_ref
        bad = np.argwhere(got != ref)
        assert bad.size == 0, f"case {case} params {prm}: {len(bad)} mismatches, first {bad[:3].tolist()}"
    s.close()
