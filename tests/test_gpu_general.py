"""GPU <-> oracle parity of sharp_run_ex:
general sizes (reading R1': replicate-extend to multiples of 4, crop),
pitched / ROI / interleaved-channel layouts, in-place calls, host and device
buffers, and the reading switches (R2, R5, R8, R9, R11, R14 alternatives) on
every kernel path.  Bit-exact outputs and exact S, like test_gpu_parity.py.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_EINVAL, SHARP_EUNSUPPORTED, SHARP_PATH_STAGED, SHARP_PATH_STEP,
                                            SHARP_PATH_TWO_PASS, SharpError, Sharpener, sharp_run_ex)

pytestmark = pytest.mark.gpu

DEFAULT = (1.0, 0.5, 0.5, 2.0)
STRONG = (2.5, 1.0, 0.25, 1.0)
FLAGS = [0, oracle.READ_INT_DOWNSCALE, oracle.READ_COLUMN_WINS, oracle.READ_INTERIOR_MEAN,
         oracle.READ_STRENGTH_EXP, oracle.READ_OSC_CONST, oracle.READ_TRUNCATE, oracle.READ_ALL,
         oracle.READ_INTERIOR_MEAN | oracle.READ_STRENGTH_EXP | oracle.READ_OSC_CONST]


@pytest.fixture(scope="module", params=["auto", "two_pass", "staged"])
def sh(request):
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    s = Sharpener()
    if request.param == "two_pass":
        s.set_path(SHARP_PATH_TWO_PASS)
    elif request.param == "staged":
        s.set_path(SHARP_PATH_STAGED)
    yield s
    s.close()


def natural(W, H, seed):
    return np.ascontiguousarray(synth.image(max(W, 16), max(H, 16), "natural", seed=seed)[:H, :W])


def ref_units(units, prm, flags):
    """oracle.sharpen_ex on each [H, W] unit -> (outs, sums)."""
    outs, sums = [], []
    for u in units:
        o, S, _ = oracle.sharpen_ex(u, *prm, flags=flags)
        outs.append(o)
        sums.append(S)
    return outs, sums


def check(out, ref, what=""):
    bad = np.argwhere(out != ref)
    assert bad.size == 0, f"{what}: {len(bad)} mismatches, first at {bad[:4].tolist()}"


# ------------------------------------------------------------ general sizes
ODD = [(5, 5), (9, 7), (13, 9), (17, 22), (30, 31), (33, 18), (250, 61), (257, 43), (963, 37), (1921, 29),
       (1918, 1081)]


@pytest.mark.parametrize("W,H", ODD)
@pytest.mark.parametrize("where", ["device", "host"])
def test_general_sizes(W, H, where, sh):
    img = natural(W, H, synth.BASE_SEED + 31 * W + H)
    t = torch.from_numpy(img)
    if where == "device":
        t = t.cuda()
    out = sh.run_ex(t, DEFAULT)
    torch.cuda.synchronize()
    ref, S, mean = oracle.sharpen_ex(img, *DEFAULT)
    check(out.cpu().numpy(), ref, f"{W}x{H}")
    st = sh.stats()
    assert st.edge_sum == S and st.edge_mean == mean


@pytest.mark.parametrize("W,H", [(16, 8), (1920, 36), (64, 48)])
def test_dense_run_ex_is_run_batch(W, H, sh):
    imgs = synth.frames(3, W, H, "natural", seed=synth.BASE_SEED + 77)
    d = torch.from_numpy(imgs).cuda()
    a = sh.run_ex(d, STRONG)
    b = sh.run_batch(d, STRONG)
    torch.cuda.synchronize()
    check(a.cpu().numpy(), b.cpu().numpy(), "run_ex vs run_batch")


# ------------------------------------------------------------ layouts
@pytest.mark.parametrize("where", ["device", "host"])
@pytest.mark.parametrize("W,H", [(37, 21), (480, 64), (1001, 33)])
def test_roi_views_with_pitch(W, H, where, sh):
    big = synth.frames(2, W + 45, H + 11, "natural", seed=synth.BASE_SEED + 5)
    t = torch.from_numpy(big)
    if where == "device":
        t = t.cuda()
    roi = t[:, 7:7 + H, 13:13 + W]              # pitch W + 45, frame stride (W + 45)(H + 11)
    out_big = torch.full_like(t, 222)
    out = out_big[:, 3:3 + H, 29:29 + W]
    sh.run_ex(roi, STRONG, out=out)
    torch.cuda.synchronize()
    units = [np.ascontiguousarray(big[f, 7:7 + H, 13:13 + W]) for f in range(2)]
    refs, sums = ref_units(units, STRONG, 0)
    ob = out_big.cpu().numpy()
    for f in range(2):
        check(ob[f, 3:3 + H, 29:29 + W], refs[f], f"frame {f}")
    # bytes outside the crops are untouched
    mask = np.ones(ob.shape, bool)
    mask[:, 3:3 + H, 29:29 + W] = False
    assert np.all(ob[mask] == 222)
    assert sh.batch_sums(2) == sums


@pytest.mark.parametrize("where", ["device", "host"])
@pytest.mark.parametrize("W,H,C", [(64, 48, 3), (33, 17, 3), (16, 12, 4), (1920, 24, 3)])
def test_interleaved_channels(W, H, C, where, sh):
    planes = synth.frames(2 * C, W, H, "natural", seed=synth.BASE_SEED + 9)
    hwc = np.ascontiguousarray(planes.reshape(2, C, H, W).transpose(0, 2, 3, 1))  # [N, H, W, C]
    t = torch.from_numpy(hwc)
    if where == "device":
        t = t.cuda()
    out = sh.run_ex(t, DEFAULT, channels_last=True)
    torch.cuda.synchronize()
    o = out.cpu().numpy()
    refs, sums = ref_units([planes[i] for i in range(2 * C)], DEFAULT, 0)
    for f in range(2):
        for c in range(C):
            check(o[f, :, :, c], refs[f * C + c], f"frame {f} channel {c}")
    assert sh.batch_sums(2 * C) == sums


def test_rgb_channels_are_independent(sh):
    """A channel's result does not depend on the other channels (own mean)."""
    W, H = 40, 24
    a = synth.frames(3, W, H, "natural", seed=synth.BASE_SEED + 1)
    b = a.copy()
    b[2] = synth.image(W, H, "noise", seed=3)
    oa = sh.run_ex(torch.from_numpy(np.ascontiguousarray(a.transpose(1, 2, 0))).cuda(), channels_last=True).cpu()
    ob = sh.run_ex(torch.from_numpy(np.ascontiguousarray(b.transpose(1, 2, 0))).cuda(), channels_last=True).cpu()
    assert torch.equal(oa[:, :, :2], ob[:, :, :2]) and not torch.equal(oa[:, :, 2], ob[:, :, 2])


@pytest.mark.parametrize("where", ["device", "host"])
@pytest.mark.parametrize("W,H", [(64, 48), (50, 30), (1920, 40)])
def test_in_place(W, H, where, sh):
    imgs = synth.frames(3, W, H, "natural", seed=synth.BASE_SEED + 13)
    refs, _ = ref_units(list(imgs), STRONG, 0)
    t = torch.from_numpy(imgs.copy())
    if where == "device":
        t = t.cuda()
    sh.run_ex(t, STRONG, out=t)
    torch.cuda.synchronize()
    o = t.cpu().numpy()
    for f in range(3):
        check(o[f], refs[f], f"frame {f}")


# ------------------------------------------------------------ reading switches
@pytest.mark.parametrize("flags", FLAGS)
@pytest.mark.parametrize("W,H", [(16, 8), (64, 48), (260, 36), (1920, 36), (33, 18)])
def test_reading_switches(W, H, flags, sh):
    imgs = synth.frames(2, max(W, 16), max(H, 16), "natural", seed=synth.BASE_SEED + W + 3 * H + flags)
    imgs = np.ascontiguousarray(imgs[:, :H, :W])
    d = torch.from_numpy(imgs).cuda()
    out = sh.run_ex(d, STRONG, flags=flags)
    torch.cuda.synchronize()
    refs, sums = ref_units(list(imgs), STRONG, flags)
    o = out.cpu().numpy()
    for f in range(2):
        check(o[f], refs[f], f"flags {flags} frame {f}")
    assert sh.batch_sums(2) == sums


@pytest.mark.parametrize("flags", [oracle.READ_INTERIOR_MEAN, oracle.READ_STRENGTH_EXP, oracle.READ_OSC_CONST])
def test_lut_switches_on_the_step_kernel(flags):
    """R8 / R9 / R11 only change the per-frame tables: the step kernel runs them."""
    s = Sharpener()
    s.set_path(SHARP_PATH_STEP)
    imgs = synth.frames(4, 1920, 72, "natural", seed=synth.BASE_SEED + flags)
    out = s.run_ex(torch.from_numpy(imgs).cuda(), DEFAULT, flags=flags)
    torch.cuda.synchronize()
    refs, _ = ref_units(list(imgs), DEFAULT, flags)
    for f in range(4):
        check(out[f].cpu().numpy(), refs[f], f"frame {f}")
    s.close()


def test_per_pixel_switches_refused_on_the_step_path():
    s = Sharpener()
    s.set_path(SHARP_PATH_STEP)
    d = torch.zeros(1, 32, 64, dtype=torch.uint8, device="cuda")
    for flags in [oracle.READ_INT_DOWNSCALE, oracle.READ_COLUMN_WINS, oracle.READ_TRUNCATE]:
        with pytest.raises(SharpError) as e:
            s.run_ex(d, flags=flags)
        assert e.value.code == SHARP_EUNSUPPORTED
    s.close()


def test_run_ex_errors():
    s = Sharpener()
    d = torch.zeros(2, 16, 16, dtype=torch.uint8, device="cuda")
    o = torch.zeros_like(d)
    for args, code in [
        (dict(n=1, channels=1, w=4, h=16), SHARP_EINVAL),           # too small
        (dict(n=0, channels=1, w=16, h=16), SHARP_EINVAL),
        (dict(n=1, channels=2, w=16, h=16), SHARP_EINVAL),          # channels > elem_stride
    ]:
        with pytest.raises(SharpError) as e:
            sharp_run_ex(s.ctx, d, None, args["n"], args["channels"], args["w"], args["h"], None, 0, o, None)
        assert e.value.code == code
    with pytest.raises(SharpError) as e:
        sharp_run_ex(s.ctx, d, None, 1, 1, 16, 16, None, 64, o, None)   # unknown switch
    assert e.value.code == SHARP_EINVAL
    with pytest.raises(SharpError) as e:                                # shifted overlap
        sharp_run_ex(s.ctx, d, None, 1, 1, 16, 16, None, 0, d[0, 1], None)
    assert e.value.code == SHARP_EINVAL
    with pytest.raises(SharpError) as e:                                # pitch < w
        sharp_run_ex(s.ctx, d, (8, 0, 1), 1, 1, 16, 16, None, 0, o, None)
    assert e.value.code == SHARP_EINVAL
    s.close()


@pytest.mark.parametrize("where", ["device", "host"])
def test_general_path_in_chunks(where):
    """chunk_frames = 1: the gather / run / scatter loop runs once per frame
    (sums of every chunk kept), also in place."""
    s = Sharpener(chunk_frames=1)
    W, H, n = 45, 27, 4
    imgs = synth.frames(n, 48, 32, "natural", seed=synth.BASE_SEED + 21)[:, :H, :W].copy()
    refs, sums = ref_units(list(imgs), STRONG, 0)
    t = torch.from_numpy(imgs.copy())
    if where == "device":
        t = t.cuda()
    out = s.run_ex(t, STRONG)
    torch.cuda.synchronize()
    for f in range(n):
        check(out[f].cpu().numpy(), refs[f], f"frame {f}")
    assert s.batch_sums(n) == sums
    s.run_ex(t, STRONG, out=t)  # in place, chunk by chunk
    torch.cuda.synchronize()
    for f in range(n):
        check(t[f].cpu().numpy(), refs[f], f"in-place frame {f}")
    s.close()


@pytest.mark.parametrize("flags", [oracle.READ_TRUNCATE | oracle.READ_INTERIOR_MEAN, oracle.READ_STRENGTH_EXP])
def test_reading_switches_host_pipeline(flags):
    """Dense host buffers with switches: the pinned-staging pipeline path."""
    s = Sharpener(chunk_frames=2)
    imgs = synth.frames(5, 1920, 40, "natural", seed=synth.BASE_SEED + 2 * flags)
    out = s.run_ex(torch.from_numpy(imgs), DEFAULT, flags=flags)
    refs, sums = ref_units(list(imgs), DEFAULT, flags)
    for f in range(5):
        check(out[f].numpy(), refs[f], f"frame {f}")
    assert s.batch_sums(5) == sums
    s.close()


@pytest.mark.parametrize("W,H,pitch_in,pitch_out", [(1928, 64, 2000, 1944), (488, 36, 528, 496), (960, 12, 1008, 968)])
def test_zero_copy_strided_roi_on_the_step_kernel(W, H, pitch_in, pitch_out):
    """Device ROIs whose strides meet the TMA rules (W % 8 == 0, input pitch
    % 16, output pitch % 8, aligned bases) run straight through the step
    kernel -- no gather / scatter copies -- including W % 16 == 8."""
    s = Sharpener()
    big = synth.frames(2, pitch_in, H + 8, "natural", seed=synth.BASE_SEED + W)
    t = torch.from_numpy(big).cuda()
    roi = t[:, 4:4 + H, 32:32 + W]                      # base 16-byte aligned (offset 4 * pitch + 32)
    ob = torch.full((2, H + 4, pitch_out), 7, dtype=torch.uint8, device="cuda")
    out = ob[:, 2:2 + H, 8:8 + W]                       # 8-byte aligned
    s.set_profiling(True)
    s.run_ex(roi, STRONG, out=out)
    torch.cuda.synchronize()
    kt = s.kernel_times()
    assert kt.step_launches == 1 and s.stats().kernels == 1   # one launch, no layout kernels
    refs, sums = ref_units([np.ascontiguousarray(big[f, 4:4 + H, 32:32 + W]) for f in range(2)], STRONG, 0)
    o = ob.cpu().numpy()
    for f in range(2):
        check(o[f, 2:2 + H, 8:8 + W], refs[f], f"frame {f}")
    mask = np.ones(o.shape, bool)
    mask[:, 2:2 + H, 8:8 + W] = False
    assert np.all(o[mask] == 7)
    assert s.batch_sums(2) == sums
    s.close()


@pytest.mark.parametrize("W,H", [(1925, 30), (13, 8), (61, 21)])
def test_general_sizes_padded_to_a_16_byte_pitch(W, H):
    """Padded width W4 % 16 == 8: the gathered scratch gets a 16-byte row pitch
    and the units run on the step kernel with strided tensor maps."""
    s = Sharpener()
    imgs = np.ascontiguousarray(synth.frames(2, W + 3, H + 3, "natural", seed=synth.BASE_SEED + 3 * W)[:, :H, :W])
    s.set_profiling(True)
    out = s.run_ex(torch.from_numpy(imgs).cuda(), STRONG)
    torch.cuda.synchronize()
    assert s.kernel_times().step_launches == 1
    refs, sums = ref_units(list(imgs), STRONG, 0)
    for f in range(2):
        check(out[f].cpu().numpy(), refs[f], f"frame {f}")
    assert s.batch_sums(2) == sums
    s.close()


@pytest.mark.parametrize("W,H", [(1928, 40), (24, 16), (3848, 12)])
def test_dense_width_8_mod_16_runs_on_the_step_kernel(W, H):
    """sharp_run_batch on device frames with W % 16 == 8 (not a TMA row stride
    in place): through a 16-byte-pitch scratch onto the step kernel."""
    s = Sharpener()
    imgs = synth.frames(3, W, H, "natural", seed=synth.BASE_SEED + W + H)
    d = torch.from_numpy(imgs).cuda()
    s.set_profiling(True)
    out = s.run_batch(d, STRONG)
    torch.cuda.synchronize()
    assert s.kernel_times().step_launches == 1
    ref, sums = oracle.sharpen_batch(imgs, *STRONG)
    check(out.cpu().numpy(), ref, f"{W}x{H}")
    assert s.batch_sums(3) == [int(x) for x in sums]
    s.close()
