"""Long chains of asynchronous calls on one context with no synchronisation
in between (the per-call counter zeroing and the scratch reuse must be
ordered on the stream): same shape, changing batch sizes and geometries,
every path interleaved on the same context, host-buffer calls in between, a
stream switch, and a user kernel writing the input right before each launch
-- all bit-exact vs the oracle, with the exact per-frame sums."""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_icpp_fanjzac15_b200 import (SHARP_PATH_AUTO, SHARP_PATH_FUSED, SHARP_PATH_RES, SHARP_PATH_STAGED,
                                            SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, Sharpener)

pytestmark = pytest.mark.gpu
PRM = (1.0, 0.5, 0.5, 2.0)


def _case(n, W, H, seed):
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + seed)
    ref, sums = oracle.sharpen_batch(imgs, *PRM)
    return torch.from_numpy(imgs).cuda(), ref, [int(x) for x in sums]


def test_back_to_back_same_shape():
    d, ref, sums = _case(2, 1920, 1080, 61)
    with Sharpener() as sh:
        sh.set_path(SHARP_PATH_STEP)
        outs = [torch.empty_like(d) for _ in range(20)]
        for o in outs:
            sh.enqueue_batch(d, o, PRM)
        torch.cuda.synchronize()
        for o in outs:
            assert np.array_equal(o.cpu().numpy(), ref)
        assert sh.batch_sums(2) == sums


def test_changing_shapes_and_paths():
    cases = [_case(1, 3840, 2160, 62), _case(5, 1280, 720, 63), _case(1, 512, 512, 64), _case(3, 1920, 1088, 65)]
    paths = [SHARP_PATH_STEP, SHARP_PATH_AUTO, SHARP_PATH_RES, SHARP_PATH_TWO_PASS, SHARP_PATH_FUSED,
             SHARP_PATH_STAGED]
    with Sharpener() as sh:
        pending = []
        for it in range(24):
            d, ref, sums = cases[it % len(cases)]
            path = paths[(it * 5) % len(paths)] if it % 3 == 0 else SHARP_PATH_STEP
            sh.set_path(path)
            o = torch.empty_like(d)
            sh.enqueue_batch(d, o, PRM)
            pending.append((o, ref))
        torch.cuda.synchronize()
        for o, ref in pending:
            assert np.array_equal(o.cpu().numpy(), ref)


def test_sync_and_host_calls_in_between():
    d, ref, sums = _case(1, 1920, 1080, 66)
    host = d.cpu().numpy()
    with Sharpener() as sh:
        sh.set_path(SHARP_PATH_STEP)
        for it in range(6):
            o = torch.empty_like(d)
            sh.enqueue_batch(d, o, PRM)
            if it % 2:
                out_h = sh.run_batch(host, PRM)  # host pipeline: zeroes the counters itself
                assert np.array_equal(out_h, ref)
            assert np.array_equal(o.cpu().numpy(), ref)
            assert sh.batch_sums(1) == sums


def test_stream_switch():
    d, ref, _ = _case(2, 1920, 1080, 67)
    with Sharpener() as sh:
        sh.set_path(SHARP_PATH_STEP)
        outs = []
        for it in range(8):
            if it % 3 == 0:
                st = torch.cuda.Stream()
                sh.set_stream(st)
            o = torch.empty_like(d)
            sh.enqueue_batch(d, o, PRM)
            outs.append(o)
        torch.cuda.synchronize()
        for o in outs:
            assert np.array_equal(o.cpu().numpy(), ref)


def test_producer_kernel_right_before_launch():
    """The input is produced by a torch kernel on the same stream immediately
    before each launch: griddepcontrol.wait must hold the step kernel until
    that kernel's writes are visible."""
    d, ref, _ = _case(1, 3840, 2160, 68)
    zero = torch.zeros_like(d)
    with Sharpener() as sh:
        sh.set_path(SHARP_PATH_STEP)
        st = torch.cuda.Stream()
        sh.set_stream(st)
        with torch.cuda.stream(st):
            buf = torch.empty_like(d)
            outs = []
            for _ in range(6):
                buf.copy_(zero)
                buf.add_(d)  # the real input, written right before the launch
                o = torch.empty_like(d)
                sh.enqueue_batch(buf, o, PRM)
                outs.append(o)
                buf = torch.empty_like(d)
        torch.cuda.synchronize()
        for o in outs:
            assert np.array_equal(o.cpu().numpy(), ref)
