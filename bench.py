#!/usr/bin/env python
"""Benchmark of the B200 sharpness pipeline (one JSON line on rank 0).

Workload (BASELINE.json configs[4], frame = configs[1]): batches of 1024
synthetic 1920x1080 8-bit frames, one process per GPU.  The frames are
independent units (each has its own pEdge mean), so the path partitions with
no collective on the data path: by default every rank sharpens its own 1024
frames ("scaling": "weak", the partitioned-path rule); --scaling strong
splits one 1024-frame batch over the ranks instead.  A step = the whole hot
path (pass 1: Sobel + reduction + LUTs; pass 2: fused downscale/upscale/
pError/Sobel/min-max/strength/preliminary/overshoot) over the batch; value =
all ranks' pixels / the slowest rank's step time.

  value  : Mpix/s, device-resident (inputs already in HBM), CUDA events on the
           launch stream, max over ranks.  The 2.1 GB batch is larger than the
           126 MB L2, so no L2 flush is needed between steps.
  e2e    : same metric through the public API with HOST (pinned) buffers:
           sharp_run_batch does H2D || compute || D2H itself.
  roofline: the dominant kernel (pass 2) -- algorithmic bytes 2 B/px (read
           the frame, write the result) / its average launch duration.
  cpu_baseline: the CPU oracle timed on a bounded sample (rank 0, N=1).

`--impl reference` times the CPU oracle (the reference arm of this tier).

`--workload bands` (not the driver's default line) times BASELINE configs[3]:
ONE --width x --height image (default 8K) row-band sharded over the N ranks
(bands.py: halo exchange by NCCL send/recv, one u64 all-reduce of the pEdge
partials, sharp_band_edge_sum / sharp_band_sharpen), bands device-resident.
"""
import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "megapixels/sec end-to-end sharpen (device-timed) and % of HBM roofline, 1/2/4/8 B200"
UNIT = "Mpix/s"
PARAMS = (1.0, 0.5, 0.5, 2.0)  # DESIGN.md R16 defaults
ALG_BYTES_PER_PX = 2.0         # compulsory: 1 B in + 1 B out


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


class ClockSampler:
    """Samples SM clock and clock-event reasons with NVML while running."""
    BITS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
            0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks"}

    def __init__(self, index, period=0.02):
        self.index, self.period = index, period
        self.samples, self.reasons = [], set()
        self.max_mhz = None
        self._stop = threading.Event()
        self.ok = True
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.ok = False

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for b, name in self.BITS.items():
                    if r & b:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# Test hook: SHARP_BENCH_SHARE_GPU=1 maps every rank onto the visible GPUs
# round-robin and uses gloo for the plumbing (NCCL refuses two ranks on one
# GPU), so the multi-rank code path can be exercised on a one-GPU box.  Never
# set for a measurement.
SHARE_GPU = os.environ.get("SHARP_BENCH_SHARE_GPU") == "1"


def dist_setup():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if SHARE_GPU:
        import torch
        local %= max(1, torch.cuda.device_count())
    return world, rank, local


def bind_to_gpu_numa_node(torch, local):
    """Pin this rank's threads to the CPUs of its GPU's NUMA node (before the
    pinned host buffers are first touched), so the e2e leg's H2D / D2H read
    and write NUMA-local memory.  Best effort: returns the node or None."""
    try:
        pr = torch.cuda.get_device_properties(local)
        bus = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
        node = int(open(f"/sys/bus/pci/devices/{bus}/numa_node").read())
        if node < 0:
            return None
        cpus = set()
        for part in open(f"/sys/devices/system/node/node{node}/cpulist").read().strip().split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        cpus &= os.sched_getaffinity(0)
        if cpus:
            os.sched_setaffinity(0, cpus)
            return node
    except (OSError, ValueError, AttributeError):
        pass
    return None


def init_group(torch, dist, local):
    if SHARE_GPU:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))


KERNEL_SOURCES = {  # the sources a kernel's SASS depends on (profiles are keyed on their hash)
    "step": ["kernels_tma.cu", "tma_common.cuh", "device_common.cuh", "kernels.h"],
    "res": ["kernels_res.cu", "tma_common.cuh", "device_common.cuh", "kernels.h"],
}


def kernel_source_hash(kind):
    import hashlib
    h = hashlib.sha256()
    for f in KERNEL_SOURCES[kind]:
        h.update(open(os.path.join(ROOT, "paper_conf_icpp_fanjzac15_b200", "csrc", f), "rb").read())
    return h.hexdigest()


def committed_profile(kind="step"):
    """The newest committed ncu capture summary of this kernel
    (profiles/<round>/traffic*.json), if it was taken from the CURRENT kernel
    sources (else None: a stale capture is not reported)."""
    import glob
    for f in sorted(glob.glob(os.path.join(ROOT, "profiles", "*", "traffic*.json")), reverse=True):
        try:
            t = json.load(open(f))
        except Exception:
            continue
        if t.get("kernel_kind", "step") != kind:
            continue
        if t.get("source_sha256") != kernel_source_hash(kind):
            return None
        t["_file"] = os.path.relpath(f, ROOT)
        return t
    return None


def traffic_per_launch(px_per_launch, kind="step"):
    """DRAM bytes (read + write) per launch of the dominant kernel, from the
    committed ncu --set full capture of this kernel (dram bytes per output
    pixel), scaled to this launch; None without a capture of the current
    kernel sources."""
    t = committed_profile(kind)
    return float(t["dram_bytes_per_px"]) * px_per_launch if t else None


def issue_profile(kind="step"):
    """Warp instructions per output pixel of the dominant kernel, from the
    committed capture of the current kernel sources, or None."""
    t = committed_profile(kind)
    return float(t["warp_instr_per_px"]) if t else None


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def issue_roofline(px_per_launch, k_avg_ms, sm_mhz, n_sms):
    """The binding resource: instruction issue.  Peak =
    4 warp-instructions per clock per SM (one per SMSP scheduler) at the SM
    clock measured during the timed region; achieved = the committed
    capture's warp-instructions per pixel x pixels per launch / the live
    launch duration."""
    wipp = issue_profile()
    if wipp is None or not sm_mhz:
        return None
    achieved = wipp * px_per_launch / (k_avg_ms * 1e-3) / 1e9
    peak = 4.0 * n_sms * sm_mhz * 1e6 / 1e9
    return {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gwarp-instr/s", "frac": achieved / peak,
            "warp_instr_per_px": wipp, "thread_instr_per_px": 32 * wipp,
            "peak_source": f"4 issue slots/clk/SM x {n_sms} SMs x measured SM clock (B200_PROFILING / B300_MICROARCH)"}


def cpu_oracle_rate(frames, threads):
    """Oracle Mpix/s on `frames` ([k,H,W]) with `threads` OpenMP threads."""
    import oracle
    t0 = time.perf_counter()
    oracle.sharpen_batch(frames, *PARAMS, threads=threads)
    dt = time.perf_counter() - t0
    return frames.size / dt / 1e6, dt


def run_reference(args, world, rank):
    """Reference arm of this tier: the CPU oracle, as it stands, on host cores."""
    if rank != 0:
        return
    import synth
    cores = len(os.sched_getaffinity(0))
    sample = args.ref_sample
    idx = list(range(0, args.frames, max(1, args.frames // sample)))[:sample]
    frames = np.stack([synth.image(args.width, args.height, "natural", seed=synth.BASE_SEED + 5 + i) for i in idx])
    for _ in range(args.warmup):
        cpu_oracle_rate(frames[:1], cores)
    rates, times = [], []
    for _ in range(args.steps):
        r, dt = cpu_oracle_rate(frames, cores)
        rates.append(r)
        times.append(dt)
    value = float(np.median(rates))
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": float(np.median(times) * 1e3),
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f32",
        "data": "synthetic", "config": workload_config(args, world),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": f"{len(idx)} of {args.frames} frames per step (every "
                                   f"{max(1, args.frames // sample)}th), OpenMP over frames"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(args, world):
    weak = getattr(args, "scaling", "weak") == "weak"
    if weak:
        wl = (f"{args.frames} x {args.width}x{args.height} u8 frames per GPU (BASELINE configs[4]'s batch on each "
              f"of {world} GPU(s); frame = configs[1])")
        par = f"independent frames, {args.frames} per GPU on {world} GPU(s), no collective on the data path"
    else:
        wl = f"{args.frames} x {args.width}x{args.height} u8 frames (BASELINE configs[4]; frame = configs[1])"
        par = f"frames split over {world} GPU(s), no collective on the data path"
    return {"workload": wl,
            "frames": args.frames * (world if weak else 1), "frames_per_gpu": args.frames if weak else None,
            "width": args.width, "height": args.height,
            "params": dict(zip(["amount", "gamma", "osc_gain", "osc_scale"], PARAMS)),
            "parallelism": par,
            "l2": "batch (2.1 GB in + out) > 126 MB L2: no flush needed between steps"}


def run_bands_workload(args, world, rank, local):
    """One image, row bands over the ranks (BASELINE configs[3])."""
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_icpp_fanjzac15_b200 import Sharpener, shard
    from paper_conf_icpp_fanjzac15_b200.bands import band_rows, exchange_halos, sharpen_band

    torch.cuda.set_device(local)
    if world > 1:
        init_group(torch, dist, local)
    W, H = args.width, args.height
    r0, r1 = band_rows(H, world, rank)
    img = synth.image(W, H, "natural", seed=synth.BASE_SEED + 3)  # every rank generates, keeps its rows
    h_own = torch.from_numpy(img[r0:r1].copy()).pin_memory()
    h_out = torch.empty_like(h_own).pin_memory()
    own = h_own.to(f"cuda:{local}")
    out = torch.empty_like(own)
    # Rotate over enough input copies (>= 256 MB) that no step finds its
    # input in the 126 MB L2 left by the previous steps.
    ncopy = max(1, -(-(256 << 20) // own.numel()))
    owns = [own] + [own.clone() for _ in range(ncopy - 1)]
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    sh = Sharpener(device=local)
    sh.set_stream(stream)
    if args.exchange in ("p2p", "fused", "one"):
        # peer-memory exchange: halos and the u64 partials stored straight
        # into the neighbours' / all ranks' windows (CUDA IPC over NVLink),
        # epoch-flagged; no NCCL on the data path.  "fused": the partials'
        # all-reduce runs inside the band's single step-kernel launch.
        from paper_conf_icpp_fanjzac15_b200.bands import P2PBand
        p2p = P2PBand(sh, W, H)
        epoch = [0]
        # ranks sharing one GPU (the SHARP_BENCH_SHARE_GPU test hook) bound
        # their persistent grids so that every band's launch can run
        cap = 0
        if SHARE_GPU and world > torch.cuda.device_count():
            cap = max(1, (2 * torch.cuda.get_device_properties(local).multi_processor_count) // world)

        def step(src, dst):
            p2p.own.copy_(src)  # this image's rows into the window (the NCCL path copies them too)
            epoch[0] += 1
            if args.exchange == "one":
                p2p.step_one_launch(epoch[0], dst, PARAMS, grid_cap=cap)
            elif args.exchange == "fused":
                p2p.step_fused(epoch[0], dst, PARAMS, grid_cap=cap)
            else:
                p2p.step(epoch[0], dst, PARAMS)
    else:
        def step(src, dst):
            band = exchange_halos(src, H, r0, r1)
            sharpen_band(sh, band, W, H, r0, r1, PARAMS, out=dst)

    for _ in range(args.warmup):
        step(own, out)
    torch.cuda.synchronize()
    sh.set_profiling(True)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    shard.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for i in range(args.steps):
            step(owns[i % ncopy], out)
        ev1.record(stream)
        torch.cuda.synchronize()
    shard.barrier()
    ms_step = shard.max_over_ranks(ev0.elapsed_time(ev1) / args.steps, device=f"cuda:{local}")
    kt = sh.kernel_times()
    sh.set_profiling(False)
    value = W * H / (ms_step * 1e-3) / 1e6
    # dominant kernel: the band's pass-2 launch (reads its rows + halo, writes
    # its rows), or the fused band launch (pass 1 + all-reduce + pass 2)
    if args.exchange in ("fused", "one"):
        k_avg = kt.step_ms / max(1, kt.step_launches)
        px = kt.pixels / max(1, kt.step_launches)
    else:
        k_avg = kt.pass2_ms / max(1, kt.pass2_launches)
        px = kt.pixels / max(1, kt.pass2_launches)
    pk, pk_src = peaks()
    peak = float(pk["hbm_gbs"])
    achieved = ALG_BYTES_PER_PX * px / (k_avg * 1e-3) / 1e9
    parity = None
    if rank == 0 and not args.no_cpu:
        import oracle
        ref, _, _ = oracle.sharpen(img, *PARAMS)
        parity = {"rows_checked": r1 - r0, "mismatched_pixels": int((out.cpu().numpy() != ref[r0:r1]).sum())}
    # e2e: this rank's rows from pinned host memory, result back to pinned host memory
    t_e2e = []
    for _ in range(max(args.e2e_steps, 0)):
        shard.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        own.copy_(h_own, non_blocking=True)
        step(own, out)
        h_out.copy_(out, non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        t_e2e.append(e0.elapsed_time(e1))
    e2e_ms = shard.max_over_ranks(float(np.median(t_e2e)), device=f"cuda:{local}") if t_e2e else float("nan")
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"one {W}x{H} u8 image, row bands over {world} GPU(s) (BASELINE configs[3])",
                       "width": W, "height": H, "bands": world, "exchange": args.exchange,
                       "parallelism": ("row bands: 4-row halo exchange (NCCL send/recv) + u64 all-reduce"
                                       if args.exchange == "nccl" else
                                       "row bands: halo rows + u64 partials stored into peer windows "
                                       "(CUDA IPC / NVLink, epoch flags), no NCCL on the data path" +
                                       {"fused": "; pass 1 + all-reduce + pass 2 in one launch per band",
                                        "one": "; halo push + pass 1 + all-reduce + pass 2 in ONE launch per band"}
                                       .get(args.exchange, "")),
                       "l2": f"inputs rotated over {ncopy} copies (>= 256 MB > 126 MB L2)"},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": None,
                         "kernel": ("step_kernel (fused band)" if args.exchange in ("fused", "one")
                                    else "step_kernel (band pass 2)"),
                         "peak_source": pk_src, "alg_bytes_per_px": ALG_BYTES_PER_PX, "px_per_launch": px,
                         "kernel_avg_ms": k_avg, "pass1_avg_ms": kt.pass1_ms / max(1, kt.pass1_launches)},
            "e2e": {"value": W * H / (e2e_ms * 1e-3) / 1e6, "unit": UNIT, "h2d_bytes_per_step": W * H,
                    "d2h_bytes_per_step": W * H, "ms_per_step": e2e_ms,
                    "api": "bands.sharpen_band (pinned host rows -> device -> pinned host)"},
            # per band: [halo] + step(pass 1) + finish + [all-reduce] + arm + step(pass 2)
            "gpu_launches": {"p2p": 6, "fused": 2, "one": 1, "nccl": 4}[args.exchange] * args.steps,
            "clocks": clk.summary(),
            "cpu_baseline": None,
            "parity": parity,
        }
        print(json.dumps(line), flush=True)
    sh.close()
    if world > 1:
        dist.destroy_process_group()


# Compulsory HBM bytes per output pixel of the staged base design (every
# stage materialised): K1 1 + 1/4, K3 1/4 + 4, K4 1 + 2,
# K5 2, K6 2 + 8, K7 1 + 4 + 8 + 1.
STAGED_BYTES_PER_PX = {"downscale": 1.25, "border": 0.0, "center": 4.25, "sobel": 3.0, "reduction": 2.0,
                       "strength": 10.0, "sharpness": 14.0}


def run_ladder_workload(args, world, rank, local):
    """The optimisation ladder (sec. V, Fig. 12 / Fig. 14)
    on BASELINE configs[2] (4K frames, "kernel-fusion roofline study"): the
    paper's staged base design (one kernel per stage, the Fig. 13 per-stage
    breakdown), then one optimisation per rung -- fusion, the strength table,
    vectorisation / data reuse, the persistent TMA kernel, the TMEM-resident
    pEdge -- each timed on the same device-resident batch (> L2), all
    bit-identical; plus the optimised kernel's per-stage instruction shares
    (the Fig. 13(c) analogue) from a committed capture."""
    import torch

    import synth
    from paper_conf_icpp_fanjzac15_b200 import (SHARP_PATH_FUSED, SHARP_PATH_FUSED_EXP, SHARP_PATH_RES,
                                                SHARP_PATH_STAGED, SHARP_PATH_STEP, SHARP_PATH_TWO_PASS, Sharpener)

    if world > 1:
        if rank == 0:
            print(json.dumps({"workload": "ladder", "skipped": "single-GPU study"}))
        return
    torch.cuda.set_device(local)
    W, H, n = args.width, args.height, args.frames
    imgs = synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 2)
    d_in = torch.from_numpy(imgs).cuda()
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    pk, pk_src = peaks()
    peak = float(pk["hbm_gbs"])
    ladder = [("staged (paper base: 7 kernels per frame, every stage in HBM, per-pixel f64 exponentiation)",
               SHARP_PATH_STAGED, 34.5),
              ("+ fusion (scalar: 1 px / thread, 4 kernels per frame, per-pixel f64 exponentiation)",
               SHARP_PATH_FUSED_EXP, 3.25),
              ("+ strength table (the exponentiations once per frame from the reduced mean)", SHARP_PATH_FUSED, 3.25),
              ("+ vectorisation / data reuse (8 px / lane f16x2 SIMD, shuffled halos, 2 kernels per chunk)",
               SHARP_PATH_TWO_PASS, 3.0),
              ("+ persistent TMA kernel (whole batch in ONE launch, in-kernel reduction barrier and tables)",
               SHARP_PATH_STEP, ALG_BYTES_PER_PX),
              ("+ TMEM-resident pEdge (pass 2 reuses pass 1's Sobel; DRAM ~2 B/px)", SHARP_PATH_RES, ALG_BYTES_PER_PX)]
    rungs, outs = [], {}
    for name, path, alg in ladder:
        sh = Sharpener(device=local)
        sh.set_stream(stream)
        sh.set_path(path)
        d_out = torch.empty_like(d_in)
        for _ in range(args.warmup):
            sh.enqueue_batch(d_in, d_out, PARAMS)
        torch.cuda.synchronize()
        sh.set_profiling(True)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for _ in range(args.steps):
            sh.enqueue_batch(d_in, d_out, PARAMS)
        ev1.record(stream)
        torch.cuda.synchronize()
        ms = ev0.elapsed_time(ev1) / args.steps
        rung = {"path": name, "ms_per_step": ms, "mpix_s": n * W * H / (ms * 1e-3) / 1e6,
                "launches_per_step": sh.stats().kernels, "alg_bytes_per_px": alg}
        if path == SHARP_PATH_STAGED:
            st = sh.stage_times()
            tot = sum(st.values()) or 1.0
            rung["stages"] = {k: {"ms_per_frame": v / (args.steps * n), "share": v / tot,
                                  "alg_bytes_per_px": STAGED_BYTES_PER_PX[k],
                                  "achieved_gbs": (STAGED_BYTES_PER_PX[k] * W * H / (v / (args.steps * n) * 1e-3)
                                                   / 1e9) if v > 0 and STAGED_BYTES_PER_PX[k] else None}
                              for k, v in st.items()}
        elif path == SHARP_PATH_TWO_PASS:
            kt = sh.kernel_times()
            rung["pass1_share"] = kt.pass1_ms / max(1e-9, kt.pass1_ms + kt.pass2_ms)
        rung["hbm_frac_alg2"] = ALG_BYTES_PER_PX * n * W * H / (ms * 1e-3) / 1e9 / peak
        sh.set_profiling(False)
        outs[path] = d_out
        rungs.append(rung)
        sh.close()
    identical = all(bool(torch.equal(o, outs[SHARP_PATH_STEP])) for o in outs.values())
    parity = None
    if not args.no_cpu:
        import oracle
        ref, _ = oracle.sharpen_batch(imgs[:1], *PARAMS)
        parity = {"frames_checked": 1, "mismatched_pixels": int((outs[SHARP_PATH_STEP][:1].cpu().numpy() != ref).sum())}
    base = rungs[0]["ms_per_step"]
    for i, r in enumerate(rungs):
        r["speedup_vs_staged"] = base / r["ms_per_step"]
        r["speedup_vs_previous"] = rungs[i - 1]["ms_per_step"] / r["ms_per_step"] if i else 1.0
    # Fig. 13(c) analogue for the optimised kernel: its instruction share per
    # stage (SASS attribution of a committed ncu capture of the current sources)
    shares = None
    try:
        import glob
        f = sorted(glob.glob(os.path.join(ROOT, "profiles", "*", "stage_shares.json")))[-1]
        t = json.load(open(f))
        if t.get("source_sha256") == kernel_source_hash("step"):
            shares = {"source": os.path.relpath(f, ROOT), "thread_instr_per_px": t["thread_instr_per_px"],
                      "shares": t["shares"]}
    except (IndexError, OSError, ValueError, KeyError):
        pass
    line = {"metric": METRIC, "workload": "ladder", "unit": UNIT, "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{n} x {W}x{H} u8 frames (BASELINE configs[2]: kernel-fusion roofline study)",
                       "l2": f"batch {2 * n * W * H / 1e6:.0f} MB in + out > 126 MB L2"},
            "hbm_peak_gbs": peak, "peak_source": pk_src, "ladder": rungs, "paths_identical": identical,
            "step_kernel_stage_shares": shares, "parity": parity}
    print(json.dumps(line), flush=True)


def free_port():
    import socket
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def self_launch(args):
    """`--gpus N` (N > 1) outside torchrun: re-run this command as N ranks under
    torch.distributed.run (one process per GPU, rendezvous on 127.0.0.1), the
    launch the driver uses; returns the exit code.  Fails loudly when N
    exceeds the visible GPUs (the reference arm runs on host cores and the
    SHARP_BENCH_SHARE_GPU test hook maps ranks onto the visible GPUs)."""
    import subprocess
    if args.impl != "reference" and not SHARE_GPU:
        import torch
        n = torch.cuda.device_count()
        if args.gpus > n:
            print(f"bench.py: --gpus {args.gpus} but only {n} GPU(s) are visible", file=sys.stderr)
            return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.run(cmd, env=dict(os.environ, OMP_NUM_THREADS=os.environ.get("OMP_NUM_THREADS", "1"))).returncode


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--frames", type=int, default=1024,
                    help="batch size: per GPU with --scaling weak, in total with --scaling strong")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak (default): every rank sharpens its own --frames frames (independent units, the "
                         "partitioned-path rule); strong: --frames split over the ranks")
    ap.add_argument("--width", type=int, default=1920)
    ap.add_argument("--height", type=int, default=1080)
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-sample", type=int, default=128)
    ap.add_argument("--ref-sample", type=int, default=16)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--workload", default="batch", choices=["batch", "bands", "ladder"])
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "p2p", "fused", "one"],
                    help="bands workload: NCCL send/recv + all-reduce, the peer-memory exchange kernels, or "
                         "the peer-memory halo push + ONE fused launch per band (all-reduce inside), or "
                         "one launch per band with the halo push inside too")
    args = ap.parse_args()
    if args.gpus < 1:
        ap.error("--gpus must be >= 1")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(self_launch(args))
    world, rank, local = dist_setup()
    if "WORLD_SIZE" in os.environ and world != args.gpus and rank == 0:
        print(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}; measuring {world} rank(s)", file=sys.stderr)
    if args.workload == "bands" and args.width == 1920 and args.height == 1080:
        args.width, args.height = 7680, 4320  # configs[3]: 8K
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    if args.workload == "bands":
        run_bands_workload(args, world, rank, local)
        return
    if args.workload == "ladder":
        if args.width == 1920 and args.height == 1080:
            args.width, args.height = 3840, 2160  # configs[2]: 4K
        if args.frames == 1024:
            args.frames = 32
        run_ladder_workload(args, world, rank, local)
        return

    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_icpp_fanjzac15_b200 import Sharpener
    from paper_conf_icpp_fanjzac15_b200 import shard
    from paper_conf_icpp_fanjzac15_b200.binding import _params as sharp_params_of

    torch.cuda.set_device(local)
    if world > 1:
        init_group(torch, dist, local)
    W, H = args.width, args.height
    numa = bind_to_gpu_numa_node(torch, local) if world > 1 else None
    if args.scaling == "weak":
        start, n = rank * args.frames, args.frames
    else:
        start, n = shard.frame_range(args.frames, world, rank)
    fb = W * H
    # Inputs: pinned host (for e2e) and a device copy (device-resident value).
    h_in = torch.empty((n, H, W), dtype=torch.uint8).pin_memory()
    # (torchrun sets OMP_NUM_THREADS=1: give each rank its share of the cores for input generation)
    gen_threads = max(1, len(os.sched_getaffinity(0)) // max(1, world))
    synth.frames(n, W, H, "natural", seed=synth.BASE_SEED + 5 + start, out=h_in.numpy(), threads=gen_threads)
    h_out = torch.empty_like(h_in).pin_memory()
    d_in = h_in.to(f"cuda:{local}")
    d_out = torch.empty_like(d_in)
    # A dedicated (non-default) stream: the library launches on it and the
    # CUDA events below are recorded on it.
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    sh = Sharpener(device=local)
    sh.set_stream(stream)

    barrier = shard.barrier

    def max_over_ranks(x):
        return shard.max_over_ranks(x, device=f"cuda:{local}")

    # ---- device-resident timed region
    prm = sharp_params_of(PARAMS)  # marshalled once: the loop times the library, not ctypes
    for _ in range(args.warmup):
        sh.enqueue_batch(d_in, d_out, prm)
    torch.cuda.synchronize()
    launches_per_step = sh.stats().kernels
    # Per-launch kernel events ride inside the timed region for batches; for a
    # latency-sized step (a few frames, ~20 us) two extra event records per
    # launch would be a visible part of the step, so there the kernel times
    # come from a second, profiled pass over the same steps.
    latency_regime = n <= 8
    sh.set_profiling(not latency_regime)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            sh.enqueue_batch(d_in, d_out, prm)
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier()
    ms_step = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
    if latency_regime:
        sh.set_profiling(True)
        for _ in range(args.steps):
            sh.enqueue_batch(d_in, d_out, prm)
        torch.cuda.synchronize()
    kt = sh.kernel_times()
    sh.set_profiling(False)
    # Latency regime: the same calls captured in a CUDA graph and replayed
    # ("graph of 1000 reps / 1000"): the device cost of a call
    # without the host's per-call launch work.
    graph = None
    if latency_regime:
        try:
            reps = 200
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                for _ in range(reps):
                    sh.enqueue_batch(d_in, d_out, prm)
            g.replay()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(5):
                g.replay()
            e1.record(stream)
            torch.cuda.synchronize()
            graph = {"reps_per_graph": reps, "ms_per_call": e0.elapsed_time(e1) / (5 * reps)}
        except Exception as ex:  # capture is an extra, never a failure of the run
            graph = {"unavailable": f"{type(ex).__name__}: {ex}"[:200]}
    # ---- strong scaling beside the weak line (BASELINE configs[4]: ONE batch
    # of --frames frames split over the ranks): same kernels, each rank's
    # share of the batch, the slowest rank's time
    strong = None
    if world > 1 and args.scaling == "weak":
        _, sn = shard.frame_range(args.frames, world, rank)
        sh.enqueue_batch(d_in[:sn], d_out[:sn], prm)
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            sh.enqueue_batch(d_in[:sn], d_out[:sn], prm)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ms_strong = max_over_ranks(e0.elapsed_time(e1) / args.steps)
        strong = {"scaling": "strong", "value": args.frames * fb / (ms_strong * 1e-3) / 1e6, "unit": UNIT,
                  "ms_per_step": ms_strong, "frames_total": args.frames, "frames_per_gpu": sn,
                  "workload": f"one batch of {args.frames} x {W}x{H} frames split over {world} GPU(s)"}
    total_px = args.frames * fb * (world if args.scaling == "weak" else 1)  # all ranks' frames
    value = total_px / (ms_step * 1e-3) / 1e6

    # dominant kernel: the step kernel (TMA path: pass 1 of chunk c+1 fused
    # with pass 2 of chunk c) or, on the generic path, pass 2.
    if kt.step_launches:
        kname = "step_kernel (pass 1 of chunk c+1 + pass 2 of chunk c)"
        k_ms, k_launches, k_share = kt.step_ms, kt.step_launches, 1.0
    else:
        kname = "sharpen_kernel (pass 2)"
        k_ms, k_launches = kt.pass2_ms, kt.pass2_launches
        k_share = kt.pass2_ms / max(1e-9, kt.pass1_ms + kt.pass2_ms)
    px_per_launch = kt.pixels / max(1, k_launches)
    k_avg_ms = k_ms / max(1, k_launches)
    pk, pk_src = peaks()
    peak = float(pk["hbm_gbs"])
    achieved = ALG_BYTES_PER_PX * px_per_launch / (k_avg_ms * 1e-3) / 1e9
    step_achieved = ALG_BYTES_PER_PX * total_px / world / (ms_step * 1e-3) / 1e9

    # ---- parity spot check of this run's outputs (two frames, vs the oracle)
    parity = None
    if rank == 0 and not args.no_cpu:
        import oracle
        chk = [0, n - 1]
        ref, _ = oracle.sharpen_batch(h_in.numpy()[chk], *PARAMS)
        got = d_out[chk].cpu().numpy()
        parity = {"frames_checked": len(chk), "mismatched_pixels": int((got != ref).sum())}

    # ---- e2e through the public API with host (pinned) buffers
    sh.set_stream(None)
    t_e2e = []
    if args.e2e_steps > 0:
        sh.run_batch(h_in, PARAMS, h_out)  # warm the staging buffers
        barrier()
        for _ in range(args.e2e_steps):
            barrier()
            t0 = time.perf_counter()
            sh.run_batch(h_in, PARAMS, h_out)
            t_e2e.append(time.perf_counter() - t0)
    e2e_ms = max_over_ranks(float(np.median(t_e2e)) * 1e3) if t_e2e else float("nan")
    e2e_value = total_px / (e2e_ms * 1e-3) / 1e6

    # ---- CPU oracle baseline (rank 0, N=1 only)
    cpu = None
    paper_context = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cores = len(os.sched_getaffinity(0))
        idx = list(range(0, n, max(1, n // args.cpu_sample)))[:args.cpu_sample]
        rate, dt = cpu_oracle_rate(h_in.numpy()[idx], cores)
        cpu = {"value": rate, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
               "sample": f"{len(idx)} of {n} frames (every {max(1, n // args.cpu_sample)}th), "
                         f"{dt:.1f} s wall on {cores} threads"}
        # The paper's headline is end-to-end GPU (with transfers) vs a
        # SEQUENTIAL CPU program (L376, L396-L398): the analogous ratio here is
        # e2e vs the oracle on one thread (4 sampled frames).  Context only:
        # the oracle is deliberately plain, not the paper's optimised C.
        rate1, dt1 = cpu_oracle_rate(h_in.numpy()[idx[:4]], 1)
        cpu["one_thread"] = {"value": rate1, "unit": UNIT, "sample": f"{min(4, len(idx))} frames, {dt1:.1f} s"}
        paper_context = {"paper_gpu_vs_sequential_cpu_e2e": "10.7-69.3x (FirePro W8000 vs i5-3470, 256^2..4096^2; "
                                                            "PAPER.md L396-L398, L666)",
                         "this_run_e2e_vs_oracle_one_thread": e2e_value / rate1,
                         "this_run_device_vs_oracle_one_thread": value / rate1}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": workload_config(args, world),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic_per_launch(px_per_launch),
                         "traffic_source": ((committed_profile() or {}).get("_file") or
                                            "none: no ncu capture of the current kernel sources is committed"),
                         "kernel": kname, "peak_source": pk_src,
                         "alg_bytes_per_px": ALG_BYTES_PER_PX, "px_per_launch": px_per_launch,
                         "kernel_avg_ms": k_avg_ms, "kernel_launches": k_launches,
                         "kernel_share_of_step": k_share, "step_frac": step_achieved / peak,
                         "kernel_events": ("a second, profiled pass over the same steps (latency regime)"
                                           if latency_regime else "per launch, inside the timed region")},
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": total_px,
                    "d2h_bytes_per_step": total_px, "ms_per_step": e2e_ms,
                    "api": "sharp_run_batch(pinned host in, pinned host out)"},
            "issue_roofline": issue_roofline(px_per_launch, k_avg_ms, clk.summary().get("sm_mhz"),
                                             torch.cuda.get_device_properties(local).multi_processor_count),
            "gpu_launches": launches_per_step * args.steps,
            "strong_scaling": strong,
            "clocks": clk.summary(),
            "cpu_baseline": cpu,
            "paper_context": paper_context,
            "parity": parity,
            "cuda_graph": graph,
            "host_numa_binding": "ranks pinned to their GPU's NUMA node" if numa is not None else None,
        }
        print(json.dumps(line), flush=True)
    sh.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
