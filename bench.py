#!/usr/bin/env python
"""Benchmark of the star-image render path (BASELINE.json metric) -- one JSON line on rank 0.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config T] [--method tiled|atomic]

A step is one frame: the whole hot path (per-star prep + binning + CSR + tile accumulation) over one synthetic
catalogue resident in HBM, written to a device-resident fp32 image.  N=1 renders the north-star frame T (4096x4096,
1M uniform stars, R=15, sigma=2.5).  Under torchrun (N>1) the job is weak-scaled: the frame is 4096 wide and 4096*N
tall with N*1M stars replicated on every rank; each step every rank routes the catalogue to its 4096-row band on the
device (starsim_route_band), renders the band and the bands are assembled with one NCCL
all-gather (STARSIM_EXCHANGE=fused: the peer-memory exchange fused into the tile epilogue), all inside the step.
Every line also carries `strong_C5`: the C5 frame (16384^2, 10M stars) on 1 GPU and split over the N ranks (render,
exchange and frame times, efficiencies, NCCL algbw/busbw, bitwise validation of the assembled frame).

Timing: W untimed warm-up steps; the L2 (126 MB) is flushed by writing a 256 MiB buffer before every step (the frame's
79 MB of inputs+image would otherwise stay L2-resident); each step is bracketed by CUDA events on the render stream;
barrier + synchronize on both sides of the timed region; max over ranks.  `e2e` repeats the step through the same
C-ABI call with the catalogue copied in from pinned host memory and the image copied back, inside the timed region.
`roofline` is for the dominant kernel (k_tile), timed live with the library's per-kernel CUDA events.
`cpu_baseline` / --impl reference time the fp64 oracle on the host cores (bounded sample).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "star-pixel updates/s and frames/s at 1/2/4/8 B200; % of FP32/SFU roofline"
UNIT = "star-pixel updates/s"
FLUSH_BYTES = 256 << 20


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="T")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="N > 1: weak = a W x (H N) frame with N n stars, one H-row band per rank (default); strong = "
                         "the --config frame itself split into N bands (the north star's C5 target: --config C5)")
    ap.add_argument("--method", default="tiled", choices=["tiled", "atomic"])
    ap.add_argument("--tile-kernel", default="auto", choices=["auto", "lists", "sb", "ws", "t8"],
                    help="starsim_set_tile_kernel mode (A/B comparisons; the default is the product path)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-strong", action="store_true", help="skip the strong_C5 record (C5 frame split over N bands)")
    ap.add_argument("--no-wide", action="store_true", help="skip the wide-ROI record (C4 at R = 63)")
    return ap.parse_args()


# ------------------------------------------------------------------------------------------------ roofline model
def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured (MEASURED_PEAKS.json)"
    return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback (B200_PROFILING.md)"


def fp32_sfu_peak_updates(sm_mhz, U, E, sms=148):
    """Roofline rate of the separable-PSF work: per SM per clock 128 FP32 FMA (measured
    126-128, bench_micro) and 16 MUFU.EX2 (measured 16.0).  T* = max(U / P_fma, E / P_mufu); peak = U / T*."""
    f = sm_mhz * 1e6
    p_fma = sms * 128 * f
    p_mufu = sms * 16 * f
    t_star = max(U / p_fma, E / p_mufu)
    return U / t_star, t_star


# ------------------------------------------------------------------------------------------------ clocks (NVML)
class ClockSampler:
    def __init__(self, index=0, period=0.005):
        self.samples, self.reasons, self.period, self.index = [], set(), period, index
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)

    def _run(self):
        nv = self.nv
        names = {getattr(nv, k): k for k in dir(nv) if k.startswith("nvmlClocksEventReason") or
                 k.startswith("nvmlClocksThrottleReason")}
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h) if hasattr(
                    nv, "nvmlDeviceGetCurrentClocksEventReasons") else nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for bit, name in names.items():
                    if isinstance(bit, int) and bit and (r & bit) == bit and bit not in (0xFFFFFFFFFFFFFFFF,):
                        if "None" in name or "All" in name or "Unknown" in name:
                            continue
                        self.reasons.add(name.replace("nvmlClocksEventReason", "").replace(
                            "nvmlClocksThrottleReason", ""))
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "note": "nvml unavailable"}
        hi = [s for s in self.samples if s > 0.5 * max(self.samples)]
        return {"sm_mhz": statistics.median(hi), "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


# ------------------------------------------------------------------------------------------------ workload
def workload(cfg_name, world, rank, scaling="weak"):
    import synth
    cfg = synth.CONFIGS[cfg_name]
    if world == 1 or scaling == "strong":
        return cfg, cfg.field(), cfg.H, (0, cfg.H)
    # weak scaling: frame W x (H*world), world*n stars; every rank holds the full catalogue (replicated)
    H = cfg.H * world
    big = synth.Config(f"{cfg.name}x{world}", cfg.W, H, cfg.n * world, cfg.R, cfg.sigma, cfg.kind, cfg.seed)
    return big, big.field(), H, None


def units_of(f, W, H, R):
    """U, E over the frame with the exact per-star clipping of the method (numpy, same rules as the oracle)."""
    import numpy as np
    x, y, m = (a.astype(np.float64) for a in (f.x, f.y, f.mag))
    ok = np.isfinite(x) & np.isfinite(y) & np.isfinite(m)
    fx = np.floor(x)
    if R % 2:
        lx = fx + (x >= fx + 0.5) - (R - 1) // 2
        fy = np.floor(y)
        ly = fy + (y >= fy + 0.5) - (R - 1) // 2
    else:
        lx = fx + 1 - R // 2
        ly = np.floor(y) + 1 - R // 2
    w = np.minimum(lx + R - 1, W - 1) - np.maximum(lx, 0) + 1
    h = np.minimum(ly + R - 1, H - 1) - np.maximum(ly, 0) + 1
    ok &= (w > 0) & (h > 0)
    return int((w * h)[ok].sum()), int((w + h)[ok].sum())


# ------------------------------------------------------------------------------------------------ CPU baseline
def cpu_model():
    """The host CPU model name (lscpu / /proc/cpuinfo) for the baseline's context."""
    try:
        for line in open("/proc/cpuinfo"):
            if line.lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    try:
        import subprocess
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.strip().lower().startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:  # noqa: BLE001
        pass
    return None


def _oracle_rate(f, W, H, cfg, A, threads, budget_s):
    """U/s of the fp64 oracle on a prefix of the catalogue sized for ~budget_s on `threads` threads."""
    import oracle
    import synth
    n_cal = max(1000, f.n // 500)
    t0 = time.perf_counter()
    oracle.render(f.x[:n_cal], f.y[:n_cal], f.mag[:n_cal], W, H, cfg.sigma, cfg.R, A, threads=threads)
    dt = time.perf_counter() - t0
    n_s = int(min(f.n, max(n_cal, n_cal * budget_s / max(dt, 1e-6))))
    t0 = time.perf_counter()
    oracle.render(f.x[:n_s], f.y[:n_s], f.mag[:n_s], W, H, cfg.sigma, cfg.R, A, threads=threads)
    dt = time.perf_counter() - t0
    U, _ = units_of(synth.Field(f.x[:n_s], f.y[:n_s], f.mag[:n_s]), W, H, cfg.R)
    return U / dt, n_s, dt


def cpu_baseline(cfg, f, W, H, budget_s=12.0):
    """The fp64 oracle as it stands on all host cores, and on one core, each on a prefix of the catalogue sized for
    ~budget_s."""
    import synth
    threads = os.cpu_count() or 1
    A = synth.bench_gain(cfg.sigma)
    v, n_s, dt = _oracle_rate(f, W, H, cfg, A, threads, budget_s)
    v1, n1, dt1 = _oracle_rate(f, W, H, cfg, A, 1, budget_s * 0.75)
    return {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"first {n_s} of {f.n} stars of the same frame ({W}x{H}, R={cfg.R}), fp64 oracle, "
                      f"{threads} pthreads over row bands, {dt:.2f} s wall (includes zeroing the fp64 image)",
            "seconds": dt,
            "single_thread": {"value": v1, "unit": UNIT, "cores": 1,
                              "sample": f"first {n1} of {f.n} stars, 1 thread, {dt1:.2f} s wall"}}


# ------------------------------------------------------------------------------------------------ reference arm
def run_reference(args, world, rank):
    if rank != 0:
        return
    import oracle
    import synth
    cfg, f, H, _ = workload(args.config, 1, 0)
    W = cfg.W
    A = synth.bench_gain(cfg.sigma)
    threads = os.cpu_count() or 1
    total_budget = 150.0
    per_step = total_budget / max(1, args.steps + args.warmup)
    n_cal = max(1000, f.n // 500)
    t0 = time.perf_counter()
    oracle.render(f.x[:n_cal], f.y[:n_cal], f.mag[:n_cal], W, H, cfg.sigma, cfg.R, A, threads=threads)
    dt = time.perf_counter() - t0
    n_s = int(min(f.n, max(n_cal, n_cal * per_step / max(dt, 1e-6))))
    sub = synth.Field(f.x[:n_s], f.y[:n_s], f.mag[:n_s])
    U, _ = units_of(sub, W, H, cfg.R)
    for _ in range(args.warmup):
        oracle.render(sub.x, sub.y, sub.mag, W, H, cfg.sigma, cfg.R, A, threads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.render(sub.x, sub.y, sub.mag, W, H, cfg.sigma, cfg.R, A, threads=threads)
        times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    value = U / (ms * 1e-3)
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": f"{cfg.name}: {W}x{H}, {cfg.n} uniform stars, R={cfg.R}, sigma={cfg.sigma:g}",
                       "sample_stars": n_s, "frames_per_s_equiv": value / max(1, units_of(f, W, H, cfg.R)[0])},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "cpu_model": cpu_model(),
                             "sample": f"first {n_s} of {f.n} stars per step, fp64 oracle, {threads} pthreads"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------------ strong scaling, C5
def wide_roi_record(args, ctx, stream, flush, dev, sm_mhz, R=63):
    """C4 at R = 63 (100K clustered stars, sigma = R/6): frame ms through AUTO (k_tile_wide), its tile kernel's live ms
    and FP32/SFU roofline fraction, the list kernel (STARSIM_TILE_LISTS) and the atomic kernel on the same frame.  Each
    frame timed like the headline (K steps, L2 flushed before each, CUDA events on the render stream)."""
    import synth
    import torch
    cfg = synth.with_R(synth.CONFIGS["C4"], R)
    f = cfg.field()
    W, H, sig = cfg.W, cfg.H, cfg.sigma
    A = synth.bench_gain(sig)
    U, E = units_of(f, W, H, R)
    x, y, m = (torch.from_numpy(a).to(dev) for a in (f.x, f.y, f.mag))
    out = torch.empty((H, W), dtype=torch.float32, device=dev)

    def frames(fn, profile=False):
        for _ in range(max(3, args.warmup)):
            fn()
        torch.cuda.synchronize()
        if profile:
            ctx.profile(True)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(float(i))
                ev[i][0].record(stream)
                fn()
                ev[i][1].record(stream)
        torch.cuda.synchronize()
        kt = None
        if profile:
            kt = ctx.kernel_times()
            ctx.profile(False)
        return sum(a.elapsed_time(b) for a, b in ev) / args.steps, kt

    def tiled():
        ctx.render(x, y, m, W, H, sig, R, A, out=out, stream=stream)

    rec = {"workload": f"C4: {W}x{H}, {f.n} clustered stars, R={R}, sigma={sig:.2f}", "updates_per_frame": U,
           "exps_per_frame": E}
    ms, _ = frames(tiled)
    _, kt = frames(tiled, profile=True)
    tile_ms = kt["tile"][0] / max(1, kt["tile"][1])
    peak_rate, t_star = fp32_sfu_peak_updates(sm_mhz, U, E)
    rec["tiled"] = {"kernel": "k_tile_wide", "ms_per_frame": ms, "frames_per_s": 1e3 / ms, "updates_per_s": U / (ms * 1e-3),
                    "tile_kernel_ms": tile_ms,
                    "binning_ms": sum(kt[k][0] for k in ("prep", "sort", "csr") if k in kt) / args.steps}
    rec["roofline"] = {"bound": "alu", "kernel": "k_tile_wide", "achieved": U / (tile_ms * 1e-3) / 1e9,
                       "peak": peak_rate / 1e9, "unit": "Gupdates/s", "frac": t_star / (tile_ms * 1e-3),
                       "t_star_us": t_star * 1e6}
    ctx.set_tile_kernel("lists")
    try:
        ms_l, _ = frames(tiled)
        _, kt_l = frames(tiled, profile=True)
    finally:
        ctx.set_tile_kernel(args.tile_kernel)
    rec["lists"] = {"kernel": "k_tile", "ms_per_frame": ms_l, "tile_kernel_ms": kt_l["tile"][0] / max(1, kt_l["tile"][1])}
    ms_a, _ = frames(lambda: ctx.render_atomic(x, y, m, W, H, sig, R, A, out=out, stream=stream))
    rec["atomic"] = {"kernel": "k_atomic", "ms_per_frame": ms_a}
    return rec


def strong_c5(args, world, rank, ctx, stream, flush, dev):
    """The north star's strong-scaling target on the C5 frame (16384 x 16384, 10M uniform stars, R=15), measured in
    every run: t_1 = one GPU renders the whole frame (each rank does it alone, max over ranks); for N > 1 t_render =
    route + render of the rank's band, t_exchange = the NCCL all-gather of the bands alone, t_frame = both (NCCL),
    t_frame_fused = the fused peer-memory exchange when available; each timed like the headline (K steps, L2 flushed,
    CUDA events on the render stream, max over ranks).  eff = t_1 / (N t).  The assembled frames are compared with the
    single-GPU frame on the device, all rows (must be bitwise equal: tile-aligned bands)."""
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_ipps_lizzh12_b200 import dist as sdist
    cfg = synth.CONFIGS["C5"]
    f = cfg.field()
    W, H, R, sigma = cfg.W, cfg.H, cfg.R, cfg.sigma
    A = synth.bench_gain(sigma)
    U, _ = units_of(f, W, H, R)
    x, y, m = (torch.from_numpy(a).to(dev) for a in (f.x, f.y, f.mag))
    K = max(3, min(args.steps, 10))

    def t_of(fn):
        for _ in range(2):
            with torch.cuda.stream(stream):
                fn()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        for i in range(K):
            with torch.cuda.stream(stream):
                flush.fill_(float(i))
                ev[i][0].record(stream)
                fn()
                ev[i][1].record(stream)
        torch.cuda.synchronize()
        t = torch.tensor([sum(a.elapsed_time(b) for a, b in ev) / K], device=dev, dtype=torch.float64)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    single = torch.empty((H, W), dtype=torch.float32, device=dev)
    t1 = t_of(lambda: ctx.render(x, y, m, W, H, sigma, R, A, out=single, stream=stream))
    rec = {"workload": f"C5: {W}x{H}, {f.n} uniform stars, R={R}, sigma={sigma:g}; N = {world} bands",
           "n_gpus": world, "steps": K, "t_1gpu_ms": t1, "updates_per_frame": U,
           "updates_per_s_1gpu": U / (t1 * 1e-3)}
    if world == 1:
        rec["note"] = "N = 1: the single-GPU frame time every N > 1 run divides by (eff = t_1 / (N t_N))"
        del single
        return rec
    prow = sdist.padded_band_rows(H, world)
    row0, rows = sdist.band_rows(H, world, rank)
    band = torch.zeros((prow, W), dtype=torch.float32, device=dev)
    full = torch.empty((world * prow, W), dtype=torch.float32, device=dev)

    def render():
        if rows > 0:
            ctx.render_band_routed(x, y, m, W, H, row0, rows, sigma, R, A, out=band[:rows], stream=stream)

    def gather():
        dist.all_gather_into_tensor(full, band)

    t_render = t_of(render)  # (allocates the routed-catalogue buffers the routing-only timing below reuses)
    t_route = t_of(lambda: ctx.route_band(x, y, m, H, row0, max(rows, 1), R, out=ctx._route_buf, stream=stream))
    t_x = t_of(gather)
    t_frame = t_of(lambda: (render(), gather()))
    ok = sdist.frames_agree(full[:H], single)
    gbytes = 4 * W * prow * world  # the gathered frame (all_gather_into_tensor output)
    algbw = gbytes / (t_x * 1e-3) / 1e9
    rec.update({"t_route_ms": t_route, "t_render_ms": t_render, "t_exchange_ms": t_x, "t_frame_ms": t_frame,
                "eff_render": t1 / (world * t_render), "eff_frame": t1 / (world * t_frame),
                "exchange": {"op": "NCCL all_gather_into_tensor", "bytes": gbytes, "algbw_GBps": algbw,
                             "busbw_GBps": algbw * (world - 1) / world},
                "updates_per_s": U / (t_frame * 1e-3),
                "assembled_equals_1gpu": ok, "validation": "every rank's assembled frame vs its own single-GPU frame, "
                                                          "all pixels, bitwise (dist.frames_agree)"})
    del full
    if sdist.FusedFrame.available():
        try:
            ff = sdist.FusedFrame(H, W, dev)
            t_fused = t_of(lambda: ff.render(ctx, x, y, m, sigma, R, A, stream=stream))
            rec.update({"t_frame_fused_ms": t_fused, "eff_frame_fused": t1 / (world * t_fused),
                        "fused_equals_1gpu": sdist.frames_agree(ff.frame, single)})
            del ff
        except Exception as e:  # noqa: BLE001
            rec["fused_error"] = f"{type(e).__name__}: {e}"
    del single, band
    return rec


# ------------------------------------------------------------------------------------------------ our arm
def run_ours(args, world, rank, local_rank):
    import numpy as np
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_ipps_lizzh12_b200 import Context, dist as sdist

    dev = torch.device(f"cuda:{local_rank}")
    torch.cuda.set_device(dev)
    cfg, f, H, _ = workload(args.config, world, rank, args.scaling)
    W, R, sigma = cfg.W, cfg.R, cfg.sigma
    A = synth.bench_gain(sigma)
    U_frame, E_frame = units_of(f, W, H, R)
    ctx = Context(local_rank)
    ctx.set_tile_kernel(args.tile_kernel)
    stream = torch.cuda.Stream(dev)
    prow = sdist.padded_band_rows(H, world)
    row0, rows = sdist.band_rows(H, world, rank)
    # every rank holds the whole (replicated) catalogue; N > 1 routes it to the rank's band on the device inside every
    # step (starsim_route_band + a device star count: Context.render_band_routed), so routing is timed with the render
    x, y, m = (torch.from_numpy(a).to(dev) for a in (f.x, f.y, f.mag))
    band = torch.zeros((prow, W), dtype=torch.float32, device=dev)
    full = torch.empty((world * prow, W), dtype=torch.float32, device=dev) if world > 1 else None
    flush = torch.empty(FLUSH_BYTES // 4, dtype=torch.float32, device=dev)

    # N > 1: routed band render + NCCL all-gather (default), or the fused band exchange (STARSIM_EXCHANGE=fused: the
    # tile epilogue stores into every rank's symmetric-memory frame over NVLink between two device barriers)
    fused = None
    if world > 1 and os.environ.get("STARSIM_EXCHANGE", "allgather") == "fused" and sdist.FusedFrame.available():
        try:
            fused = sdist.FusedFrame(H, W, dev)
        except Exception as e:  # noqa: BLE001 -- fall back to the all-gather, say so in the JSON line
            print(f"bench: fused exchange unavailable ({e}); using the NCCL all-gather", file=sys.stderr)
            fused = None
    exchange = "single" if world == 1 else ("fused-p2p" if fused is not None else "nccl-allgather")

    def step(xx, yy, mm):
        with torch.cuda.stream(stream):
            if world == 1:
                if args.method == "atomic":
                    ctx.render_atomic(xx, yy, mm, W, H, sigma, R, A, out=band[:H], stream=stream)
                else:
                    ctx.render_band(xx, yy, mm, W, H, 0, H, sigma, R, A, out=band[:H], stream=stream)
            elif fused is not None:
                fused.render(ctx, xx, yy, mm, sigma, R, A, stream=stream)
            else:
                if rows > 0:
                    ctx.render_band_routed(xx, yy, mm, W, H, row0, rows, sigma, R, A, out=band[:rows], stream=stream)
                dist.all_gather_into_tensor(full, band)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(max(3, args.warmup)):
        step(x, y, m)
    barrier()
    # stars this rank renders: the whole catalogue (N = 1) or its band's routed stars (the device count, read once here)
    n_band = f.n if world == 1 else (int(ctx._route_buf[3].item()) if rows > 0 else 0)

    def timed_region(profile):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(args.steps)]
        if profile:
            ctx.profile(True)
        barrier()
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(float(i))                  # evict L2 (256 MiB > 126 MB), untimed
                ev[i][0].record(stream)
            step(x, y, m)
            ev[i][1].record(stream)
        barrier()
        kt = None
        if profile:
            kt = ctx.kernel_times()
            ctx.profile(False)
        return [a.elapsed_time(b) for a, b in ev], kt

    with ClockSampler(local_rank) as clk:
        # 1) the timed region: the product path (one CUDA-graph replay per frame)
        ms_steps, _ = timed_region(False)
        # 2) the same K steps again with every kernel bracketed by CUDA events on the render stream (direct launches,
        #    identical kernels): per-kernel durations for the roofline
        ms_prof_steps, kt = timed_region(True)
        # keep sampling clocks over >= 0.3 s of the same step so a short timed region still gets samples
        t_end = time.time() + 0.3
        while time.time() < t_end:
            step(x, y, m)
        torch.cuda.synchronize()
    ms = sum(ms_steps) / len(ms_steps)
    t = torch.tensor([ms], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    value = U_frame / (ms * 1e-3)      # updates of the whole frame (all ranks) per second

    # per-kernel live timings (this rank); launches of our own kernels per step
    launches = sum(v[1] for k, v in kt.items() if k not in ("memset",)) / args.steps
    tile_ms = kt["tile"][0] / max(1, kt["tile"][1]) if kt["tile"][1] else kt["atomic"][0] / max(1, kt["atomic"][1])
    clocks = clk.summary()
    sm_mhz = clocks["sm_mhz"] or 1965.0
    # roofline of the dominant kernel (k_tile) on this rank's band
    band_f_units = units_of(synth.Field(f.x, f.y, f.mag), W, H, R) if world == 1 else None
    U_band, E_band = (U_frame, E_frame) if world == 1 else (U_frame / world, E_frame / world)
    peak_rate, t_star = fp32_sfu_peak_updates(sm_mhz, U_band, E_band)
    peak_max, _ = fp32_sfu_peak_updates(1965.0, U_band, E_band)
    achieved = U_band / (tile_ms * 1e-3) if args.method == "tiled" else None
    peaks, peak_src = load_peaks()
    traffic, ncu_tile = None, {}
    prof = os.path.join(ROOT, "profiles", "ncu_tile_traffic.json")
    if os.path.exists(prof):
        try:
            ncu_tile = json.load(open(prof)).get(cfg.name, {})
            traffic = ncu_tile.get("dram_bytes_per_launch")
        except Exception:
            traffic, ncu_tile = None, {}
    roofline = {"bound": "alu", "kernel": "k_tile", "achieved": achieved / 1e9 if achieved else None,
                "peak": peak_rate / 1e9, "unit": "Gupdates/s", "frac": (achieved / peak_rate) if achieved else None,
                "traffic": traffic,
                "peak_basis": f"FP32/SFU roofline max(U/(148*128*f), E/(148*16*f)) at the measured SM clock "
                              f"f={sm_mhz:.0f} MHz; U={U_band}, E={E_band}; frac at 1965 MHz = "
                              f"{(achieved / peak_max) if achieved else 0:.3f}",
                "kernel_ms": tile_ms,
                "issue": ({"kernel": ncu_tile.get("kernel"), "warp_instructions": ncu_tile.get("warp_instructions"),
                           "issue_active_pct": ncu_tile.get("issue_active_pct"),
                           "fma_pipe_pct": ncu_tile.get("fma_pipe_pct"),
                           "note": "what bounds the tile kernel: instruction issue (ncu --set full, "
                                   "profiles/ncu_tile_traffic.json; DESIGN.md section 9)"}
                          if ncu_tile.get("warp_instructions") else None),
                "hbm": {"bytes": 4 * W * (rows if world > 1 else H) + 16 * n_band,
                        "achieved_GBps": (4 * W * (rows if world > 1 else H) + 16 * n_band) / (tile_ms * 1e-3) / 1e9,
                        "peak_GBps": peaks.get("hbm_gbs"), "peak_source": peak_src}}
    kernels = {k: {"ms_per_step": v[0] / args.steps, "launches_per_step": v[1] / args.steps} for k, v in kt.items()
               if v[1]}
    # the binning kernels' HBM view (north star: "achieved HBM GB/s for the binning ... passes"): algorithmic bytes per
    # step over each kernel's live time.  a1 (k_dcount): 12 B catalogue in + 16 B record + 4 B tile box
    # out per star + the count matrix; a2 column scan: the count matrix read and written; a3/a4 (k_dplace): 4 B tile
    # box per star + 4 B id per pair + the count matrix column
    if world == 1 and args.method == "tiled" and "sort" in kernels:
        ntl = (-(-W // 128)) * (-(-H // 64))
        try:
            P_pairs = int(ctx.get_bins()[2][ntl])  # tile_off[ntiles] of the last render = the (tile, star) pairs
        except Exception:  # noqa: BLE001
            P_pairs = None
        ncta = -(-f.n // 4096)
        cm = 4 * ntl * ncta
        alg = {"prep": 32 * f.n + cm, "csr": 2 * cm, "sort": 4 * f.n + (4 * P_pairs if P_pairs else 0) + cm}
        hbm_peak = peaks.get("hbm_gbs")
        for k_, b_ in alg.items():
            if k_ in kernels and kernels[k_]["ms_per_step"] > 0:
                gbs = b_ / (kernels[k_]["ms_per_step"] * 1e-3) / 1e9
                kernels[k_]["algorithmic_bytes"] = b_
                kernels[k_]["achieved_GBps"] = gbs
                kernels[k_]["frac_of_hbm_peak"] = gbs / hbm_peak if hbm_peak else None

    # NEXT-1 variant (1 GPU, tiled): the same frame with the output stage fused -- u8 gray image written by k_tile
    variants = {}
    try:  # the variants are diagnostics: a failure is recorded in the line, not fatal to the headline
        if world == 1 and args.method == "tiled":
            gray = torch.empty((H, W), dtype=torch.uint8, device=dev)
            Ag = synth.bench_gain(sigma, 8)

            def gstep():
                with torch.cuda.stream(stream):
                    ctx.render_gray(x, y, m, W, H, sigma, R, Ag, bits=8, out=gray, stream=stream)

            for _ in range(max(3, args.warmup)):
                gstep()
            barrier()
            g_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                    for _ in range(args.steps)]
            for i in range(args.steps):
                with torch.cuda.stream(stream):
                    flush.fill_(float(i))
                    g_ev[i][0].record(stream)
                gstep()
                g_ev[i][1].record(stream)
            barrier()
            g_ms = sum(a.elapsed_time(b) for a, b in g_ev) / args.steps
            variants["gray_u8"] = {"ms_per_step": g_ms, "frames_per_s": 1e3 / g_ms, "updates_per_s": U_frame / (g_ms * 1e-3),
                                   "note": "starsim_render_gray (output stage fused into k_tile, u8 image)"}
            # NEXT-2 variant: the same fp32 frame with the pixel-integrated PSF (erf profiles instead of exp)
            ctx.set_psf("integrated")
            for _ in range(max(3, args.warmup)):
                step(x, y, m)
            barrier()
            i_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                    for _ in range(args.steps)]
            for i in range(args.steps):
                with torch.cuda.stream(stream):
                    flush.fill_(float(i))
                    i_ev[i][0].record(stream)
                step(x, y, m)
                i_ev[i][1].record(stream)
            barrier()
            ctx.set_psf("point")
            i_ms = sum(a.elapsed_time(b) for a, b in i_ev) / args.steps
            variants["integrated_psf"] = {"ms_per_step": i_ms, "frames_per_s": 1e3 / i_ms,
                                          "updates_per_s": U_frame / (i_ms * 1e-3),
                                          "note": "starsim_set_psf(INTEGRATED): Eq. 2 integrated over each pixel (NEXT-2)"}
            # NEXT-3 variant: the same fp32 frame with the pixel-circle ROI (k_tile_sb masks the circle in its walk)
            ctx.set_roi("circle")
            for _ in range(max(3, args.warmup)):
                step(x, y, m)
            barrier()
            r_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                    for _ in range(args.steps)]
            for i in range(args.steps):
                with torch.cuda.stream(stream):
                    flush.fill_(float(i))
                    r_ev[i][0].record(stream)
                step(x, y, m)
                r_ev[i][1].record(stream)
            barrier()
            ctx.set_roi("square")
            r_ms = sum(a.elapsed_time(b) for a, b in r_ev) / args.steps
            variants["circle_roi"] = {"ms_per_step": r_ms, "frames_per_s": 1e3 / r_ms,
                                      "note": "starsim_set_roi(CIRCLE): the paper's 'pixel circle' ROI through the tiled "
                                              "path (NEXT-3, reading R21)"}

            # the paper's two star-centric designs on the same frame: the atomic simulator and its lookup-table variant
            for name, fn_, note in (("atomic", ctx.render_atomic, "starsim_render_atomic: the paper's parallel simulator "
                                     "(Fig. 6), red.global.add per ROI pixel, nondeterministic order"),
                                    ("lut", ctx.render_lut, "starsim_render_lut: the paper's adaptive simulator "
                                     "(PAPER.md:158-168), table at the ROI centre (reading R20, approximate off-centre)")):
                if world > 1:
                    break
                a_out = torch.empty((H, W), dtype=torch.float32, device=dev)
                for _ in range(2):
                    fn_(x, y, m, W, H, sigma, R, A, out=a_out, stream=stream)
                torch.cuda.synchronize()
                a_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                        for _ in range(args.steps)]
                for i in range(args.steps):
                    with torch.cuda.stream(stream):
                        flush.fill_(float(i))
                        a_ev[i][0].record(stream)
                        fn_(x, y, m, W, H, sigma, R, A, out=a_out, stream=stream)
                        a_ev[i][1].record(stream)
                torch.cuda.synchronize()
                a_ms = sum(a.elapsed_time(b) for a, b in a_ev) / args.steps
                variants[name] = {"ms_per_step": a_ms, "frames_per_s": 1e3 / a_ms, "updates_per_s": U_frame / (a_ms * 1e-3),
                                  "note": note}
                if name == "atomic":  # NEXT-3: the same star-centric kernel with the pixel-circle ROI
                    ctx.set_roi("circle")
                    fn_(x, y, m, W, H, sigma, R, A, out=a_out, stream=stream)
                    torch.cuda.synchronize()
                    c_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                            for _ in range(args.steps)]
                    for i in range(args.steps):
                        with torch.cuda.stream(stream):
                            flush.fill_(float(i))
                            c_ev[i][0].record(stream)
                            fn_(x, y, m, W, H, sigma, R, A, out=a_out, stream=stream)
                            c_ev[i][1].record(stream)
                    torch.cuda.synchronize()
                    ctx.set_roi("square")
                    c_ms = sum(a.elapsed_time(b) for a, b in c_ev) / args.steps
                    variants["atomic_circle"] = {"ms_per_step": c_ms, "frames_per_s": 1e3 / c_ms,
                                                 "note": "starsim_set_roi(CIRCLE) + starsim_render_atomic: the paper's "
                                                         "'pixel circle' ROI (NEXT-3, reading R21)"}
                del a_out
    except Exception as e:  # noqa: BLE001
        variants["error"] = f"{type(e).__name__}: {e}"
        torch.cuda.synchronize()
        ctx.set_psf("point")
        ctx.set_roi("square")
    # the wide-ROI end of the C4 sweep (BASELINE configs[3]: 100K clustered stars, R = 63): the sorted-corner-bin wide
    # kernel k_tile_wide (AUTO) against the list kernel k_tile and the paper's atomic design, with its own roofline
    try:
        if world == 1 and args.method == "tiled" and not args.no_wide:
            variants["wide_roi_C4_R63"] = wide_roi_record(args, ctx, stream, flush, dev, sm_mhz)
    except Exception as e:  # noqa: BLE001
        variants["wide_roi_C4_R63"] = {"error": f"{type(e).__name__}: {e}"}
        torch.cuda.synchronize()
        ctx.set_tile_kernel(args.tile_kernel)

    # e2e: the same C-ABI call with host (pinned) catalogue in and image out, copies inside the timed region
    e2e = None
    if not args.no_e2e:
        hx, hy, hm = (torch.from_numpy(a).pin_memory() for a in (f.x, f.y, f.mag))
        himg = torch.empty((rows if world > 1 else H, W), dtype=torch.float32).pin_memory()
        dx, dy, dm = (torch.empty_like(x) for _ in range(3))

        def e2e_step():
            with torch.cuda.stream(stream):
                dx.copy_(hx, non_blocking=True)
                dy.copy_(hy, non_blocking=True)
                dm.copy_(hm, non_blocking=True)
            step(dx, dy, dm)
            with torch.cuda.stream(stream):
                src = fused.frame[row0:row0 + rows] if fused is not None else band[:himg.shape[0]]
                himg[:src.shape[0]].copy_(src, non_blocking=True)

        for _ in range(2):
            e2e_step()
        barrier()
        e_ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                for _ in range(args.steps)]
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(float(i))
                e_ev[i][0].record(stream)
            e2e_step()
            e_ev[i][1].record(stream)
        barrier()
        e_ms = sum(a.elapsed_time(b) for a, b in e_ev) / args.steps
        te = torch.tensor([e_ms], device=dev, dtype=torch.float64)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e_ms = float(te.item())
        e2e = {"value": U_frame / (e_ms * 1e-3), "unit": UNIT, "ms_per_step": e_ms,
               "h2d_bytes_per_step": int(3 * 4 * f.n), "d2h_bytes_per_step": int(himg.numel() * 4),
               "note": "pinned host catalogue -> device, render, image -> pinned host, per step, one stream"
                       + ("; per rank: the whole catalogue in (routed on the device), its band out (max over ranks)"
                          if world > 1 else "")}
        if world == 1 and args.method == "tiled":
            # the same steps pipelined over two streams (one ctx, catalogue and image buffers each): step i+1's copy in
            # and render overlap step i's copy out (PCIe is full duplex); every step still moves its own catalogue in
            # and its own image out.  Timed from the first copy in to the last copy out.
            streams = [stream, torch.cuda.Stream(dev)]
            ctxs = [ctx, Context(local_rank)]
            dbufs = [(dx, dy, dm), tuple(torch.empty_like(x) for _ in range(3))]
            imgs = [band, torch.empty_like(band)]
            himgs = [himg, torch.empty_like(himg).pin_memory()]

            def p_step(i):
                s_ = i & 1
                st, cx, (ax, ay, am) = streams[s_], ctxs[s_], dbufs[s_]
                with torch.cuda.stream(st):
                    ax.copy_(hx, non_blocking=True)
                    ay.copy_(hy, non_blocking=True)
                    am.copy_(hm, non_blocking=True)
                    cx.render_band(ax, ay, am, W, H, row0, rows, sigma, R, A, out=imgs[s_][:rows], stream=st)
                    himgs[s_].copy_(imgs[s_][:himg.shape[0]], non_blocking=True)

            for i in range(4):
                p_step(i)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            e0.record(streams[0])
            streams[1].wait_event(e0)
            for i in range(args.steps):
                p_step(i)
            for k in range(2):
                e1[k].record(streams[k])
            torch.cuda.synchronize()
            p_ms = max(e0.elapsed_time(e1[k]) for k in range(2)) / args.steps
            e2e = {"value": U_frame / (p_ms * 1e-3), "unit": UNIT, "ms_per_step": p_ms,
                   "h2d_bytes_per_step": int(3 * 4 * f.n), "d2h_bytes_per_step": int(himg.numel() * 4),
                   "latency_ms_one_stream": e_ms,
                   "note": "pinned host catalogue -> device, render, image -> pinned host for every step; steps "
                           "pipelined over two streams (copy out of step i overlaps copy in + render of step i+1)"}
            # the paper's output format end to end: the same pipeline with the fused output stage (u8 gray image
            # out) -- a diagnostic next to the fp32 headline
            try:
                Ag = synth.bench_gain(sigma, 8)
                gimgs = [torch.empty((H, W), dtype=torch.uint8, device=dev) for _ in range(2)]
                hgs = [torch.empty((H, W), dtype=torch.uint8).pin_memory() for _ in range(2)]

                def g_step(i):
                    s_ = i & 1
                    st, cx, (ax, ay, am) = streams[s_], ctxs[s_], dbufs[s_]
                    with torch.cuda.stream(st):
                        ax.copy_(hx, non_blocking=True)
                        ay.copy_(hy, non_blocking=True)
                        am.copy_(hm, non_blocking=True)
                        cx.render_gray(ax, ay, am, W, H, sigma, R, Ag, bits=8, out=gimgs[s_], stream=st)
                        hgs[s_].copy_(gimgs[s_], non_blocking=True)

                for i in range(4):
                    g_step(i)
                torch.cuda.synchronize()
                g0, g1 = torch.cuda.Event(enable_timing=True), [torch.cuda.Event(enable_timing=True) for _ in range(2)]
                g0.record(streams[0])
                streams[1].wait_event(g0)
                for i in range(args.steps):
                    g_step(i)
                for k in range(2):
                    g1[k].record(streams[k])
                torch.cuda.synchronize()
                gp_ms = max(g0.elapsed_time(g1[k]) for k in range(2)) / args.steps
                e2e["gray_u8"] = {"value": U_frame / (gp_ms * 1e-3), "unit": UNIT, "ms_per_step": gp_ms,
                                  "h2d_bytes_per_step": int(3 * 4 * f.n), "d2h_bytes_per_step": int(H * W),
                                  "note": "starsim_render_gray (output stage fused), u8 image out, same two-stream "
                                          "pipeline"}
            except Exception as e:  # noqa: BLE001
                e2e["gray_u8"] = {"error": f"{type(e).__name__}: {e}"}
            ctxs[1].close()

    strong = None
    if not args.no_strong and args.method == "tiled":
        try:
            strong = strong_c5(args, world, rank, ctx, stream, flush, dev)
        except Exception as e:  # noqa: BLE001 -- a diagnostic record; the headline stands without it
            strong = {"error": f"{type(e).__name__}: {e}"}
        torch.cuda.synchronize()
    if rank != 0:
        ctx.close()
        return
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(cfg, f, W, H)
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": args.scaling,
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{cfg.name}: {W}x{H}, {cfg.n} uniform stars, R={R}, sigma={sigma:g}"
                                   + (f"; {world} bands of {prow} rows, exchange {exchange}" if world > 1 else ""),
                       "W": W, "H": H, "stars": f.n, "R": R, "sigma": sigma, "gain": A, "method": args.method,
                       "frames_per_s": 1e3 / ms, "updates_per_frame": U_frame, "exps_per_frame": E_frame,
                       "parallelism": f"bands{world}" if world > 1 else "single", "exchange": exchange,
                       "catalogue": "whole frame" if world == 1 else
                                    f"replicated on every rank; each step routes it to the rank's band on the device "
                                    f"(starsim_route_band, timed in the step; rank 0 renders {n_band} of {f.n})",
                       "l2": "flushed before every step (256 MiB write, untimed)"},
            "clocks": clocks, "gpu_launches": int(round(launches * args.steps)),
            "gpu_launches_per_step": launches, "kernels": kernels,
            "ms_per_step_direct_launch": sum(ms_prof_steps) / len(ms_prof_steps),
            "roofline": roofline, "e2e": e2e, "variants": variants, "strong_C5": strong,
            "cpu_baseline": cpu}
    print(json.dumps(line), flush=True)
    ctx.close()


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    if world > 1 and args.method == "atomic":
        # the star-centric render has no band form: it would write the whole frame into a band buffer
        print(json.dumps({"error": "--method atomic is single-GPU only (no band decomposition)"}), flush=True)
        sys.exit(2)
    import __graft_entry__
    if rank == 0 or world == 1:
        __graft_entry__.build()
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local_rank}"))
        dist.barrier()
        __graft_entry__.build()
    run_ours(args, world, rank, local_rank)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
