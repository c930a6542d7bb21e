#!/usr/bin/env python
"""Star-count and ROI sweeps of the tiled path against the atomic and lookup-table comparison kernels (the C3 / C4
"selection" study, the B200 analogue of the paper's Table III).

    python tools/sweep.py [--sweep c3|c4|all] [--steps 10] [--warmup 3] > profiles/<round>_sweep.jsonl

One JSON line per (config point, method): device ms per frame (CUDA events around each frame on the render stream,
L2 flushed before every frame, graph replay for the tiled path), star-pixel updates/s, and the tiled path's per-kernel
split (a second, profiled pass).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_lizzh12_b200 import Context  # noqa: E402


def units(f, cfg):
    """U = sum over stars of the clipped ROI area (exact integer), computed from the inputs."""
    x, y, R, W, H = f.x.astype(np.float64), f.y.astype(np.float64), cfg.R, cfg.W, cfg.H
    ok = np.isfinite(x) & np.isfinite(y) & np.isfinite(f.mag)
    fl = np.floor(np.where(ok, x, 0))
    lx = np.where(R % 2 == 1, fl + (x - fl >= 0.5) - (R - 1) // 2, fl + 1 - R // 2)
    fl = np.floor(np.where(ok, y, 0))
    ly = np.where(R % 2 == 1, fl + (y - fl >= 0.5) - (R - 1) // 2, fl + 1 - R // 2)
    w = np.clip(np.minimum(lx + R - 1, W - 1) - np.maximum(lx, 0) + 1, 0, None)
    h = np.clip(np.minimum(ly + R - 1, H - 1) - np.maximum(ly, 0) + 1, 0, None)
    return int(np.sum(np.where(ok, w * h, 0)))


def time_frames(fn, steps, warmup, stream, flush):
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    ms = []
    for i in range(steps):
        with torch.cuda.stream(stream):
            flush.fill_(float(i))
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
        fn()
        b.record(stream)
        ms.append((a, b))
    torch.cuda.synchronize()
    t = sorted(a.elapsed_time(b) for a, b in ms)
    return t[len(t) // 2], t[0], t[-1]


def run_point(ctx, label, cfg, f, steps, warmup, stream, flush, out):
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    gain = synth.bench_gain(cfg.sigma)
    U = units(f, cfg)
    res = {}
    for method in ("tiled", "atomic", "lut"):
        fn_ = {"tiled": ctx.render, "atomic": ctx.render_atomic, "lut": ctx.render_lut}[method]
        med, lo, hi = time_frames(lambda: fn_(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, gain, out=out, stream=stream),
                                  steps, warmup, stream, flush)
        line = {"sweep": label, "W": cfg.W, "H": cfg.H, "stars": f.n, "R": cfg.R, "sigma": cfg.sigma,
                "method": method, "ms_median": med, "ms_min": lo, "ms_max": hi, "updates": U,
                "updates_per_s": U / (med * 1e-3)}
        if method == "tiled":
            ctx.profile(True)
            for _ in range(3):
                fn_(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, gain, out=out, stream=stream)
            kt = ctx.kernel_times()
            ctx.profile(False)
            line["kernels_ms"] = {k: v[0] / 3 for k, v in kt.items() if v[1]}
        res[method] = med
        print(json.dumps(line), flush=True)
    print(json.dumps({"sweep": label, "stars": f.n, "R": cfg.R, "winner": min(res, key=res.get),
                      "atomic_over_tiled": res["atomic"] / res["tiled"], "lut_over_atomic": res["lut"] / res["atomic"]}),
          flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sweep", default="all", choices=["c3", "c4", "all"])
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    stream = torch.cuda.Stream()
    flush = torch.empty(256 << 18, dtype=torch.float32, device=dev)  # 256 MiB
    out = torch.empty((4096, 4096), dtype=torch.float32, device=dev)
    with Context(0) as ctx:
        if a.sweep in ("c3", "all"):
            cfg = synth.CONFIGS["C3"]
            for n in [2 ** k for k in range(10, 21)] + [10 ** 6]:
                run_point(ctx, "C3", cfg, cfg.field(n=n), a.steps, a.warmup, stream, flush, out)
        if a.sweep in ("c4", "all"):
            base = synth.CONFIGS["C4"]
            for R in (3, 5, 7, 9, 11, 15, 21, 31, 47, 63):
                cfg = synth.with_R(base, R)
                run_point(ctx, "C4", cfg, cfg.field(), a.steps, a.warmup, stream, flush, out)


if __name__ == "__main__":
    main()
