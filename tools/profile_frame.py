#!/usr/bin/env python
"""Render one synthetic frame a few times through the C ABI: the short command ncu wraps.

    python tools/profile_frame.py [--config T] [--R 15] [--n N] [--reps 5] [--atomic]

Warm-up renders first, then `reps` renders on a non-default stream with CUDA graphs off (every kernel a visible
launch).  No oracle, no timing: use `ncu -s <skip> -c <count>` to pick launches.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("STARSIM_NO_GRAPH", "1")

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_lizzh12_b200 import Context  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="T")
    ap.add_argument("--R", type=int, default=0)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--atomic", action="store_true")
    ap.add_argument("--tile", default="auto", help="tile kernel: auto | lists | sb")
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    if a.R:
        cfg = synth.with_R(cfg, a.R)
    f = cfg.field(n=a.n or None)
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    gain = synth.bench_gain(cfg.sigma)
    out = torch.empty((cfg.H, cfg.W), dtype=torch.float32, device=dev)
    with Context(0) as ctx:
        ctx.set_tile_kernel(a.tile)
        fn = ctx.render_atomic if a.atomic else ctx.render
        for _ in range(a.reps + 2):
            fn(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, gain, out=out)
        torch.cuda.synchronize()
    print(f"rendered {a.config} R={cfg.R} n={f.n} x{a.reps + 2}")


if __name__ == "__main__":
    main()
