#!/usr/bin/env python
"""Phase split of k_tile_ws (debug build with -DSTARSIM_WS_TIMING, library path in STARSIM_LIB): SM cycles per
warp-chunk of the producer phases and of the consumer phases.

    STARSIM_NVCC_EXTRA=-DSTARSIM_WS_TIMING python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)"
    python tools/ws_timing.py [--config T] [--reps 3]
"""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("STARSIM_NO_GRAPH", "1")

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_lizzh12_b200 import Context, starsim  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="T")
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    f = cfg.field()
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    out = torch.empty((cfg.H, cfg.W), dtype=torch.float32, device=dev)
    fn = starsim.lib().starsim_debug_ws_timing
    fn.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.c_int]
    buf = (ctypes.c_double * 10)()
    with Context(0) as ctx:
        ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(buf, 1)
        for _ in range(a.reps):
            ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(buf, 1)
    pn = ["records + key + match + hist", "barrier 1", "empty wait", "scan + barrier 2", "profiles + arrive"]
    cn = ["full wait", "walk", "epilogue"]
    print(f"{a.config}: {buf[5] / a.reps:.0f} producer warp-chunks, {buf[9] / a.reps:.0f} consumer warp-chunks per frame")
    tp = sum(buf[:5])
    for k, nm in enumerate(pn):
        print(f"  P {nm:30s} {buf[k] / buf[5]:9.0f} cycles/warp-chunk {buf[k] / tp:6.1%}")
    tc = sum(buf[6:9])
    for k, nm in enumerate(cn):
        print(f"  C {nm:30s} {buf[6 + k] / buf[9]:9.0f} cycles/warp-chunk {buf[6 + k] / tc:6.1%}")


if __name__ == "__main__":
    main()
