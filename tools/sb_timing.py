#!/usr/bin/env python
"""Phase split of k_tile_sb (debug build with -DSTARSIM_SB_TIMING): SM cycles per chunk and warp spent in the sort,
the scan, the profiles, the wait before the walk, and the walk itself.

    STARSIM_NVCC_EXTRA=-DSTARSIM_SB_TIMING python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)"
    python tools/sb_timing.py [--config T] [--reps 3]
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
    L = starsim.lib()
    fn = L.starsim_debug_sb_timing
    fn.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.c_int]
    buf = (ctypes.c_double * 6)()
    with Context(0) as ctx:
        ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(buf, 1)
        for _ in range(a.reps):
            ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(buf, 1)
    names = ["sort (match, hist, barrier 1)", "scan (warp 0, barrier 2)", "profiles", "wait (barrier 3)",
             "walk (accumulate)"]
    n = buf[5]
    tot = sum(buf[:5])
    print(f"{a.config}: {n / a.reps:.0f} warp-chunks per frame")
    for k, nm in enumerate(names):
        print(f"  {nm:32s} {buf[k] / n:9.0f} cycles per warp-chunk  {buf[k] / tot:6.1%}")


if __name__ == "__main__":
    main()
