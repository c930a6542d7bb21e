#!/usr/bin/env python
"""Phase split of k_tile8 (debug build with -DT8_TIMING, library in STARSIM_LIB): SM cycles per warp of the
producer and consumer phases.
    STARSIM_NVCC_EXTRA=-DT8_TIMING python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)"
    python tools/t8_timing.py [--config T]
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
    fn = starsim.lib().starsim_debug_t8_timing
    fn.argtypes = [ctypes.POINTER(ctypes.c_double), ctypes.c_int]
    b = (ctypes.c_double * 16)()
    with Context(0) as ctx:
        ctx.set_tile_kernel("t8")
        ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(b, 1)
        for _ in range(a.reps):
            ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        fn(b, 1)
    r = a.reps
    pw, cw = b[11] / r, b[12] / r  # total cycles summed over producer / consumer warps
    print(f"{cfg.W}x{cfg.H} n={f.n}: segments {b[5] / r / 4:.0f} chunks {b[6] / r / 4:.0f} (per frame)")
    for k, nm in ((1, "segment bin starts"), (3, "empty waits"), (4, "profiles + header + arrive")):
        print(f"  P {nm:40s} {b[k] / r / pw:6.1%}")
    for k, nm in ((7, "full waits"), (8, "ranges + walk + arrive"), (9, "epilogue")):
        print(f"  C {nm:40s} {b[k] / r / cw:6.1%}")
    print(f"  kernel cycles per warp (avg): producer {pw / (2 * 148 * 4):.0f}, consumer {cw / (2 * 148 * 4):.0f}")


if __name__ == "__main__":
    main()
