#!/usr/bin/env python
"""Small frames through every kernel of the library, for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck):  compute-sanitizer --tool racecheck python tools/sanitize_run.py
C1 (1024^2, 1000 stars, R=5) and a heavy-tile field (256^2, 30K stars in a 40-px disc: split tiles, partial buffers,
1024-star segments) through every tile kernel (lists, sb, ws, t8; both binning pipelines), a band, the gray epilogue,
the integrated PSF, the circle ROI, the star-centric kernels, quantize, upload_aos and the band routing; a sparse 4096 x 2048
frame (2,000 stars) for k_tile_lite; k_tile_ws fed by k_chsort; a heavy wide-ROI field (R = 47: k_tile_wide, k_tile_wws,
256-star segments and parts)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("STARSIM_NO_GRAPH", "1")
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_lizzh12_b200 import Context  # noqa: E402


def heavy(n, W, H, seed):
    rng = np.random.default_rng(seed)
    r = 40.0 * np.sqrt(rng.random(n))
    t = 2 * np.pi * rng.random(n)
    return synth.Field((W / 2 + r * np.cos(t)).astype(np.float32), (H / 2 + r * np.sin(t)).astype(np.float32),
                       rng.uniform(0, 15, n).astype(np.float32))


def main():
    quick = "--quick" in sys.argv  # racecheck: fewer frames
    only = next((a.split("=", 1)[1].split(",") for a in sys.argv if a.startswith("--kernels=")), None)
    dev = torch.device("cuda:0")
    c1 = synth.CONFIGS["C1"]
    cases = [("C1", c1.field(), c1.W, c1.H, c1.R, c1.sigma), ("heavy", heavy(30000, 256, 256, 3), 256, 256, 15, 2.5),
             ("sparse", synth.uniform_field(2000, 4096, 2048, seed=5), 4096, 2048, 15, 2.5),  # k_tile_lite
             ("wide", heavy(6000, 256, 256, 4), 256, 256, 47, 7.8)]  # k_tile_wide (sb/auto), k_tile_wws (ws/t8)
    with Context(0) as ctx:
        for name, f, W, H, R, sigma in cases:
            x, y, m = (torch.from_numpy(a).to(dev) for a in (f.x, f.y, f.mag))
            for tk in (only or (["ws", "t8"] if quick else ["lists", "sb", "ws", "t8"])):
                for binning in (["auto"] if quick else ["auto", "atomic"]):
                    ctx.set_tile_kernel(tk)
                    ctx.set_binning(binning)
                    ctx.render(x, y, m, W, H, sigma, R, 1.0)
            ctx.set_tile_kernel("auto")
            ctx.set_binning("auto")
            if only:
                continue
            ctx.render_band(x, y, m, W, H, 64, 64, sigma, R, 1.0)
            ctx.render_band_routed(x, y, m, W, H, 64, 64, sigma, R, 1.0)
            if not quick:
                ctx.set_tile_kernel("lists")
                ctx.render_gray(x, y, m, W, H, sigma, R, 1.0, bits=8)
                ctx.set_tile_kernel("auto")
                ctx.render_gray(x, y, m, W, H, sigma, R, 1.0, bits=16)
                ctx.set_psf("integrated")
                ctx.render(x, y, m, W, H, sigma, R, 1.0)
                ctx.set_psf("point")
                ctx.set_roi("circle")
                ctx.render(x, y, m, W, H, sigma, R, 1.0)
                ctx.render_atomic(x, y, m, W, H, sigma, R, 1.0)
                ctx.set_roi("square")
                ctx.render_atomic(x, y, m, W, H, sigma, R, 1.0)
                ctx.render_lut(x, y, m, W, H, sigma, R, 1.0)
                img = ctx.render(x, y, m, W, H, sigma, R, 1.0)
                ctx.quantize(img, 8)
                ctx.upload_aos(f.aos()[:1000])
            if not quick or name != "sparse":
                # k_tile_ws fed by k_chsort (a context created with STARSIM_WS_PRESORT=1)
                os.environ["STARSIM_WS_PRESORT"] = "1"
                with Context(0) as cpre:
                    cpre.set_tile_kernel("ws")
                    cpre.render(x, y, m, W, H, sigma, R, 1.0)
                del os.environ["STARSIM_WS_PRESORT"]
            torch.cuda.synchronize()
            print(name, "ok", flush=True)


if __name__ == "__main__":
    main()
