#!/usr/bin/env python
"""Graph-replayed frame time (the product path: non-default stream, one CUDA graph per frame, L2 flushed between
frames, CUDA events on the stream), median over --steps, for the tiled render and the star-centric atomic render:
    python tools/frame_time.py --config C3 --n 1000 [--R 15] [--mode auto]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ipps_lizzh12_b200 import Context  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="T")
    ap.add_argument("--R", type=int, default=0)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--mode", default="auto")
    a = ap.parse_args()
    cfg = synth.with_R(synth.CONFIGS[a.config], a.R) if a.R else synth.CONFIGS[a.config]
    f = cfg.field(a.n) if a.n else cfg.field()
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    out = torch.empty((cfg.H, cfg.W), dtype=torch.float32, device=dev)
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
    st = torch.cuda.Stream(dev)
    res = {}
    with Context(0) as ctx, torch.cuda.stream(st):
        ctx.set_tile_kernel(a.mode)
        for name, fn in (("tiled", ctx.render), ("atomic", ctx.render_atomic)):
            for _ in range(3):
                fn(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out, stream=st)
            ts = []
            for i in range(a.steps):
                flush.fill_(float(i))
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(st)
                fn(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out, stream=st)
                e1.record(st)
                st.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e3)
            res[name] = sorted(ts)[len(ts) // 2]
    print(f"{a.config}" + (f"/R{a.R}" if a.R else "") + f"/n{f.n} mode={a.mode} tiled={res['tiled']:.1f}us "
          f"atomic={res['atomic']:.1f}us ratio={res['tiled'] / res['atomic']:.2f}", flush=True)


if __name__ == "__main__":
    main()
