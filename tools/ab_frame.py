#!/usr/bin/env python
"""Device ms per frame (L2 flushed, median of --steps) of one synthetic frame for each tile kernel mode given:
    python tools/ab_frame.py --config C4 --R 15 --modes sb ws      (STARSIM_LIB selects the library build)"""
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
    ap.add_argument("--config", default="C4")
    ap.add_argument("--R", type=int, default=15)
    ap.add_argument("--n", type=int, default=0)
    ap.add_argument("--steps", type=int, default=15)
    ap.add_argument("--modes", nargs="+", default=["auto"])
    a = ap.parse_args()
    cfg = synth.with_R(synth.CONFIGS[a.config], a.R) if a.R else synth.CONFIGS[a.config]
    f = cfg.field(n=a.n or None)
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    out = torch.empty((cfg.H, cfg.W), dtype=torch.float32, device=dev)
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
    st = torch.cuda.Stream(dev)
    for mode in a.modes:
        with Context(0) as ctx:
            try:
                ctx.set_tile_kernel(mode)
            except Exception as e:  # an older library without the mode
                print(mode, "n/a", e)
                continue
            ts = []
            for i in range(a.steps + 3):
                with torch.cuda.stream(st):
                    flush.fill_(float(i))
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(st)
                    ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out, stream=st)
                    e1.record(st)
                torch.cuda.synchronize()
                if i >= 3:
                    ts.append(e0.elapsed_time(e1))
            ts.sort()
            print(f"{os.path.basename(os.environ.get('STARSIM_LIB', 'cur'))} {a.config} R={cfg.R} n={f.n} {mode}: "
                  f"{ts[len(ts) // 2] * 1e3:.1f} us")


if __name__ == "__main__":
    main()
