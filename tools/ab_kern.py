#!/usr/bin/env python
"""Per-kernel-class device ms of one synthetic frame (library per-kernel events, graphs off), median of --steps:
    STARSIM_LIB=... python tools/ab_kern.py --config T --mode t8"""
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
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--mode", default="t8")
    ap.add_argument("--n", type=int, default=0, help="override the config's star count")
    a = ap.parse_args()
    cfg = synth.with_R(synth.CONFIGS[a.config], a.R) if a.R else synth.CONFIGS[a.config]
    f = cfg.field(a.n) if a.n else cfg.field()
    dev = torch.device("cuda:0")
    x, y, m = (torch.from_numpy(v).to(dev) for v in (f.x, f.y, f.mag))
    out = torch.empty((cfg.H, cfg.W), dtype=torch.float32, device=dev)
    flush = torch.empty(64 << 20, dtype=torch.float32, device=dev)
    with Context(0) as ctx:
        ctx.set_tile_kernel(a.mode)
        for _ in range(3):
            ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
        per = []
        for i in range(a.steps):
            flush.fill_(float(i))
            torch.cuda.synchronize()
            ctx.profile(True)
            ctx.render(x, y, m, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0, out=out)
            per.append({k: v[0] for k, v in ctx.kernel_times().items()})
        names = list(per[0].keys())
        med = {k: sorted(p[k] for p in per)[len(per) // 2] * 1e3 for k in names}
    lib = os.path.basename(os.environ.get("STARSIM_LIB", "cur"))
    print(lib, a.config + (f"/R{a.R}" if a.R else "") + (f"/n{a.n}" if a.n else ""), a.mode, " ".join(f"{k}={v:.1f}us" for k, v in med.items() if v > 0))


if __name__ == "__main__":
    main()
