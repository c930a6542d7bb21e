"""Writes tests/golden/oracle_c1.json -- a regression fixture for the fp64 oracle.

Calls only oracle/ (and synth/ for the seeded inputs).  The paper prints no worked numeric example (PAPER.md: Figs 9-16
lost in extraction, Tables I-III are timings), so this fixture is NOT an independent pin: it freezes the oracle as
pinned by tests/test_oracle_pins.py, so any later change to the oracle's arithmetic shows up as a diff here and must
be justified in its commit message (task rule ③).  Also freezes the synth/ checksums of the configured fields.

Run:  python tests/golden/make_golden.py
"""
import hashlib
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth   # noqa: E402


def digest(*arrays):
    h = hashlib.sha256()
    for a in arrays:
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()[:24]


def main():
    out = {"source": "oracle/starsim_oracle.c via oracle.render (fp64); inputs synth.CONFIGS['C1'] seed 1",
           "cases": {}, "synth_checksums": {}}
    c1 = synth.CONFIGS["C1"]
    for name, (lo, hi) in {"C1": (0.0, 15.0), "C1_bright": (0.0, 2.0)}.items():
        f = c1.field(mag_lo=lo, mag_hi=hi)
        img, U = oracle.render(f.x, f.y, f.mag, c1.W, c1.H, c1.sigma, c1.R, 1.0, return_units=True)
        rng = np.random.default_rng(123)
        nz = np.flatnonzero(img)
        idx = np.sort(np.concatenate([rng.choice(nz, 48, replace=False), rng.integers(0, img.size, 16)]))
        out["cases"][name] = {
            "W": c1.W, "H": c1.H, "R": c1.R, "sigma": c1.sigma, "A": 1.0, "mag_range": [lo, hi],
            "U": int(U), "sum": float(img.sum()), "max": float(img.max()), "nonzero": int(nz.size),
            "samples": [[int(i), float(img.flat[i]).hex()] for i in idx],
        }
    for key, cfg in synth.CONFIGS.items():
        if cfg.n > 2_000_000:
            f = cfg.field(n=100_000)
            key = key + "[:100000]"
        else:
            f = cfg.field()
        out["synth_checksums"][key] = digest(f.x, f.y, f.mag)
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "oracle_c1.json")
    with open(path, "w") as fh:
        json.dump(out, fh, indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
