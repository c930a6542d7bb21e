"""Regression freeze of the pinned oracle and of the synth/ generators (tests/golden/oracle_c1.json)."""
import hashlib
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "oracle_c1.json")))


@pytest.mark.parametrize("name", ["C1", "C1_bright"])
def test_oracle_matches_frozen_c1(name):
    case = GOLD["cases"][name]
    c1 = synth.CONFIGS["C1"]
    lo, hi = case["mag_range"]
    f = c1.field(mag_lo=lo, mag_hi=hi)
    img, U = oracle.render(f.x, f.y, f.mag, case["W"], case["H"], case["sigma"], case["R"], case["A"],
                           return_units=True)
    assert U == case["U"]
    assert np.count_nonzero(img) == case["nonzero"]
    assert float(img.max()) == case["max"]
    for i, hx in case["samples"]:
        assert float(img.flat[i]) == float.fromhex(hx)
    assert abs(float(img.sum()) - case["sum"]) <= 1e-12 * case["sum"]


def test_synth_checksums_frozen():
    for key, want in GOLD["synth_checksums"].items():
        name = key.split("[")[0]
        cfg = synth.CONFIGS[name]
        f = cfg.field(n=100_000) if "[" in key else cfg.field()
        h = hashlib.sha256()
        for a in (f.x, f.y, f.mag):
            h.update(np.ascontiguousarray(a).tobytes())
        assert h.hexdigest()[:24] == want, key


def test_synth_fields_in_range():
    for cfg in synth.CONFIGS.values():
        f = cfg.field(n=min(cfg.n, 200_000))
        assert f.x.dtype == np.float32 and f.y.dtype == np.float32 and f.mag.dtype == np.float32
        assert (f.x >= 0).all() and (f.x < cfg.W).all() and (f.y >= 0).all() and (f.y < cfg.H).all()
        assert (f.mag >= 0).all() and (f.mag < 15).all()
