"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle on the same seeded inputs.

Tolerances (BASELINE.json north_star): float image max-abs error <= 1e-5 * peak and relative L2 error <= 1e-6;
quantised gray within +-1 LSB (bit-exact on identical fp32 input); binning (CSR) bit-exact.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import synth
from paper_conf_ipps_lizzh12_b200 import StarsimError

pytestmark = pytest.mark.gpu

MAX_ABS = 1e-5
REL_L2 = 1e-6


@pytest.fixture(scope="module")
def torch_dev():
    import torch
    if not torch.cuda.is_available():
        raise RuntimeError("GPU tests need a CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    return torch, torch.device("cuda:0")


@pytest.fixture(scope="module", params=["t8", "ws", "lists", "sb"])
def ctx(torch_dev, request):
    """Every test runs against the four tile kernels: "t8" (k_t8sort + the 8 x 8 lane-block kernel k_tile8, opt-in,
    R <= 17), "ws" (the warp-specialised sorted-corner-bin kernel for R <= 17, the list kernel above), "lists" (the
    per-block entry-list kernel for every R) and "sb" (the sorted-bin kernel with both roles in every warp; "auto"
    picks ws or sb by the expected list length, same images)."""
    from paper_conf_ipps_lizzh12_b200 import Context
    c = Context(0)
    c.set_tile_kernel(request.param)
    yield c
    c.close()


def to_dev(torch_dev, f):
    torch, dev = torch_dev
    return tuple(torch.from_numpy(np.ascontiguousarray(a)).to(dev) for a in (f.x, f.y, f.mag))


def errors(got, ref):
    peak = float(np.abs(ref).max()) if ref.size else 0.0
    if peak == 0.0:
        return float(np.abs(got).max()) if got.size else 0.0, 0.0
    return float(np.abs(got - ref).max()) / peak, float(np.linalg.norm(got - ref) / np.linalg.norm(ref))


def assert_parity(got, ref, what=""):
    ma, rl = errors(got.astype(np.float64), ref)
    log = os.environ.get("STARSIM_PARITY_LOG")
    if log:
        with open(log, "a") as fh:
            fh.write(json.dumps({"case": str(what), "max_abs_over_peak": ma, "rel_l2": rl}) + "\n")
    assert ma <= MAX_ABS and rl <= REL_L2, f"{what}: max_abs/peak={ma:.3e} rel_l2={rl:.3e}"


# ---------------------------------------------------------------- C1 (BASELINE configs[0]) and fig2

@pytest.mark.parametrize("mags", [(0.0, 15.0), (0.0, 2.0)])
@pytest.mark.parametrize("method", ["render", "render_atomic"])
def test_c1_parity(torch_dev, ctx, mags, method):
    cfg = synth.CONFIGS["C1"]
    f = cfg.field(mag_lo=mags[0], mag_hi=mags[1])
    ref = oracle.render(f.x, f.y, f.mag, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0)
    img = getattr(ctx, method)(*to_dev(torch_dev, f), cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0)
    assert_parity(img.cpu().numpy(), ref, f"C1 {method} {mags}")


@pytest.mark.parametrize("R", [10, 11])
def test_fig2_parity(torch_dev, ctx, R):
    cfg = synth.CONFIGS["fig2"]
    f = cfg.field(mag_lo=0.0, mag_hi=2.0)
    ref = oracle.render(f.x, f.y, f.mag, cfg.W, cfg.H, 1.0, R, 1.0)
    for method in ("render", "render_atomic"):
        img = getattr(ctx, method)(*to_dev(torch_dev, f), cfg.W, cfg.H, 1.0, R, 1.0)
        assert_parity(img.cpu().numpy(), ref, f"fig2 R={R} {method}")


# ---------------------------------------------------------------- randomized edge cases

def fuzz_cases(count=40):
    rng = np.random.default_rng(2024)
    cases = []
    for k in range(count):
        W, H = int(rng.integers(1, 300)), int(rng.integers(1, 300))
        n = int(rng.integers(0, 2000))
        R = int(rng.integers(1, 64))
        sigma = float(np.exp(rng.uniform(math.log(0.3), math.log(20.0))))
        cases.append((k, W, H, n, R, sigma))
    # explicit extremes: 1x1 image, empty catalogue, R = 1, largest R, R = 16 (window switch), tile-multiple sizes
    cases += [(100, 1, 1, 10, 1, 1.0), (101, 64, 64, 0, 5, 1.0), (102, 65, 33, 500, 16, 2.0),
              (103, 300, 200, 300, 255, 40.0), (104, 256, 256, 2000, 15, 2.5), (105, 33, 1, 50, 7, 1.0)]
    return cases


@pytest.mark.parametrize("case", fuzz_cases(), ids=lambda c: f"k{c[0]}-{c[1]}x{c[2]}-n{c[3]}-R{c[4]}")
def test_fuzz_parity(torch_dev, ctx, case):
    k, W, H, n, R, sigma = case
    f = synth.adversarial_field(n, W, H, R, seed=k + 7) if k % 2 else synth.uniform_field(n, W, H, seed=k, mag_hi=2.0)
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0)
    img = ctx.render(*to_dev(torch_dev, f), W, H, sigma, R, 1.0).cpu().numpy()
    if not np.any(ref):
        assert not np.any(img)
    else:
        assert_parity(img, ref, f"fuzz {case}")
    img_a = ctx.render_atomic(*to_dev(torch_dev, f), W, H, sigma, R, 1.0).cpu().numpy()
    if np.any(ref):
        assert_parity(img_a, ref, f"fuzz atomic {case}")


# ---------------------------------------------------------------- binning bit-exact (CSR)

@pytest.mark.parametrize("name,n,R,kind", [("small", 3000, 15, "uniform"), ("adv", 2000, 9, "adversarial"),
                                            ("wide", 500, 63, "uniform"), ("clustered", 20000, 15, "clustered"),
                                            ("r1", 5000, 1, "uniform")])
def test_bins_bit_exact(torch_dev, ctx, name, n, R, kind):
    W, H = 700, 530
    if kind == "adversarial":
        f = synth.adversarial_field(n, W, H, R, seed=5)
    elif kind == "clustered":
        f = synth.clustered_field(n, W, H, seed=6)
    else:
        f = synth.uniform_field(n, W, H, seed=7)
    ctx.render(*to_dev(torch_dev, f), W, H, R / 6, R, 1.0)
    tw, th, off, ids = ctx.get_bins()
    ntiles = (-(-W // tw)) * (-(-H // th))
    ref_off, ref_ids = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
    assert np.array_equal(off[:ntiles + 1], ref_off)
    assert np.array_equal(ids, ref_ids)


# ---------------------------------------------------------------- determinism and translation

def test_deterministic_and_tile_translation(torch_dev, ctx):
    torch, dev = torch_dev
    W, H = 512, 384
    f = synth.uniform_field(20000, W - 128, H - 64, seed=3, mag_hi=2.0)
    # positions on a 1/256 grid so that x + 128 and y + 64 are exact in fp32
    f = synth.Field(np.round(f.x * 256).astype(np.float32) / np.float32(256),
                    np.round(f.y * 256).astype(np.float32) / np.float32(256), f.mag)
    x, y, m = to_dev(torch_dev, f)
    a = ctx.render(x, y, m, W, H, 2.5, 15, 7.0)
    b = ctx.render(x, y, m, W, H, 2.5, 15, 7.0)
    assert torch.equal(a, b)
    # shift by whole tiles: every per-pixel sum sees the same stars in the same order
    c = ctx.render(x + 128, y + 64, m, W, H, 2.5, 15, 7.0)
    assert torch.equal(a[:H - 64, :W - 128], c[64:, 128:])


# ---------------------------------------------------------------- bands (multi-GPU decomposition, one device)

@pytest.mark.parametrize("G", [2, 4, 8])
def test_bands_concatenate_to_frame(torch_dev, ctx, G):
    torch, dev = torch_dev
    W, H = 640, 512
    f = synth.uniform_field(15000, W, H, seed=G, mag_hi=2.0)
    x, y, m = to_dev(torch_dev, f)
    full = ctx.render(x, y, m, W, H, 2.5, 15, 1.0)
    rows = H // G
    bands = [ctx.render_band(x, y, m, W, H, g * rows, rows, 2.5, 15, 1.0) for g in range(G)]
    assert torch.equal(torch.cat(bands, 0), full)


@pytest.mark.parametrize("R,sigma", [(11, 1.8), (41, 6.8), (65, 10.8)])
def test_unaligned_band_matches_oracle(torch_dev, ctx, R, sigma):
    W, H = 200, 150
    f = synth.adversarial_field(800, W, H, R, seed=9)
    ref = oracle.render_band(f.x, f.y, f.mag, W, H, 37, 61, sigma, R, 1.0)
    got = ctx.render_band(*to_dev(torch_dev, f), W, H, 37, 61, sigma, R, 1.0).cpu().numpy()
    assert_parity(got, ref, f"band 37+61 R={R}")


# ---------------------------------------------------------------- quantiser

@pytest.mark.parametrize("bits", [8, 16])
def test_quantize(torch_dev, ctx, bits):
    torch, dev = torch_dev
    cfg = synth.CONFIGS["C1"]
    f = cfg.field(mag_lo=0.0, mag_hi=4.0)
    A = synth.bench_gain(cfg.sigma, bits)
    img = ctx.render(*to_dev(torch_dev, f), cfg.W, cfg.H, cfg.sigma, cfg.R, A)
    q = ctx.quantize(img, bits).cpu().numpy()
    # bit-exact on the same fp32 input
    q_same = oracle.quantize(img.cpu().numpy().astype(np.float64), bits)
    assert np.array_equal(q, q_same)
    # within +-1 LSB of quantising the fp64 oracle image
    ref = oracle.render(f.x, f.y, f.mag, cfg.W, cfg.H, cfg.sigma, cfg.R, A)
    q_ref = oracle.quantize(ref, bits)
    d = np.abs(q.astype(np.int64) - q_ref.astype(np.int64))
    assert d.max() <= 1


def test_quantize_edge_values(torch_dev, ctx):
    torch, dev = torch_dev
    vals = np.array([0.0, -0.0, -3.0, 0.49999997, 0.5, 0.50000006, 1.5, 2.5, 254.5, 254.49998, 255.49998, 255.5,
                     1e30, np.inf, -np.inf, np.nan, 65534.5, 65535.5, 7.0], dtype=np.float32)
    for off in range(4):   # misaligned heads exercise the scalar path
        v = np.concatenate([np.zeros(off, np.float32), vals, np.full(5, 3.7, np.float32)])
        t = torch.from_numpy(v).to(dev)
        for bits in (8, 16):
            got = ctx.quantize(t, bits).cpu().numpy()
            assert np.array_equal(got, oracle.quantize(v.astype(np.float64), bits))


# ---------------------------------------------------------------- fused gray output (NEXT-1)

@pytest.mark.parametrize("bits", [8, 16])
@pytest.mark.parametrize("W,H", [(1024, 1024), (1003, 517)])
def test_render_gray_is_quantize_of_render(torch_dev, ctx, bits, W, H):
    """starsim_render_gray == starsim_quantize(starsim_render) bit for bit (same fp32 sums, same exact rounding), on
    vector-aligned and odd widths; and within +-1 LSB of quantising the fp64 oracle."""
    torch, dev = torch_dev
    f = synth.uniform_field(6000, W, H, seed=21, mag_lo=0.0, mag_hi=6.0)
    A = synth.bench_gain(1.5, bits)
    args = to_dev(torch_dev, f)
    img = ctx.render(*args, W, H, 1.5, 9, A)
    q_two_pass = ctx.quantize(img, bits).cpu().numpy()
    # into a buffer prefilled with a sentinel: every pixel must be written
    pre = torch.full((H, W), 0xAB, dtype=torch.uint8 if bits == 8 else torch.uint16, device=dev)
    q_fused = ctx.render_gray(*args, W, H, 1.5, 9, A, bits=bits, out=pre).cpu().numpy()
    assert q_fused.dtype == (np.uint8 if bits == 8 else np.uint16)
    assert np.array_equal(q_fused, q_two_pass)
    ref = oracle.quantize(oracle.render(f.x, f.y, f.mag, W, H, 1.5, 9, A, threads=_threads()), bits)
    assert np.abs(q_fused.astype(np.int64) - ref.astype(np.int64)).max() <= 1


# ---------------------------------------------------------------- heavy tiles (split into parts)

def _dense_field(n, W, H, cx, cy, spread, seed):
    u = synth.uniform01(seed, 0, 0, 3 * n)
    x = (cx + (u[:n] - 0.5) * spread).astype(np.float32)
    y = (cy + (u[n:2 * n] - 0.5) * spread).astype(np.float32)
    m = (u[2 * n:] * 3.0).astype(np.float32)
    return synth.Field(x, y, m)


def test_heavy_tile_split_parity_and_bands(torch_dev, ctx):
    """A tile with far more than SPLIT_LEN (1024) stars is rendered as several parts reduced in fixed order: parity
    against the oracle, run-to-run determinism, and bitwise equality of tile-aligned bands with the frame."""
    torch, dev = torch_dev
    W, H, R, sigma = 512, 384, 15, 2.5
    f = _dense_field(9000, W, H, 200.0, 150.0, 40.0, seed=31)
    args = to_dev(torch_dev, f)
    a = ctx.render(*args, W, H, sigma, R, 1.0)
    tw, th, off, ids = ctx.get_bins()
    assert int(np.diff(off).max()) > 4 * 1024  # some tile is split into >= 5 parts
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    assert_parity(a.cpu().numpy(), ref, "heavy tile")
    assert torch.equal(a, ctx.render(*args, W, H, sigma, R, 1.0))
    bands = [ctx.render_band(*args, W, H, g * 64, 64, sigma, R, 1.0) for g in range(H // 64)]
    assert torch.equal(torch.cat(bands, 0), a)


# ---------------------------------------------------------------- boundary contract (T1)

def test_einval_leaves_out_untouched(torch_dev, ctx):
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import StarsimError, starsim as S
    f = synth.uniform_field(10, 32, 32, seed=1)
    x, y, m = to_dev(torch_dev, f)
    out = torch.full((32, 32), 7.0, device=dev)
    bad = [dict(width=0), dict(height=40000), dict(sigma=0.0), dict(sigma=float("nan")), dict(roi=0),
           dict(roi=256), dict(gain=-1.0), dict(gain=float("inf"))]
    for b in bad:
        kw = dict(width=32, height=32, sigma=1.0, roi=5, gain=1.0)
        kw.update(b)
        with pytest.raises(StarsimError) as e:
            S.starsim_render(ctx.h, x, y, m, kw["width"], kw["height"], kw["sigma"], kw["roi"], kw["gain"], out)
        assert e.value.code == -1
    with pytest.raises(StarsimError):
        S.starsim_render_band(ctx.h, x, y, m, 32, 32, 20, 13, 1.0, 5, 1.0, out)
    with pytest.raises(StarsimError):
        S.starsim_quantize(ctx.h, out, 7, torch.empty(32, 32, dtype=torch.uint8, device=dev))
    torch.cuda.synchronize()
    assert bool((out == 7.0).all())


def test_empty_catalogue_gives_zero_image(torch_dev, ctx):
    torch, dev = torch_dev
    e = torch.empty(0, dtype=torch.float32, device=dev)
    out = torch.full((70, 90), 5.0, device=dev)
    ctx.render(e, e, e, 90, 70, 1.0, 5, 1.0, out=out)
    assert bool((out == 0).all())
    out.fill_(5.0)
    ctx.render_atomic(e, e, e, 90, 70, 1.0, 5, 1.0, out=out)
    assert bool((out == 0).all())


def test_upload_aos_splits_the_paper_record(torch_dev, ctx):
    f = synth.uniform_field(12345, 1000, 800, seed=2)
    x, y, m = ctx.upload_aos(f.aos())
    assert np.array_equal(x.cpu().numpy(), f.x) and np.array_equal(y.cpu().numpy(), f.y)
    assert np.array_equal(m.cpu().numpy(), f.mag)


def test_kernel_times_recorded(torch_dev, ctx):
    cfg = synth.CONFIGS["C1"]
    f = cfg.field()
    args = to_dev(torch_dev, f)
    ctx.profile(True)
    ctx.render(*args, cfg.W, cfg.H, cfg.sigma, cfg.R, 1.0)
    t = ctx.kernel_times()
    ctx.profile(False)
    # the t8 mode adds its corner-bin sort (k_t8sort) to the sort class
    # sb may hand the light tiles to k_tile_lite (a second launch); C1's 1000 stars are binned by k_dsmall alone
    # (class "prep"), the t8 mode adds its corner-bin sort (k_t8sort) to the sort class
    assert t["tile"][1] in (1, 2) and t["tile"][0] > 0 and t["prep"][1] == 1 and t["sort"][1] in (0, 1)
    assert t["csr"][1] == 0
    assert t["route"][1] == 0
    ctx.profile(True)
    ctx.route_band(*args, cfg.H, 0, 64, cfg.R)
    t = ctx.kernel_times()
    ctx.profile(False)
    assert t["route"][1] == 2 and t["route"][0] > 0


# ---------------------------------------------------------------- B200-scale frames (full images, threaded oracle)

def _threads():
    import os
    return max(1, os.cpu_count() or 1)


@pytest.mark.parametrize("name", ["C2", "T"])
def test_full_frame_parity(torch_dev, ctx, name):
    cfg = synth.CONFIGS[name]
    f = cfg.field(mag_lo=0.0, mag_hi=15.0)
    A = synth.bench_gain(cfg.sigma)
    ref = oracle.render(f.x, f.y, f.mag, cfg.W, cfg.H, cfg.sigma, cfg.R, A, threads=_threads())
    img = ctx.render(*to_dev(torch_dev, f), cfg.W, cfg.H, cfg.sigma, cfg.R, A).cpu().numpy()
    assert_parity(img, ref, name)


@pytest.mark.parametrize("R", [3, 15, 21, 31, 47, 63])
def test_c4_clustered_parity(torch_dev, ctx, R):
    cfg = synth.with_R(synth.CONFIGS["C4"], R)
    f = cfg.field()
    A = synth.bench_gain(cfg.sigma)
    ref = oracle.render(f.x, f.y, f.mag, cfg.W, cfg.H, cfg.sigma, cfg.R, A, threads=_threads())
    img = ctx.render(*to_dev(torch_dev, f), cfg.W, cfg.H, cfg.sigma, cfg.R, A).cpu().numpy()
    assert_parity(img, ref, cfg.name)


def test_c5_whole_bands(torch_dev, ctx):
    """16384^2, 10M stars, R=15 in the bench's launch configuration (32,768 tiles: the atomic-slot binning and its
    two-kernel tile scan k_scan_a / k_scan_b): 8 whole 64-row bands spread over the frame (first, last, both sides of
    the tile-row and half-frame boundaries) against the oracle's band render."""
    cfg = synth.CONFIGS["C5"]
    f = cfg.field()
    A = synth.bench_gain(cfg.sigma)
    img = ctx.render(*to_dev(torch_dev, f), cfg.W, cfg.H, cfg.sigma, cfg.R, A)
    for row0 in [0, 64, 4032, 8128, 8192, 12288, 16256, 16320]:
        ref = oracle.render_band(f.x, f.y, f.mag, cfg.W, cfg.H, row0, 64, cfg.sigma, cfg.R, A)
        assert_parity(img[row0:row0 + 64].cpu().numpy(), ref, f"C5 band {row0}")


@pytest.mark.parametrize("mode", ["auto", "atomic"])
def test_bins_bit_exact_over_4096_tiles(torch_dev, mode):
    """CSR bit-exact on a frame of more than 4,096 tiles (8320 x 4096: 65 x 64 = 4,160 tiles, 300K stars), which
    runs the two-kernel tile scan (k_scan_a / k_scan_b; the deterministic binning covers <= 2,048 tiles, so both
    binning settings take the atomic-slot pipeline here), and the image against the oracle on sampled bands."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    W, H, R = 8320, 4096, 15
    f = synth.uniform_field(300000, W, H, seed=41, mag_hi=2.0)
    with Context(0) as c:
        c.set_binning(mode)
        img = c.render(*to_dev(torch_dev, f), W, H, 2.5, R, 1.0)
        tw, th, off, ids = c.get_bins()
    ntiles = (-(-W // tw)) * (-(-H // th))
    assert ntiles > 4096
    ref_off, ref_ids = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
    assert np.array_equal(off[:ntiles + 1], ref_off)
    assert np.array_equal(ids, ref_ids)
    for row0 in [0, 2048, 4032]:
        ref = oracle.render_band(f.x, f.y, f.mag, W, H, row0, 64, 2.5, R, 1.0)
        assert_parity(img[row0:row0 + 64].cpu().numpy(), ref, f">4096 tiles band {row0}")


# ---------------------------------------------------------------- NEXT-2: pixel-integrated PSF

@pytest.fixture()
def ctx_integrated(ctx):
    ctx.set_psf("integrated")
    yield ctx
    ctx.set_psf("point")


@pytest.mark.parametrize("W,H,n,R,sigma", [(1024, 1024, 1000, 5, 1.0), (301, 177, 3000, 15, 2.5),
                                           (256, 256, 400, 63, 10.5), (120, 90, 500, 7, 0.4),
                                           (4096, 2048, 5000, 15, 2.5)])  # sparse: k_tile_lite
def test_integrated_psf_parity(torch_dev, ctx_integrated, W, H, n, R, sigma):
    f = synth.uniform_field(n, W, H, seed=R + n, mag_lo=0.0, mag_hi=3.0)
    args = to_dev(torch_dev, f)
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads(), psf="integrated")
    assert_parity(ctx_integrated.render(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref, f"integrated tiled {W}x{H}")
    assert_parity(ctx_integrated.render_atomic(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref,
                  f"integrated atomic {W}x{H}")


def test_integrated_psf_mode_switch_and_einval(torch_dev, ctx):
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import StarsimError
    f = synth.uniform_field(500, 200, 200, seed=3, mag_lo=0.0, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    a = ctx.render(*args, 200, 200, 1.5, 9, 1.0)
    ctx.set_psf("integrated")
    b = ctx.render(*args, 200, 200, 1.5, 9, 1.0)
    ctx.set_psf("point")
    c = ctx.render(*args, 200, 200, 1.5, 9, 1.0)
    assert torch.equal(a, c) and not torch.equal(a, b)
    with pytest.raises(StarsimError):
        ctx.set_psf(7)


# ---------------------------------------------------------------- the two binning pipelines and tile kernels agree

@pytest.mark.parametrize("name,W,H,n,R,kind", [("uniform", 700, 530, 20000, 15, "uniform"),
                                                ("clustered", 1024, 768, 30000, 9, "clustered"),
                                                ("adversarial", 300, 200, 3000, 5, "adversarial"),
                                                ("wide", 640, 512, 2000, 65, "uniform")])
def test_binning_pipelines_identical(torch_dev, name, W, H, n, R, kind):
    """dbin.cu (deterministic counting sort) and bin.cu (atomic slots + per-tile sort) build the same CSR, so the
    image is bitwise the same; both equal the oracle's bins (reading R18)."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    if kind == "clustered":
        f = synth.clustered_field(n, W, H, seed=21)
    elif kind == "adversarial":
        f = synth.adversarial_field(n, W, H, R, seed=22)
    else:
        f = synth.uniform_field(n, W, H, seed=23, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    res = {}
    for mode in ("auto", "atomic"):
        with Context(0) as c:
            c.set_binning(mode)
            img = c.render(*args, W, H, R / 6, R, 1.0)
            res[mode] = (img, c.get_bins())
    (ia, (tw, th, oa, da)), (ib, (_, _, ob, db)) = res["auto"], res["atomic"]
    ntiles = (-(-W // tw)) * (-(-H // th))
    assert np.array_equal(oa[:ntiles + 1], ob[:ntiles + 1]) and np.array_equal(da, db)
    assert torch.equal(ia, ib)
    ref_off, ref_ids = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
    assert np.array_equal(oa[:ntiles + 1], ref_off) and np.array_equal(da, ref_ids)


@pytest.mark.parametrize("R,psf", [(18, "point"), (25, "integrated"), (33, "point"), (34, "point"), (49, "point"),
                                   (50, "integrated"), (65, "point")])
def test_wide_roi_kernel(torch_dev, R, psf):
    """k_tile_wide (17 < R <= 65, sorted corner bins over <= 5 bands x 9 strips) at each band-slot count's edges:
    parity against the oracle, within rounding of the list kernel k_tile (a different fixed order), deterministic,
    and tile-aligned bands bitwise the frame -- on a 537 x 411 frame (ragged tiles) with stars off every border."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    W, H, sigma = 537, 411, R / 6.0
    f = synth.adversarial_field(4000, W, H, R, seed=R)
    args = to_dev(torch_dev, f)
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads(), psf=psf)
    out = {}
    for mode in ("auto", "lists"):
        with Context(0) as c:
            c.set_tile_kernel(mode)
            c.set_psf(psf)
            a = c.render(*args, W, H, sigma, R, 1.0)
            assert_parity(a.cpu().numpy(), ref, f"wide R={R} {psf} {mode}")
            if mode == "auto":
                assert torch.equal(a, c.render(*args, W, H, sigma, R, 1.0))
                bands = [c.render_band(*args, W, H, g * 64, min(64, H - g * 64), sigma, R, 1.0)
                         for g in range(-(-H // 64))]
                assert torch.equal(torch.cat(bands, 0), a)
            out[mode] = a.double().cpu().numpy()
    peak = float(np.abs(ref).max())
    assert float(np.abs(out["auto"] - out["lists"]).max()) <= 1e-5 * peak


@pytest.mark.parametrize("psf", ["point", "integrated"])
@pytest.mark.parametrize("W,H,n,R,seed,kind", [(537, 411, 4000, 33, 5, "adv"), (1000, 700, 20000, 47, 6, "uniform"),
                                               (512, 384, 9000, 63, 7, "dense")])
def test_wide_ws_equals_sync_bitwise(torch_dev, psf, W, H, n, R, seed, kind):
    """k_tile_wws (warp-specialised, mode ws) and k_tile_wide (both roles in every warp, modes auto / sb) sum every
    pixel in the same order: bitwise-identical images, incl. heavy tiles split into parts."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    if kind == "dense":
        f = _dense_field(n, W, H, 200.0, 150.0, 40.0, seed=seed)
    elif kind == "adv":
        f = synth.adversarial_field(n, W, H, R, seed=seed)
    else:
        f = synth.uniform_field(n, W, H, seed=seed, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    out = {}
    for mode in ("ws", "sb"):
        with Context(0) as c:
            c.set_tile_kernel(mode)
            c.set_psf(psf)
            out[mode] = c.render(*args, W, H, R / 6.0, R, 1.0)
    assert torch.equal(out["ws"], out["sb"])


@pytest.mark.parametrize("R", [31, 63])
def test_wide_roi_heavy_tiles(torch_dev, ctx, R):
    """Clustered wide-ROI field with tiles of > 4 x SPLIT_LEN stars (split into parts): parity, determinism, bands
    bitwise the frame -- for k_tile_wide (auto / sb / ws / t8 modes) and k_tile (lists)."""
    torch, dev = torch_dev
    W, H, sigma = 512, 384, R / 6.0
    f = _dense_field(9000, W, H, 200.0, 150.0, 40.0, seed=33)
    args = to_dev(torch_dev, f)
    a = ctx.render(*args, W, H, sigma, R, 1.0)
    tw, th, off, ids = ctx.get_bins()
    assert int(np.diff(off).max()) > 4 * 1024
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    assert_parity(a.cpu().numpy(), ref, f"wide heavy R={R}")
    assert torch.equal(a, ctx.render(*args, W, H, sigma, R, 1.0))
    bands = [ctx.render_band(*args, W, H, g * 64, 64, sigma, R, 1.0) for g in range(H // 64)]
    assert torch.equal(torch.cat(bands, 0), a)


def test_tile_kernels_agree_within_rounding(torch_dev):
    """k_tile_sb and k_tile sum each pixel in different (fixed) orders: equal up to fp32 rounding, both at parity."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    W, H, R = 1000, 700, 15
    f = synth.uniform_field(60000, W, H, seed=24, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    out = {}
    for mode in ("auto", "lists"):
        with Context(0) as c:
            c.set_tile_kernel(mode)
            out[mode] = c.render(*args, W, H, 2.5, R, 1.0).double().cpu().numpy()
    ref = oracle.render(f.x, f.y, f.mag, W, H, 2.5, R, 1.0, threads=_threads())
    for mode in out:
        assert_parity(out[mode], ref, f"tile kernel {mode}")
    peak = float(np.abs(ref).max())
    assert float(np.abs(out["auto"] - out["lists"]).max()) <= 1e-5 * peak


@pytest.mark.parametrize("psf", ["point", "integrated"])
@pytest.mark.parametrize("W,H,n,R,seed", [(1000, 700, 60000, 15, 24), (4096, 4096, 1000000, 15, 1),
                                          (301, 177, 3000, 17, 5), (700, 500, 0, 9, 6),
                                          (4096, 4096, 2000, 15, 7), (2048, 2048, 20000, 9, 8),
                                          (1024, 1024, 1000, 5, 9), (515, 301, 700, 17, 10), (256, 256, 300, 1, 11),
                                          (640, 384, 2500, 12, 12)])
def test_ws_equals_sb_bitwise(torch_dev, psf, W, H, n, R, seed):
    """The warp-specialised kernel (auto) sums every pixel in k_tile_sb's order: the images are identical bit for bit,
    also with heavy tiles split into parts (the clustered field) and with the integrated PSF.  The sparse fields put
    most tiles on k_tile_sb's light-item path (lists of <= SB_LITE_MAX stars, evaluated per lane without slots),
    which must give the chunked path's bits exactly (ws has no light path)."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    f = synth.uniform_field(n, W, H, seed=seed, mag_hi=15.0)
    if n == 60000:
        f = _dense_field(n, W, H, 500.0, 350.0, 120.0, seed=seed)
    args = to_dev(torch_dev, f)
    out = {}
    for mode in ("ws", "sb"):
        with Context(0) as c:
            c.set_tile_kernel(mode)
            c.set_psf(psf)
            out[mode] = c.render(*args, W, H, R / 6, R, 1.0)
    assert torch.equal(out["ws"], out["sb"])


@pytest.mark.parametrize("W,H,n,R,seed", [(1000, 700, 60000, 15, 24), (4096, 4096, 1000000, 15, 1),
                                          (515, 301, 700, 17, 10), (700, 500, 0, 9, 6)])
def test_ws_presorted_equals_sb_bitwise(torch_dev, monkeypatch, W, H, n, R, seed):
    """k_tile_ws fed by k_chsort (STARSIM_WS_PRESORT=1: every 256-star chunk presorted by corner bin, records in walk
    order) gives k_tile_sb's image bit for bit -- split heavy tiles, empty frames and R = 17 included."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    f = synth.uniform_field(n, W, H, seed=seed, mag_hi=15.0)
    if n == 60000:
        f = _dense_field(n, W, H, 500.0, 350.0, 120.0, seed=seed)
    args = to_dev(torch_dev, f)
    monkeypatch.setenv("STARSIM_WS_PRESORT", "1")
    with Context(0) as c:
        c.set_tile_kernel("ws")
        pre = c.render(*args, W, H, R / 6, R, 1.0)
    monkeypatch.delenv("STARSIM_WS_PRESORT")
    with Context(0) as c:
        c.set_tile_kernel("sb")
        ref = c.render(*args, W, H, R / 6, R, 1.0)
    assert torch.equal(pre, ref)


@pytest.mark.parametrize("W,H,n,R,seed", [(4096, 4096, 1000000, 15, 3), (700, 530, 20000, 9, 4),
                                          (1000, 700, 60000, 15, 24), (640, 1024, 5000, 31, 5)])
def test_fused_binning_same_csr_and_image(torch_dev, monkeypatch, W, H, n, R, seed):
    """k_dfused (STARSIM_DFUSED=1: count, column scan and placement in one cooperative launch with two grid barriers)
    writes the CSR of the oracle's bins bit for bit and the same image as the three-kernel binning."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    f = synth.uniform_field(n, W, H, seed=seed, mag_hi=15.0)
    if n == 60000:
        f = _dense_field(n, W, H, 500.0, 350.0, 120.0, seed=seed)
    args = to_dev(torch_dev, f)
    with Context(0) as c:
        ref = c.render(*args, W, H, 2.5, R, 1.0)
    monkeypatch.setenv("STARSIM_DFUSED", "1")
    with Context(0) as c:
        img = c.render(*args, W, H, 2.5, R, 1.0)
        tw, th, off, ids = c.get_bins()
    assert torch.equal(img, ref)
    ro, ri = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
    assert np.array_equal(off[:ro.size], ro) and np.array_equal(ids, ri)


@pytest.mark.parametrize("W,H,n,R,seed,kind", [(1024, 1024, 1000, 5, 1, "uniform"), (4096, 4096, 1000, 11, 2, "uniform"),
                                               (700, 530, 1024, 15, 3, "adv"), (300, 200, 900, 17, 4, "dense"),
                                               (129, 65, 1, 9, 5, "uniform"), (256, 256, 0, 7, 6, "uniform"),
                                               (1024, 1024, 2252, 11, 7, "uniform"), (4096, 2048, 4096, 15, 8, "adv"),
                                               (300, 200, 4000, 15, 9, "dense"),  # > 1,024 stars in a tile
                                               (4096, 2048, 8000, 11, 10, "uniform"), (1024, 1024, 30000, 9, 11, "uniform"),
                                               (256, 192, 9000, 13, 12, "dense")])
def test_sparse_path_is_bitwise_sb(torch_dev, W, H, n, R, seed, kind):
    """STARSIM_TILE_AUTO renders small catalogues (<= 32,768 stars, stars x tiles <= 8 M) through the sparse path (k_srec + k_tile_sparse: no
    binning launches, every tile CTA builds its own list; lists over 1,024 stars summed in segments, reading R19):
    the same image as k_tile_sb bit for bit -- point and
    integrated PSF, square and circle ROI, fp32 and u8 -- at parity with the oracle, bands bitwise the frame, and
    starsim_get_bins afterwards (binned on demand) the oracle's CSR."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    if kind == "adv":
        f = synth.adversarial_field(n, W, H, R, seed=seed)
    elif kind == "dense":
        f = _dense_field(n, W, H, 150.0, 100.0, 20.0, seed=seed)
    else:
        f = synth.uniform_field(n, W, H, seed=seed, mag_hi=15.0)
    args = to_dev(torch_dev, f) if n else (torch.empty(0, device=dev),) * 3
    sigma = R / 6
    with Context(0) as a, Context(0) as b:
        b.set_tile_kernel("sb")
        for psf in ("point", "integrated"):
            for roi in ("square", "circle"):
                for c in (a, b):
                    c.set_psf(psf)
                    c.set_roi(roi)
                ia = a.render(*args, W, H, sigma, R, 1.0)
                assert torch.equal(ia, b.render(*args, W, H, sigma, R, 1.0)), (psf, roi)
                ga = a.render_gray(*args, W, H, sigma, R, 1.0, bits=8)
                assert torch.equal(ga, b.render_gray(*args, W, H, sigma, R, 1.0, bits=8)), (psf, roi)
        for c in (a, b):
            c.set_psf("point")
            c.set_roi("square")
        img = a.render(*args, W, H, sigma, R, 1.0)
        if n:
            assert_parity(img.cpu().numpy(), oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0), f"sparse {W}x{H}")
        bands = [a.render_band(*args, W, H, g * 64, min(64, H - g * 64), sigma, R, 1.0) for g in range(-(-H // 64))]
        assert torch.equal(torch.cat(bands, 0), img)
        a.render(*args, W, H, sigma, R, 1.0)
        tw, th, off, ids = a.get_bins()
        ro, ri = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
        assert np.array_equal(off[:ro.size], ro) and np.array_equal(ids, ri)


def test_mode_setters_einval(torch_dev):
    from paper_conf_ipps_lizzh12_b200 import Context, StarsimError
    with Context(0) as c:
        for fn in (c.set_binning, c.set_tile_kernel, c.set_roi):
            with pytest.raises(StarsimError):
                fn(7)


# ---------------------------------------------------------------- fused band exchange (multi-destination epilogue)

@pytest.mark.parametrize("tile_kernel", ["auto", "ws", "lists", "sb"])
def test_render_band_to_writes_every_destination(torch_dev, tile_kernel):
    """starsim_render_band_to: every band lands, bitwise equal to starsim_render_band, in each destination frame at its
    rows (the epilogue of the fused exchange; on one GPU the destinations are local frames standing in for peers)."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    W, H, R, G = 640, 512, 15, 4
    f = synth.uniform_field(12000, W, H, seed=31, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    with Context(0) as c:
        c.set_tile_kernel(tile_kernel)
        full = c.render(*args, W, H, 2.5, R, 1.0)
        frames = [torch.full((H, W), -1.0, device=dev) for _ in range(3)]
        rows = H // G
        for g in range(G):
            c.render_band_to(*args, W, H, g * rows, rows, 2.5, R, 1.0, frames)
        for fr in frames:
            assert torch.equal(fr, full)
        # a single destination with an unaligned band leaves the other rows untouched
        one = torch.full((H, W), -1.0, device=dev)
        c.render_band_to(*args, W, H, 37, 100, 2.5, R, 1.0, [one])
        band = c.render_band(*args, W, H, 37, 100, 2.5, R, 1.0)
        assert torch.equal(one[37:137], band)
        assert bool((one[:37] == -1).all()) and bool((one[137:] == -1).all())


def test_render_band_to_einval(torch_dev):
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context, StarsimError
    f = synth.uniform_field(10, 64, 64, seed=1)
    args = to_dev(torch_dev, f)
    with Context(0) as c:
        fr = torch.zeros((64, 64), device=dev)
        with pytest.raises(StarsimError):
            c.render_band_to(*args, 64, 64, 0, 64, 1.0, 5, 1.0, [fr] * 9)
        with pytest.raises(StarsimError):
            c.render_band_to(*args, 64, 64, 60, 10, 1.0, 5, 1.0, [fr])
        with pytest.raises(StarsimError):
            c.render_band_to(*args, 64, 64, 0, 64, 1.0, 5, 1.0, [fr, 0])


def test_fused_frame_single_rank(torch_dev):
    """FusedFrame (symmetric-memory frame + render_band_to + device barrier) on a one-rank NCCL group: the frame equals
    the plain render bitwise.  Skipped where this torch build / driver has no symmetric memory."""
    torch, dev = torch_dev
    import torch.distributed as dist
    from paper_conf_ipps_lizzh12_b200 import Context
    from paper_conf_ipps_lizzh12_b200 import dist as sdist
    own = not dist.is_initialized()
    if own:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        try:
            ff = sdist.FusedFrame(384, 512, dev)
        except Exception as e:  # no symmetric memory support here
            pytest.skip(f"symmetric memory unavailable: {e}")
        f = synth.uniform_field(5000, 512, 384, seed=32, mag_hi=2.0)
        args = to_dev(torch_dev, f)
        with Context(0) as c:
            ref = c.render(*args, 512, 384, 2.5, 15, 1.0)
            got = ff.render(c, *args, 2.5, 15, 1.0)
            torch.cuda.synchronize()
            assert torch.equal(got, ref)
    finally:
        if own:
            dist.destroy_process_group()


# ---------------------------------------------------------------- NEXT-4: lookup-table (adaptive simulator) comparison

@pytest.mark.parametrize("W,H,n,R,sigma,kind", [(1024, 1024, 1000, 5, 1.0, "uniform"), (700, 530, 5000, 15, 2.5, "adv"),
                                                 (300, 200, 2000, 10, 1.7, "uniform"), (512, 384, 3000, 63, 10.5, "uniform")])
def test_lut_parity(torch_dev, ctx, W, H, n, R, sigma, kind):
    """starsim_render_lut against the oracle's render_lut (reading R20), and exact vs render for pixel-centred stars."""
    f = synth.adversarial_field(n, W, H, R, seed=41) if kind == "adv" else synth.uniform_field(n, W, H, seed=42,
                                                                                                  mag_hi=2.0)
    ref = oracle.render_lut(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    got = ctx.render_lut(*to_dev(torch_dev, f), W, H, sigma, R, 1.0).cpu().numpy()
    assert_parity(got, ref, f"lut {W}x{H} R={R}")
    if R % 2:
        fc = synth.Field(np.round(f.x).astype(np.float32), np.round(f.y).astype(np.float32), f.mag)
        ref_c = oracle.render(fc.x, fc.y, fc.mag, W, H, sigma, R, 1.0, threads=_threads())
        got_c = ctx.render_lut(*to_dev(torch_dev, fc), W, H, sigma, R, 1.0).cpu().numpy()
        assert_parity(got_c, ref_c, f"lut pixel-centred R={R}")


def test_lut_einval(torch_dev, ctx):
    from paper_conf_ipps_lizzh12_b200 import StarsimError
    f = synth.uniform_field(10, 64, 64, seed=1)
    with pytest.raises(StarsimError):
        ctx.render_lut(*to_dev(torch_dev, f), 64, 64, 1.0, 65, 1.0)


# ---------------------------------------------------------------- NEXT-3: the "pixel circle" ROI (reading R21)

@pytest.mark.parametrize("W,H,n,R,sigma,kind", [(1024, 1024, 1000, 5, 1.0, "uniform"), (700, 530, 5000, 15, 2.5, "adv"),
                                                 (300, 200, 2000, 10, 1.7, "uniform"), (512, 384, 3000, 63, 10.5, "uniform"),
                                                 (4096, 2048, 6000, 15, 2.5, "adv"),  # sparse: k_tile_lite
                                                 (700, 530, 6000, 21, 3.5, "adv"), (640, 520, 8000, 31, 5.2, "uniform"),
                                                 (600, 500, 4000, 41, 6.8, "adv")])    # R > 17: k_tile's masked walk
def test_circle_roi_parity(torch_dev, ctx, W, H, n, R, sigma, kind):
    """starsim_set_roi(CIRCLE): the atomic, lookup-table and tiled renders against the oracle's circle ROI (the tiled
    path masks the circle in k_tile_sb's walk for R <= 17 and in k_tile's above; bands bitwise the frame); the square
    ROI works again once it is back."""
    f = synth.adversarial_field(n, W, H, R, seed=43) if kind == "adv" else synth.uniform_field(n, W, H, seed=44,
                                                                                                  mag_hi=2.0)
    args = to_dev(torch_dev, f)
    ctx.set_roi("circle")
    try:
        ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads(), roi="circle")
        assert_parity(ctx.render_atomic(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref, f"circle atomic R={R}")
        if R <= 63:
            ref_l = oracle.render_lut(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads(), roi="circle")
            assert_parity(ctx.render_lut(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref_l, f"circle lut R={R}")
        img = ctx.render(*args, W, H, sigma, R, 1.0)
        assert_parity(img.cpu().numpy(), ref, f"circle tiled R={R}")
        bands = [ctx.render_band(*args, W, H, g * 64, min(64, H - g * 64), sigma, R, 1.0)
                 for g in range(-(-H // 64))]
        assert torch_dev[0].equal(torch_dev[0].cat(bands, 0), img)
        g8 = ctx.render_gray(*args, W, H, sigma, R, 1.0, bits=8)
        assert torch_dev[0].equal(g8, ctx.quantize(img, 8))
    finally:
        ctx.set_roi("square")
    ref_sq = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    assert_parity(ctx.render(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref_sq, f"square after circle R={R}")


@pytest.mark.parametrize("n,W,H,R,G,kind", [(0, 64, 64, 5, 1, "uniform"), (1, 64, 64, 5, 1, "uniform"),
                                             (20001, 700, 530, 9, 3, "adv"), (50000, 640, 1024, 15, 4, "uniform"),
                                             (1000000, 4096, 4096, 15, 8, "uniform")])
def test_route_band_parity(torch_dev, ctx, n, W, H, R, G, kind):
    """starsim_route_band against oracle.route_band (the exact ROI-row rule, pinned in test_dist_cpu.py): the routed
    count and the compacted x, y, mag bit for bit, in catalogue order, for every band -- ragged 4096-star blocks,
    non-finite and far-off coordinates (adversarial field), an empty catalogue, and the full 1M-star T catalogue."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import dist as sdist
    f = synth.adversarial_field(n, W, H, R, seed=12) if kind == "adv" else synth.uniform_field(n, W, H, seed=12)
    args = to_dev(torch_dev, f) if n else (torch.empty(0, device=dev),) * 3
    for g in range(G):
        row0, rows = sdist.band_rows(H, G, g)
        if rows == 0:
            continue
        xo, yo, mo, nd = ctx.route_band(*args, H, row0, rows, R)
        torch.cuda.synchronize()
        idx = oracle.route_band(f.y, R, row0, rows)
        k = int(nd.item())
        assert k == idx.size, (g, k, idx.size)
        for got, ref in ((xo, f.x), (yo, f.y), (mo, f.mag)):
            assert np.array_equal(got[:k].cpu().numpy().view(np.uint32), ref[idx].view(np.uint32)), g


@pytest.mark.parametrize("W,H,n,R,G", [(640, 1024, 40000, 15, 4),      # bands of <= 2048 tiles: dbin.cu binning
                                       (16384, 2176, 200000, 15, 2),   # 2176 tiles per band: bin.cu's pipeline
                                       (640, 1024, 20000, 47, 4)])     # wide ROIs: k_tile_wide (256-star parts)
def test_band_from_routed_catalogue_is_bitwise_the_band(torch_dev, ctx, W, H, n, R, G):
    """A band rendered from the device-routed catalogue (starsim_route_band + starsim_set_star_count:
    Context.render_band_routed, what every rank does per frame for N > 1) equals the band rendered from the whole
    catalogue bit for bit -- same tile lists in the same relative order -- for every tile kernel and both binning
    pipelines; the CUDA graph of the routed render replays with a count that changes between frames."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import dist as sdist
    f = synth.uniform_field(n, W, H, seed=77, mag_hi=15.0)
    full = to_dev(torch_dev, f)
    st = torch.cuda.Stream(dev)  # a non-default stream: the renders go through the captured CUDA graph
    with torch.cuda.stream(st):
        for g in range(G):
            row0, rows = sdist.band_rows(H, G, g)
            a = ctx.render_band(*full, W, H, row0, rows, 2.5, R, 1.0, stream=st)
            b = ctx.render_band_routed(*full, W, H, row0, rows, 2.5, R, 1.0, stream=st)
            st.synchronize()
            assert torch.equal(a, b), g
        # same buffers, new content and a different routed count: the replayed graph reads the new device count
        row0, rows = sdist.band_rows(H, G, 0)
        out = torch.empty((rows, W), dtype=torch.float32, device=dev)
        ctx.render_band_routed(*full, W, H, row0, rows, 2.5, R, 1.0, out=out, stream=st)
        full[1][: n // 2] = full[1][: n // 2] * 0.5  # move half the stars towards row 0: more of them in band 0
        ctx.render_band_routed(*full, W, H, row0, rows, 2.5, R, 1.0, out=out, stream=st)
        a = ctx.render_band(*full, W, H, row0, rows, 2.5, R, 1.0, stream=st)
        st.synchronize()
        assert torch.equal(a, out)
        # a band no star reaches: a zero image from a zero device count
        far = tuple(t.clone() for t in full)
        far[1].fill_(float(H + 1000))
        z = ctx.render_band_routed(*far, W, H, row0, rows, 2.5, R, 1.0, stream=st)
        st.synchronize()
        assert int(ctx._route_buf[3].item()) == 0 and not z.any()


def test_set_star_count_semantics_and_einval(torch_dev, ctx):
    """With a device count set, tiled renders take the first min(n, count) stars; the star-centric renders refuse."""
    torch, dev = torch_dev
    W, H, R = 300, 200, 9
    f = synth.uniform_field(5000, W, H, seed=5)
    args = to_dev(torch_dev, f)
    cnt = torch.tensor([1234], dtype=torch.int32, device=dev)
    ctx.set_star_count(cnt)
    try:
        a = ctx.render(*args, W, H, 1.5, R, 1.0)
        with pytest.raises(StarsimError):
            ctx.render_atomic(*args, W, H, 1.5, R, 1.0)
        with pytest.raises(StarsimError):
            ctx.render_lut(*args, W, H, 1.5, R, 1.0)
        cnt.fill_(10 ** 6)  # larger than n: all n stars
        c = ctx.render(*args, W, H, 1.5, R, 1.0)
    finally:
        ctx.set_star_count(None)
    b = ctx.render(*(t[:1234] for t in args), W, H, 1.5, R, 1.0)
    assert torch.equal(a, b)
    assert torch.equal(c, ctx.render(*args, W, H, 1.5, R, 1.0))
    with pytest.raises(ValueError):  # the binding checks output sizes before the library is called
        ctx.render(*args, W, H, 1.5, R, 1.0, out=torch.empty((H - 1, W), dtype=torch.float32, device=dev))
    with pytest.raises(ValueError):
        ctx.render_band(*args, W, H, 0, 64, 1.5, R, 1.0, out=torch.empty((63, W), dtype=torch.float32, device=dev))


def test_unsplit_huge_tile_lists(torch_dev, ctx):
    """More heavy-tile parts than the partial-buffer pool holds (PART_CAP = 2048): the frame's heavy tiles are not
    split and a work item carries a whole tile list of ~10^5 stars.  Every tile kernel then sums it in SPLIT_LEN
    segments exactly as it would sum the parts (reading R19; the segment partials go through a per-CTA scratch tile),
    so the north-star tolerance holds (~120,000 fp32 additions per pixel, 2M stars in 60 x 60 px, each sequential
    chain <= 1,024 stars long) and the result is bitwise the same whether or not the planner split the tile: the
    bands below have fewer heavy tiles each, so they are split, and still equal the frame bit for bit."""
    torch, dev = torch_dev
    W, H, R, sigma = 256, 256, 15, 2.5
    f = _dense_field(2000000, W, H, 130.0, 130.0, 60.0, seed=5)
    args = to_dev(torch_dev, f)
    a = ctx.render(*args, W, H, sigma, R, 1.0)
    tw, th, off, ids = ctx.get_bins()
    assert int(np.diff(off).max()) > 100000
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    assert_parity(a.cpu().numpy(), ref, "unsplit huge tile lists")
    assert torch.equal(a, ctx.render(*args, W, H, sigma, R, 1.0))
    bands = [ctx.render_band(*args, W, H, g * 64, 64, sigma, R, 1.0) for g in range(H // 64)]
    assert torch.equal(torch.cat(bands, 0), a)


@pytest.mark.parametrize("R", [33, 63])
def test_wide_unsplit_huge_tile_lists(torch_dev, R):
    """Wide ROIs (parts and segments of WIDE_SPLIT = 256 stars) with more parts than the pool holds: the frame's tiles
    are walked whole in 256-star segments, the bands are split into parts -- bitwise the same; the warp-specialised
    and the synchronous kernels agree bitwise; parity against the oracle."""
    torch, dev = torch_dev
    from paper_conf_ipps_lizzh12_b200 import Context
    W, H, sigma = 256, 256, R / 6.0
    f = _dense_field(400000, W, H, 130.0, 130.0, 60.0, seed=6)
    args = to_dev(torch_dev, f)
    ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, threads=_threads())
    out = {}
    for mode in ("ws", "sb"):
        with Context(0) as c:
            c.set_tile_kernel(mode)
            a = c.render(*args, W, H, sigma, R, 1.0)
            if mode == "ws":
                tw, th, off, ids = c.get_bins()
                assert int(np.sum(np.ceil(np.diff(off) / 256.0))) > 2048  # the pool overflows: nothing split
            assert_parity(a.cpu().numpy(), ref, f"wide unsplit R={R} {mode}")
            bands = [c.render_band(*args, W, H, g * 64, 64, sigma, R, 1.0) for g in range(H // 64)]
            assert torch.equal(torch.cat(bands, 0), a)
            out[mode] = a
    assert torch.equal(out["ws"], out["sb"])


def test_circle_roi_with_integrated_psf(torch_dev, ctx):
    """NEXT-2 and NEXT-3 together on the star-centric kernels: the pixel-integrated PSF over the pixel-circle ROI."""
    W, H, n, R, sigma = 400, 300, 3000, 15, 2.5
    f = synth.uniform_field(n, W, H, seed=45, mag_hi=2.0)
    args = to_dev(torch_dev, f)
    ctx.set_roi("circle")
    ctx.set_psf("integrated")
    try:
        ref = oracle.render(f.x, f.y, f.mag, W, H, sigma, R, 1.0, psf="integrated", roi="circle")
        assert_parity(ctx.render_atomic(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref, "circle integrated atomic")
        ref_l = oracle.render_lut(f.x, f.y, f.mag, W, H, sigma, R, 1.0, psf="integrated", roi="circle")
        assert_parity(ctx.render_lut(*args, W, H, sigma, R, 1.0).cpu().numpy(), ref_l, "circle integrated lut")
    finally:
        ctx.set_roi("square")
        ctx.set_psf("point")
