"""Pins of the fp64 oracle (oracle/) to things other than itself -- SURVEY.md §8(c) "What pins each part".

The paper prints no numeric worked example (its figures were lost; Tables I-III hold timings only), so every pin is a
closed form, an invariant, a library routine on a special case, or brute force on tiny inputs.  Each is chosen so
that a plausible slip in the oracle (a dropped 1/(2 pi d^2), 2d^2 vs d^2, a sign, x/y transposed, a pixel-centre
offset of 1/2, an off-by-one ROI bound, unstable binning, v+0.5 rounding) fails at least one of them.
"""
import math
from fractions import Fraction

import numpy as np
import pytest
from scipy import ndimage
from scipy.stats import norm

import oracle
import synth


def theta_mass(u, sigma, nmax=30):
    """Poisson summation: (1/(sqrt(2 pi) sigma)) sum_k exp(-(k-u)^2/(2 sigma^2)) = sum_n exp(-2 pi^2 sigma^2 n^2)
    cos(2 pi n u).  The right side is the Fourier-side closed form of the point-sampled 1-D Gaussian mass."""
    return 1.0 + 2.0 * sum(math.exp(-2.0 * math.pi ** 2 * sigma ** 2 * n * n) * math.cos(2 * math.pi * n * u)
                           for n in range(1, nmax))


def star(x, y, m=0.0):
    return (np.array([x], np.float32), np.array([y], np.float32), np.array([m], np.float32))


# ---------------------------------------------------------------- Eq. 2 normalisation and exponent: ROI mass

@pytest.mark.parametrize("sigma", [0.5, 1.0, 1.5, 2.5])
@pytest.mark.parametrize("u,v", [(0.0, 0.0), (0.3, -0.45), (-0.25, 0.125)])
def test_wide_roi_mass_matches_poisson_closed_form(sigma, u, v):
    # one m=0 star (g = A = 1) near the centre of a 101x101 image with a 41-px ROI (truncation < 1e-14)
    x, y, m = star(50 + u, 50 + v)
    img = oracle.render(x, y, m, 101, 101, sigma, 41, 1.0)
    expect = theta_mass(float(x[0]) - 50, sigma) * theta_mass(float(y[0]) - 50, sigma)
    assert abs(img.sum() - expect) < 1e-13


@pytest.mark.parametrize("R,sigma,expect", [
    # centred-star ROI masses of the point-sampled model: C1, C2, T/C5, C4 at R=63
    (5, 1.0, 0.98181476105437437), (9, 1.5, 0.99551483498249382), (15, 2.5, 0.99495146217965957),
    (63, 10.5, 0.99462770988573979)])
def test_centred_roi_mass_matches_separable_closed_form(R, sigma, expect):
    h = (R - 1) // 2
    one_d = sum(norm.pdf(k, scale=sigma) for k in range(-h, h + 1))   # library 1-D pdf, not the oracle's formula
    assert abs(one_d * one_d - expect) < 1e-14                         # the tabulated value is that closed form
    c = R  # centre pixel, image 2R+1 wide
    x, y, m = star(c, c)
    img = oracle.render(x, y, m, 2 * R + 1, 2 * R + 1, sigma, R, 1.0)
    assert abs(img.sum() - expect) < 1e-13


def test_centred_mass_is_not_erf_squared():
    # the model is point-sampled (reading R9): the erf^2 mass of a pixel-integrated PSF differs by ~0.0065 at C1
    x, y, m = star(5, 5)
    img = oracle.render(x, y, m, 11, 11, 1.0, 5, 1.0)
    erf2 = math.erf(2.5 / math.sqrt(2)) ** 2
    assert abs(img.sum() - erf2) > 5e-3


# ---------------------------------------------------------------- first moment: x/y orientation and pixel centre

@pytest.mark.parametrize("sigma", [1.5, 2.5])
def test_centroid_is_star_position(sigma):
    x, y, m = star(40.3125, 23.71875)          # x != y, on a 1/256 grid
    img = oracle.render(x, y, m, 80, 48, sigma, 41, 1.0)
    py, px = np.mgrid[0:48, 0:80]
    s = img.sum()
    assert abs((img * px).sum() / s - 40.3125) < 1e-9
    assert abs((img * py).sum() / s - 23.71875) < 1e-9
    # row-major with y = row: the peak sits at row round(y), column round(x)
    r, c = np.unravel_index(np.argmax(img), img.shape)
    assert (r, c) == (24, 40)


# ---------------------------------------------------------------- symmetry (Eq. 2 "spatially symmetrical")

@pytest.mark.parametrize("R", [5, 9, 15])
def test_pixel_centred_star_is_symmetric_bitwise(R):
    x, y, m = star(25, 25)
    img = oracle.render(x, y, m, 51, 51, R / 6, R, 3.0)
    assert np.array_equal(img, img[::-1, :])
    assert np.array_equal(img, img[:, ::-1])
    assert np.array_equal(img, img.T)


def test_mirror_pair_gives_mirrored_image():
    a = oracle.render(*star(25 + 0.25, 25 - 0.375), 51, 51, 1.3, 9, 1.0)
    b = oracle.render(*star(25 - 0.25, 25 + 0.375), 51, 51, 1.3, 9, 1.0)
    assert np.array_equal(a, b[::-1, ::-1])


# ---------------------------------------------------------------- library routine: scipy correlate with norm.pdf kernel

@pytest.mark.parametrize("R,sigma", [(1, 0.7), (3, 0.5), (5, 1.0), (9, 1.5), (15, 2.5)])
def test_integer_stars_equal_scipy_correlate(R, sigma):
    W, H = 64, 48
    rng = np.random.default_rng(R)
    n = 40
    xs = rng.integers(-R, W + R, n).astype(np.float32)   # includes stars partly and wholly off the image
    ys = rng.integers(-R, H + R, n).astype(np.float32)
    ms = rng.uniform(0, 3, n).astype(np.float32)
    A = 2.0
    img = oracle.render(xs, ys, ms, W, H, sigma, R, A)
    # impulses on a padded canvas so off-image stars still spread into the image; kernel from the library pdf
    pad = R
    canvas = np.zeros((H + 2 * pad, W + 2 * pad))
    for xi, yi, mi in zip(xs, ys, ms):
        canvas[int(yi) + pad, int(xi) + pad] += A * 2.512 ** (-float(mi))
    h = (R - 1) // 2
    k1 = norm.pdf(np.arange(-h, h + 1), scale=sigma)
    K = np.outer(k1, k1)
    ref = ndimage.correlate(canvas, K, mode="constant", cval=0.0)[pad:pad + H, pad:pad + W]
    assert np.max(np.abs(img - ref)) <= 1e-13 * max(1.0, np.max(np.abs(ref)))


# ---------------------------------------------------------------- brute force: no ROI cut-off on tiny inputs

@pytest.mark.parametrize("seed", [1, 2, 3])
def test_huge_roi_equals_full_evaluation_bitwise(seed):
    rng = np.random.default_rng(seed)
    W, H = int(rng.integers(5, 40)), int(rng.integers(5, 40))
    n = int(rng.integers(1, 30))
    xs = rng.uniform(-5, W + 5, n).astype(np.float32)
    ys = rng.uniform(-5, H + 5, n).astype(np.float32)
    ms = rng.uniform(0, 15, n).astype(np.float32)
    R = 2 * max(W, H) + 11
    a = oracle.render(xs, ys, ms, W, H, 1.7, R, 1.0)
    b = oracle.render_full(xs, ys, ms, W, H, 1.7, 1.0)
    assert np.array_equal(a, b)


def test_finite_roi_loses_exactly_the_outside_mass():
    # isolated interior star: full - ROI = g * (Mx_img*My_img - Mx_R*My_R), 1-D sums from the library pdf
    W, H, R, sigma = 41, 37, 7, 1.6
    x, y, m = star(20.375, 17.8125, 1.0)
    full = oracle.render_full(x, y, m, W, H, sigma, 1.0)
    roi = oracle.render(x, y, m, W, H, sigma, R, 1.0)
    g = 2.512 ** -1.0
    lo_x, lo_y = 20 - 3, 18 - 3
    Mx_img = norm.pdf(np.arange(W) - 20.375, scale=sigma).sum()
    My_img = norm.pdf(np.arange(H) - 17.8125, scale=sigma).sum()
    Mx_R = norm.pdf(np.arange(lo_x, lo_x + R) - 20.375, scale=sigma).sum()
    My_R = norm.pdf(np.arange(lo_y, lo_y + R) - 17.8125, scale=sigma).sum()
    assert abs((full.sum() - roi.sum()) - g * (Mx_img * My_img - Mx_R * My_R)) < 1e-14


def test_corner_star_is_clipped_not_renormalised():
    W, H, R, sigma = 30, 20, 7, 1.2
    x, y, m = star(0.2, -0.3, 0.5)
    img = oracle.render(x, y, m, W, H, sigma, R, 1.0)
    cols = np.arange(0, 0 + 4)        # ROI columns -3..3, in image 0..3
    rows = np.arange(0, -3 + 7)       # ROI rows -3..3 (round(-0.3) = 0), in image 0..3
    X, Y = float(x[0]), float(y[0])   # the fp32 coordinates, widened exactly
    expect = 2.512 ** -0.5 * norm.pdf(cols - X, scale=sigma).sum() * norm.pdf(rows - Y, scale=sigma).sum()
    assert abs(img.sum() - expect) < 1e-14
    assert np.count_nonzero(img) == 16


# ---------------------------------------------------------------- superposition, scaling, translation (Eq. 3)

def test_superposition_and_gain_scaling():
    f = synth.uniform_field(300, 96, 80, seed=11)
    a = oracle.render(f.x, f.y, f.mag, 96, 80, 1.4, 9, 1.0)
    b1 = oracle.render(f.x[:150], f.y[:150], f.mag[:150], 96, 80, 1.4, 9, 1.0)
    b2 = oracle.render(f.x[150:], f.y[150:], f.mag[150:], 96, 80, 1.4, 9, 1.0)
    assert np.max(np.abs(a - (b1 + b2))) <= 4e-16 * np.max(a)
    a2 = oracle.render(f.x, f.y, f.mag, 96, 80, 1.4, 9, 2.0)
    assert np.array_equal(a2, 2.0 * a)


def test_integer_translation_is_exact():
    rng = np.random.default_rng(5)
    n = 60
    xs = (rng.integers(20 * 256, 60 * 256, n) / 256.0).astype(np.float32)
    ys = (rng.integers(20 * 256, 40 * 256, n) / 256.0).astype(np.float32)
    ms = rng.uniform(0, 5, n).astype(np.float32)
    a = oracle.render(xs, ys, ms, 100, 70, 1.5, 9, 1.0)
    b = oracle.render(xs + np.float32(7), ys + np.float32(3), ms, 100, 70, 1.5, 9, 1.0)
    assert np.array_equal(a[:-3, :-7], b[3:, 7:])


# ---------------------------------------------------------------- Eq. 1 magnitude law

def test_magnitude_law():
    assert oracle.brightness(0.0, 3.25) == 3.25
    base = oracle.render(*star(12.3, 8.6, 4.0), 25, 18, 1.1, 7, 1.0)
    fainter = oracle.render(*star(12.3, 8.6, 5.0), 25, 18, 1.1, 7, 1.0)
    nz = base != 0
    assert np.max(np.abs(base[nz] / fainter[nz] - 2.512)) < 1e-13
    # Pogson's 5 magnitudes ~ factor 100 (2.512^5 = 100.02...), the textbook reading of Eq. 1
    assert abs(oracle.brightness(0, 1) / oracle.brightness(5, 1) - 100.0) < 0.03


# ---------------------------------------------------------------- exact ROI origin (reading R7)

def _adversarial_coords():
    vals = [0.0, -0.0, 0.49999997, 0.5, 0.50000006, 1.5, 2.5, -0.5, -0.49999997, -1.5, 1e-30, -1e-30,
            4095.5, 4095.4999, 16383.5, 3.0, -3.0, 7.25]
    out = []
    for v in vals:
        f = np.float32(v)
        out += [f, np.nextafter(f, np.float32(np.inf)), np.nextafter(f, np.float32(-np.inf))]
    rng = np.random.default_rng(9)
    out += list(rng.uniform(-300, 5000, 2000).astype(np.float32))
    k = rng.integers(-200, 5000, 500).astype(np.float32)
    out += list(k + np.float32(0.5)) + list(np.nextafter(k + np.float32(0.5), np.float32(0)))
    return out


@pytest.mark.parametrize("R", [1, 2, 3, 4, 5, 15, 16, 63])
def test_roi_lo_is_exact_and_nearest(R):
    for c in _adversarial_coords():
        lo = oracle.roi_lo(float(c), R)
        exact = math.floor(Fraction(float(c)) + 1 - Fraction(R, 2))
        assert lo == exact, (c, R)
        # the R integers lo..lo+R-1 are the R nearest to c (ties at k+1/2 resolved upward)
        fc = Fraction(float(c))
        inside = [abs(Fraction(k) - fc) for k in range(lo, lo + R)]
        outside = [abs(Fraction(lo - 1) - fc), abs(Fraction(lo + R) - fc)]
        assert max(inside) <= min(outside)


# ---------------------------------------------------------------- binning CSR, brute force

@pytest.mark.parametrize("R", [1, 3, 5, 8, 15])
@pytest.mark.parametrize("tw,th", [(8, 8), (16, 4), (32, 32)])
def test_bins_equal_brute_force(R, tw, th):
    W, H = 50, 37
    f = synth.adversarial_field(120, W, H, R, seed=R * 100 + tw)
    off, ids = oracle.bins(f.x, f.y, f.mag, W, H, R, tw, th)
    ntx, nty = -(-W // tw), -(-H // th)
    exp_off, exp_ids = [0], []
    for ty in range(nty):
        for tx in range(ntx):
            tile = {(px, py) for py in range(ty * th, min(H, (ty + 1) * th)) for px in range(tx * tw, min(W, (tx + 1) * tw))}
            for i in range(f.n):
                xi, yi, mi = float(f.x[i]), float(f.y[i]), float(f.mag[i])
                if not (math.isfinite(xi) and math.isfinite(yi) and math.isfinite(mi)):
                    continue
                if abs(xi) > 1e5 or abs(yi) > 1e5:
                    continue
                lx = math.floor(Fraction(xi) + 1 - Fraction(R, 2))
                ly = math.floor(Fraction(yi) + 1 - Fraction(R, 2))
                if any((px, py) in tile for py in range(ly, ly + R) for px in range(lx, lx + R)):
                    exp_ids.append(i)
            exp_off.append(len(exp_ids))
    assert off.tolist() == exp_off
    assert ids.tolist() == exp_ids


# ---------------------------------------------------------------- quantiser (reading R13)

@pytest.mark.parametrize("bits", [8, 16])
def test_quantize_exact(bits):
    qmax = 2 ** bits - 1
    vals = [0.0, -0.0, -1.0, 0.49999997, 0.5, 0.50000006, 1.4999999, 1.5, 2.5, 254.5, 254.49998, 255.0, 255.5,
            65534.5, 65535.4, 65535.5, 1e9, float("inf"), float("-inf"), float("nan"), 0.5 - 2 ** -54]
    rng = np.random.default_rng(bits)
    vals += list(rng.uniform(-2, qmax + 3, 3000))
    v = np.array(vals, dtype=np.float64)
    q = oracle.quantize(v, bits)
    for vi, qi in zip(vals, q.tolist()):
        if math.isnan(vi) or vi <= 0:
            e = 0
        elif math.isinf(vi):
            e = qmax
        else:
            e = min(qmax, math.floor(Fraction(vi) + Fraction(1, 2)))
        assert qi == e, (vi, qi, e)


# ---------------------------------------------------------------- bookkeeping: units, bands, threads, bad stars

def test_units_count_roi_pixels_brute_force():
    W, H, R = 40, 30, 5
    f = synth.adversarial_field(80, W, H, R, seed=3)
    U, E, live = oracle.units(f.x, f.y, f.mag, W, H, R)
    cover = np.zeros((H, W), np.int64)
    ee = 0
    for i in range(f.n):
        roi = oracle.star_roi(float(f.x[i]), float(f.y[i]), float(f.mag[i]), W, H, R)
        if roi:
            x0, x1, y0, y1 = roi
            cover[y0:y1 + 1, x0:x1 + 1] += 1
            ee += (x1 - x0 + 1) + (y1 - y0 + 1)
    assert U == cover.sum() and E == ee


def test_band_and_threads_are_bitwise_slices():
    f = synth.uniform_field(500, 120, 90, seed=4)
    full = oracle.render(f.x, f.y, f.mag, 120, 90, 1.2, 7, 1.0)
    band = oracle.render_band(f.x, f.y, f.mag, 120, 90, 32, 40, 1.2, 7, 1.0)
    assert np.array_equal(band, full[32:72])
    mt = oracle.render(f.x, f.y, f.mag, 120, 90, 1.2, 7, 1.0, threads=5)
    assert np.array_equal(mt, full)


def test_nonfinite_stars_contribute_nothing():
    f = synth.uniform_field(50, 64, 64, seed=8)
    x, y, m = f.x.copy(), f.y.copy(), f.mag.copy()
    x[3], y[10], m[20] = np.nan, np.inf, -np.inf
    keep = np.ones(50, bool)
    keep[[3, 10, 20]] = False
    a = oracle.render(x, y, m, 64, 64, 1.0, 5, 1.0)
    b = oracle.render(x[keep], y[keep], m[keep], 64, 64, 1.0, 5, 1.0)
    assert np.array_equal(a, b)


def test_even_roi_side_uses_nearest_pixels():
    # R even (the paper's 10x10 test1 ROI): columns floor(x)-R/2+1 .. floor(x)+R/2
    x, y, m = star(10.7, 10.2)
    img = oracle.render(x, y, m, 21, 21, 2.0, 4, 1.0)
    cols = np.nonzero(img.any(axis=0))[0].tolist()
    rows = np.nonzero(img.any(axis=1))[0].tolist()
    assert cols == [9, 10, 11, 12] and rows == [9, 10, 11, 12]


# ---------------------------------------------------------------- NEXT-2: pixel-integrated PSF (psf="integrated")

def _erf_mass_1d(lo, hi, u, sigma):
    """Telescoped closed form of the 1-D pixel masses over pixels lo..hi: (1/2)[erf((hi+1/2-u)/(sqrt2 s)) -
    erf((lo-1/2-u)/(sqrt2 s))] (the per-pixel differences cancel pairwise)."""
    s = math.sqrt(2.0) * sigma
    return 0.5 * (math.erf((hi + 0.5 - u) / s) - math.erf((lo - 0.5 - u) / s))


@pytest.mark.parametrize("sigma", [0.5, 1.0, 2.5])
@pytest.mark.parametrize("u,v", [(0.0, 0.0), (0.3, -0.45), (-0.49, 0.2)])
@pytest.mark.parametrize("R", [5, 15])
def test_integrated_roi_mass_telescopes(sigma, u, v, R):
    x, y, m = star(40 + u, 40 + v)
    img = oracle.render(x, y, m, 81, 81, sigma, R, 1.0, psf="integrated")
    lx, ly = oracle.roi_lo(float(x[0]), R), oracle.roi_lo(float(y[0]), R)
    expect = (_erf_mass_1d(lx, lx + R - 1, float(x[0]), sigma) * _erf_mass_1d(ly, ly + R - 1, float(y[0]), sigma))
    assert abs(img.sum() - expect) < 1e-13
    # exactly the ROI pixels are lit
    assert np.count_nonzero(img) == R * R


@pytest.mark.parametrize("sigma,X,Y,px,py", [(0.7, 10.3, 9.8, 10, 10), (0.7, 10.3, 9.8, 11, 9),
                                             (1.5, 4.0, 4.0, 6, 3), (0.4, 2.5, 2.5, 2, 3)])
def test_integrated_pixel_equals_numerical_quadrature(sigma, X, Y, px, py):
    from scipy import integrate
    f = lambda yy, xx: math.exp(-((xx - X) ** 2 + (yy - Y) ** 2) / (2 * sigma * sigma)) / (2 * math.pi * sigma ** 2)
    q, err = integrate.dblquad(f, px - 0.5, px + 0.5, py - 0.5, py + 0.5, epsabs=1e-14, epsrel=1e-12)
    assert abs(oracle.psf(px, py, X, Y, sigma, "integrated") - q) < 1e-12


def test_integrated_tends_to_point_sampled_for_wide_psf():
    # for sigma >> 1 px the pixel integral of the Gaussian is its centre value times (1 + f''/(24 f) per axis):
    # (a - b) / b = [(dx^2/s^2 - 1) + (dy^2/s^2 - 1)] / (24 s^2) + O(s^-4)   (midpoint rule error, exact 2nd order)
    s = 20.0
    for px, py in [(0, 0), (3, -2), (10, 7)]:
        dx, dy = px - 0.2, py + 0.1
        a = oracle.psf(px, py, 0.2, -0.1, s, "integrated")
        b = oracle.psf(px, py, 0.2, -0.1, s, "point")
        pred = ((dx * dx / (s * s) - 1.0) + (dy * dy / (s * s) - 1.0)) / (24.0 * s * s)
        assert abs((a - b) / b - pred) < 2e-7


def test_integrated_symmetric_and_full_evaluation_bitwise():
    x, y, m = star(12, 12)
    img = oracle.render(x, y, m, 25, 25, 1.3, 9, 1.0, psf="integrated")
    assert np.array_equal(img, img[::-1, ::-1]) and np.array_equal(img, img.T)
    f = synth.uniform_field(30, 24, 20, seed=5, mag_lo=0.0, mag_hi=3.0)
    a = oracle.render(f.x, f.y, f.mag, 24, 20, 1.1, 2 * 24 + 1, 1.0, psf="integrated")
    b = oracle.render_full(f.x, f.y, f.mag, 24, 20, 1.1, 1.0, psf="integrated")
    assert np.array_equal(a, b)


# ---------------------------------------------------------------- NEXT-4: the adaptive simulator's table (reading R20)

@pytest.mark.parametrize("R", [1, 2, 5, 10, 15, 16])
def test_lut_positions_are_the_roi_centres(R):
    """lut_positions snaps every coordinate to the centre of its ROI: lo + (R-1)/2 with lo the oracle's exact roi_lo
    (pinned above against Fraction), checked on the adversarial coordinates."""
    cs = np.array(_adversarial_coords()[:4000], dtype=np.float32)
    sx, _ = oracle.lut_positions(cs, cs, R)
    for c, s in zip(cs, sx):
        assert float(s) == oracle.roi_lo(float(c), R) + 0.5 * (R - 1)
        # the snapped star has the same ROI (the table is laid over the star's own R nearest pixels)
        assert oracle.roi_lo(float(s), R) == oracle.roi_lo(float(c), R)


def test_lut_equals_render_for_pixel_centred_stars():
    """For stars on pixel centres and odd R the table is exact: render_lut == render bitwise; sub-pixel stars move."""
    rng_ = np.random.default_rng(40)
    W, H, R = 120, 90, 9
    x = rng_.integers(-5, W + 5, 300).astype(np.float32)
    y = rng_.integers(-5, H + 5, 300).astype(np.float32)
    m = rng_.uniform(0, 5, 300).astype(np.float32)
    a = oracle.render_lut(x, y, m, W, H, 1.5, R, 1.0)
    b = oracle.render(x, y, m, W, H, 1.5, R, 1.0)
    assert np.array_equal(a, b)
    c = oracle.render_lut(x + np.float32(0.3), y - np.float32(0.2), m, W, H, 1.5, R, 1.0)
    assert np.array_equal(c, b)                      # |offset| < 1/2: same centres
    d = oracle.render(x + np.float32(0.3), y - np.float32(0.2), m, W, H, 1.5, R, 1.0)
    assert not np.array_equal(d, b)


def test_lut_star_mass_is_the_centred_closed_form():
    """A sub-pixel star rendered by the table carries the centred ROI mass g * M1(0)^2 (C1: 0.98181476105437437),
    not its own sub-pixel mass, and its image is symmetric about the ROI centre."""
    x, y, m = star(10.3, 9.8)
    img = oracle.render_lut(x, y, m, 21, 21, 1.0, 5, 1.0)
    assert abs(img.sum() - 0.98181476105437437) < 1e-13
    assert np.array_equal(img, img[::-1, ::-1]) and np.array_equal(img, img.T)
    assert img[10, 10] == img.max()


# ---------------------------------------------------------------- NEXT-3: the "pixel circle" ROI (reading R21)

# Gauss's circle problem: N(n) = #{(u, v) in Z^2 : u^2 + v^2 <= n} (OEIS A057655: N(6) = 21, N(12) = 37, N(20) = 69,
# N(56) = 177).  For odd R the circle inscribed in the R x R ROI is centred on a pixel with radius R/2, so it holds
# N(floor(R^2/4)) pixels; for R = 4 the centre is a pixel corner and the pixels are the 12 half-integer points
# (+-1/2, +-1/2), (+-1/2, +-3/2), (+-3/2, +-1/2) within radius 2.
@pytest.mark.parametrize("R,count", [(5, 21), (7, 37), (9, 69), (15, 177), (4, 12)])
def test_circle_roi_holds_the_gauss_circle_count(R, count):
    x, y, m = star(40.0, 40.0)
    img, U = oracle.render(x, y, m, 81, 81, 1e4, R, 1.0, return_units=True, roi="circle")  # flat PSF: all > 0
    assert int(np.count_nonzero(img)) == count and U == count
    sq = oracle.render(x, y, m, 81, 81, 1e4, R, 1.0, roi="square")
    assert int(np.count_nonzero(sq)) == R * R


@pytest.mark.parametrize("R", [5, 8, 15])
def test_circle_roi_is_the_square_minus_its_corners(R):
    """Inside the circle the value is the square ROI's bitwise; the square's four corner pixels are always outside,
    the four edge midpoints (odd R) inside; and a pixel-centred star's circle image is dihedrally symmetric."""
    x, y, m = star(30.0, 30.0, 0.5)
    sq = oracle.render(x, y, m, 61, 61, 2.0, R, 1.0)
    ci = oracle.render(x, y, m, 61, 61, 2.0, R, 1.0, roi="circle")
    inside = ci != 0
    assert np.array_equal(ci[inside], sq[inside]) and np.all(sq[~inside & (sq != 0)] > 0)
    lo = oracle.roi_lo(30.0, R)
    for (py, px) in [(lo, lo), (lo, lo + R - 1), (lo + R - 1, lo), (lo + R - 1, lo + R - 1)]:
        assert ci[py, px] == 0 and sq[py, px] > 0
    if R % 2:
        c = lo + (R - 1) // 2
        for (py, px) in [(lo, c), (c, lo), (lo + R - 1, c), (c, lo + R - 1)]:
            assert ci[py, px] > 0
        for t in (ci.T, ci[::-1, :], ci[:, ::-1], ci[::-1, ::-1].T):
            assert np.array_equal(t, ci)


def test_circle_roi_superposition_and_clipping():
    """The circle only masks: linear in the catalogue, and a circle cut by the image border keeps exactly the in-image
    pixels of the full circle rendered in a larger frame (shifted by a whole number of pixels)."""
    f = synth.uniform_field(40, 64, 48, seed=3, mag_hi=3.0)
    a = oracle.render(f.x[:20], f.y[:20], f.mag[:20], 64, 48, 1.3, 9, 1.0, roi="circle")
    b = oracle.render(f.x[20:], f.y[20:], f.mag[20:], 64, 48, 1.3, 9, 1.0, roi="circle")
    ab = oracle.render(f.x, f.y, f.mag, 64, 48, 1.3, 9, 1.0, roi="circle")
    assert np.allclose(a + b, ab, rtol=1e-14, atol=0)
    x, y, m = star(1.0, 2.0)
    small = oracle.render(x, y, m, 20, 20, 1.5, 11, 1.0, roi="circle")
    big = oracle.render(x + 10, y + 10, m, 40, 40, 1.5, 11, 1.0, roi="circle")
    assert np.array_equal(small, big[10:30, 10:30])


def test_circle_roi_integrated_psf_keeps_the_circle_and_the_masses():
    """psf="integrated" with roi="circle": the circle's pixels carry exactly the integrated square-ROI values (the
    mask only removes pixels), and a pixel-centred star's image stays dihedrally symmetric."""
    x, y, m = star(20.0, 20.0)
    sq = oracle.render(x, y, m, 41, 41, 1.8, 11, 1.0, psf="integrated")
    ci = oracle.render(x, y, m, 41, 41, 1.8, 11, 1.0, psf="integrated", roi="circle")
    inside = ci != 0
    assert int(inside.sum()) == 97  # Gauss circle N(30) = 97 (OEIS A057655) for R = 11: r^2 = 30.25
    assert np.array_equal(ci[inside], sq[inside])
    for t in (ci.T, ci[::-1, :], ci[:, ::-1]):
        assert np.array_equal(t, ci)
