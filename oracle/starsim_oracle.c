/*
 * oracle/starsim_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously correct fp64 CPU implementation of the star intensity model with Gaussian blur of
 * C. Li et al., "Implementing High-performance Intensity Model with Blur Effect on GPUs for Large-scale Star Image
 * Simulation" (IPDPS-W 2012), /root/reference/PAPER.md.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code, header, table or constant with the
 * CUDA path under paper_conf_ipps_lizzh12_b200/ and includes nothing from it.
 *
 * Every function follows the paper's definitions in the paper's order:
 *   Eq. 1 (Sec. II)   g(m) = A * 2.512^(-m)
 *   Eq. 2 (Sec. II)   mu(x,y) = 1/(2 pi d^2) * exp(-((x-X)^2 + (y-Y)^2) / (2 d^2))
 *   Eq. 3 (Sec. II)   phi(m,x,y) = g(m) * mu(x,y), pixel (x,y) restricted to the star's ROI
 *   Fig. 5 (Sec. III.A) sequential loop: for each star, for each ROI row, for each ROI column,
 *          if the pixel is inside the image, imagePixel[pixelY*img_width+pixelX] += gray.
 * Readings of points the paper leaves open are DESIGN.md "Readings" R1..R17:
 *   - the ROI is a square of side R (Fig. 1 caption PAPER.md:19, Fig. 5 loops PAPER.md:106);
 *   - its columns are the R integers nearest to the star's x (ties at k+1/2 round up), i.e.
 *     lo = floor(x + 1 - R/2) evaluated exactly; likewise rows from y;
 *   - pixel (px,py) is sampled at the integer coordinate (px,py) (point-sampled Eq. 2);
 *   - stars with a non-finite x, y or m, or whose clipped ROI is empty, contribute nothing;
 *   - accumulation is fp64 in star-index order (the paper's loop order).
 *
 * NEXT-2: a pixel-integrated variant of Eq. 2 -- the pixel value is the Gaussian of Eq. 2 integrated
 * over the pixel square [px-1/2, px+1/2] x [py-1/2, py+1/2] instead of sampled at its centre (psf mode 1), with the
 * same ROI, clipping and order.  Mode 0 is the paper's point-sampled Eq. 2.
 *
 * NEXT-3 (reading R21): the paper's literal "pixel circle" ROI -- mode bit 1.
 * The ROI is then the pixels of the square ROI above whose centres lie in the circle inscribed in that square: with
 * lo_x, lo_y its first column and row, pixel (px,py) belongs iff
 *   (2 (px - lo_x) - (R - 1))^2 + (2 (py - lo_y) - (R - 1))^2 <= R^2      (integers: an exact decision),
 * then clipped to the image as before.
 *
 * Pins (tests/test_oracle_pins.py, all "-m 'not gpu'"): Poisson-summation closed form of the point-sampled ROI mass,
 * first moment (centroid), reflection/transpose symmetry, scipy.ndimage.correlate with a kernel built from
 * scipy.stats.norm.pdf, brute-force no-ROI evaluation on tiny inputs, superposition, integer translation, magnitude
 * law, exact ROI origin against fractions.Fraction, brute-force binning, exact quantiser.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#ifndef M_PI
#define M_PI 3.14159265358979323846
#endif

/* Eq. 1: brightness of a star of magnitude m, A = "proportion factor". */
double oracle_brightness(double m, double A) { return A * pow(2.512, -m); }

/* Eq. 2: Gaussian PSF rate at pixel (px,py) of a star centred at (X,Y), deviation delta. */
double oracle_psf(double px, double py, double X, double Y, double delta) {
    double dx = px - X, dy = py - Y;
    return 1.0 / (2.0 * M_PI * delta * delta) * exp(-(dx * dx + dy * dy) / (2.0 * delta * delta));
}

/* NEXT-2: Eq. 2 integrated over the pixel square -- a product of two 1-D integrals of the normalised Gaussian,
 * (1/2) [erf((p + 1/2 - X) / (sqrt(2) d)) - erf((p - 1/2 - X) / (sqrt(2) d))], each taken in the form without
 * cancellation (erfc of the same-signed side). */
static double pixel_mass_1d(double p, double X, double delta) {
    double s = 1.0 / (sqrt(2.0) * delta);
    double a = (p - 0.5 - X) * s, b = (p + 0.5 - X) * s;
    if (a >= 0.0) return 0.5 * (erfc(a) - erfc(b));
    if (b <= 0.0) return 0.5 * (erfc(-b) - erfc(-a));
    return 0.5 * (erf(b) - erf(a));
}
double oracle_psf_integrated(double px, double py, double X, double Y, double delta) {
    return pixel_mass_1d(px, X, delta) * pixel_mass_1d(py, Y, delta);
}
static double psf_of(int mode, double px, double py, double X, double Y, double delta) {
    return (mode & 1) ? oracle_psf_integrated(px, py, X, Y, delta) : oracle_psf(px, py, X, Y, delta);
}

/* NEXT-3 (reading R21): is ROI pixel (i, j) = (row, column) offsets from the square's first row/column inside the
 * circle inscribed in the R x R square? */
static int in_circle(int64_t i, int64_t j, int32_t R) {
    int64_t u = 2 * j - (R - 1), v = 2 * i - (R - 1);
    return u * u + v * v <= (int64_t)R * R;
}
int oracle_in_circle(int64_t i, int64_t j, int32_t R) { return in_circle(i, j, R); }

/* First ROI column (or row) of a star at coordinate c: the R integers nearest to c, ties at k+1/2 upward, i.e.
 * lo = floor(c + 1 - R/2) in exact arithmetic (reading R7).  With f = floor(c) (exact):
 *   R even: 1 - R/2 is an integer, so lo = f + 1 - R/2;
 *   R odd:  lo = floor(c + 1/2) - (R-1)/2 and floor(c + 1/2) = f + [c >= f + 1/2].
 * Only exact operations are used (floor, integer shifts, and a comparison against f + 1/2, which is exact for the
 * |c| < 2^28 the caller guarantees): the rounded sum c + (1 - R/2) is NOT exact for tiny negative c. */
int64_t oracle_roi_lo(float c, int32_t R) {
    double f = floor((double)c);
    if (R % 2 == 0) return (int64_t)f + 1 - R / 2;
    return (int64_t)f + (((double)c >= f + 0.5) ? 1 : 0) - (R - 1) / 2;
}

/* A star is skipped when a coordinate or magnitude is not finite (reading R11) or its ROI cannot touch the image.
 * Returns 1 and the clipped ROI [*x0,*x1] x [*y0,*y1] if the star contributes. */
static int star_roi(float x, float y, float m, int32_t W, int32_t H, int32_t R,
                    int64_t* x0, int64_t* x1, int64_t* y0, int64_t* y1) {
    if (!isfinite(x) || !isfinite(y) || !isfinite(m)) return 0;
    /* far outside: no ROI pixel can be inside the image (and keeps oracle_roi_lo exact) */
    if ((double)x < -(double)R - 2.0 || (double)x > (double)W + R + 2.0) return 0;
    if ((double)y < -(double)R - 2.0 || (double)y > (double)H + R + 2.0) return 0;
    int64_t lx = oracle_roi_lo(x, R), ly = oracle_roi_lo(y, R);
    int64_t a = lx < 0 ? 0 : lx, b = lx + R - 1 > W - 1 ? W - 1 : lx + R - 1;
    int64_t c = ly < 0 ? 0 : ly, d = ly + R - 1 > H - 1 ? H - 1 : ly + R - 1;
    if (a > b || c > d) return 0;
    *x0 = a; *x1 = b; *y0 = c; *y1 = d;
    return 1;
}

/* Public helper for tests: clipped ROI of one star, or 0 if it is skipped. */
int oracle_star_roi(float x, float y, float m, int32_t W, int32_t H, int32_t R, int64_t* out4) {
    return star_roi(x, y, m, W, H, R, &out4[0], &out4[1], &out4[2], &out4[3]);
}

/* Fig. 5 over rows [row0, row0+rows) of the image only; img is rows*W doubles, zeroed here.
 * Brightness is hoisted out of the pixel loop (reading R15: the value is identical). */
static void render_rows(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                        int32_t row0, int32_t rows, double delta, int32_t R, double A, int32_t mode, double* img) {
    memset(img, 0, sizeof(double) * (size_t)rows * (size_t)W);
    for (int64_t i = 0; i < n; ++i) {
        int64_t x0, x1, y0, y1;
        if (!star_roi(x[i], y[i], mag[i], W, H, R, &x0, &x1, &y0, &y1)) continue;
        double g = oracle_brightness((double)mag[i], A);              /* Eq. 1 */
        double X = (double)x[i], Y = (double)y[i];
        int64_t lx = oracle_roi_lo(x[i], R), ly = oracle_roi_lo(y[i], R); /* the square's first column / row */
        if (y0 < row0) y0 = row0;
        if (y1 > row0 + rows - 1) y1 = row0 + rows - 1;
        for (int64_t py = y0; py <= y1; ++py)                            /* Fig. 5: pixelY over the ROI */
            for (int64_t px = x0; px <= x1; ++px) {                      /* Fig. 5: pixelX over the ROI */
                if ((mode & 2) && !in_circle(py - ly, px - lx, R)) continue; /* NEXT-3: the pixel circle */
                img[(size_t)(py - row0) * (size_t)W + (size_t)px] +=
                    g * psf_of(mode, (double)px, (double)py, X, Y, delta); /* Eq. 3 */
            }
    }
}

/* The oracle image (Eqs. 1-3, Fig. 5): img[py*W+px], fp64, H*W entries.  Returns U = sum of clipped ROI areas. */
int64_t oracle_render(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                      double delta, int32_t R, double A, int32_t mode, double* img) {
    render_rows(x, y, mag, n, W, H, 0, H, delta, R, A, mode, img);
    int64_t U = 0;
    for (int64_t i = 0; i < n; ++i) {
        int64_t x0, x1, y0, y1;
        if (!star_roi(x[i], y[i], mag[i], W, H, R, &x0, &x1, &y0, &y1)) continue;
        if (!(mode & 2)) { U += (x1 - x0 + 1) * (y1 - y0 + 1); continue; }
        int64_t lx = oracle_roi_lo(x[i], R), ly = oracle_roi_lo(y[i], R);
        for (int64_t py = y0; py <= y1; ++py)
            for (int64_t px = x0; px <= x1; ++px) U += in_circle(py - ly, px - lx, R);
    }
    return U;
}

/* Rows [row0, row0+rows) of the oracle image (used for band tests): img is rows*W. */
void oracle_render_band(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                        int32_t row0, int32_t rows, double delta, int32_t R, double A, int32_t mode, double* img) {
    render_rows(x, y, mag, n, W, H, row0, rows, delta, R, A, mode, img);
}

/* Same image, the rows split over nthreads pthreads (each thread owns whole rows and walks the stars in index order,
 * so every pixel sees the same additions in the same order: the result is bitwise equal to oracle_render).
 * Used only to time the CPU baseline on all host cores. */
struct band_job { const float *x, *y, *mag; int64_t n; int32_t W, H, row0, rows; double delta; int32_t R; double A;
                  int32_t mode; double* img; };
static void* band_main(void* p) {
    struct band_job* j = (struct band_job*)p;
    render_rows(j->x, j->y, j->mag, j->n, j->W, j->H, j->row0, j->rows, j->delta, j->R, j->A, j->mode,
                j->img + (size_t)j->row0 * (size_t)j->W);
    return NULL;
}
int oracle_render_mt(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                     double delta, int32_t R, double A, int32_t mode, double* img, int32_t nthreads) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > H) nthreads = H;
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)nthreads);
    struct band_job* jobs = (struct band_job*)malloc(sizeof(struct band_job) * (size_t)nthreads);
    if (!th || !jobs) { free(th); free(jobs); return -1; }
    for (int t = 0; t < nthreads; ++t) {
        int32_t r0 = (int32_t)((int64_t)H * t / nthreads), r1 = (int32_t)((int64_t)H * (t + 1) / nthreads);
        struct band_job j = {x, y, mag, n, W, H, r0, r1 - r0, delta, R, A, mode, img};
        jobs[t] = j;
        pthread_create(&th[t], NULL, band_main, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th); free(jobs);
    return 0;
}

/* No ROI cut-off (Fig. 1 left): every star against every pixel, pixel-centric (Fig. 3a).
 * For tiny inputs only.  Skips non-finite stars like the ROI version. */
void oracle_render_full(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H,
                        double delta, double A, int32_t mode, double* img) {
    for (int32_t py = 0; py < H; ++py)
        for (int32_t px = 0; px < W; ++px) {
            double v = 0.0;
            for (int64_t i = 0; i < n; ++i) {
                if (!isfinite(x[i]) || !isfinite(y[i]) || !isfinite(mag[i])) continue;
                v += oracle_brightness((double)mag[i], A) * psf_of(mode, px, py, (double)x[i], (double)y[i], delta);
            }
            img[(size_t)py * (size_t)W + (size_t)px] = v;
        }
}

/* Band routing (the definition starsim_route_band computes): the indices, in catalogue order,
 * of the stars whose ROI rows [ly, ly + R - 1] -- ly the first ROI row of reading R7 -- meet rows
 * [row0, row0 + rows).  Only y decides; a non-finite y is never routed (reading R11).  Returns the count. */
int64_t oracle_route_band(const float* y, int64_t n, int32_t R, int32_t row0, int32_t rows, int64_t* idx) {
    int64_t k = 0;
    for (int64_t i = 0; i < n; ++i) {
        if (!isfinite(y[i])) continue;
        /* far from the band: no ROI row can meet it (and keeps oracle_roi_lo exact) */
        if ((double)y[i] < (double)row0 - R - 2.0 || (double)y[i] > (double)row0 + rows + R + 2.0) continue;
        int64_t ly = oracle_roi_lo(y[i], R);
        if (ly <= (int64_t)row0 + rows - 1 && ly + R - 1 >= (int64_t)row0) idx[k++] = i;
    }
    return k;
}

/* Binning definition (get_bins): image tiles of tw x th pixels, ntx = ceil(W/tw) per row,
 * key = ty*ntx + tx.  For each contributing star in index order, one pair per tile its clipped ROI overlaps, tiles in
 * row-major order; then a stable sort by key, i.e. star-index order inside each tile.  Output: CSR
 * tile_off[ntiles+1] and ids[P].  Returns P, or -1 if ids_cap is too small (tile_off is still filled). */
int64_t oracle_bins(const float* x, const float* y, const float* mag, int64_t n, int32_t W, int32_t H, int32_t R,
                    int32_t tw, int32_t th, uint32_t* tile_off, uint32_t* ids, int64_t ids_cap) {
    int64_t ntx = (W + tw - 1) / tw, nty = (H + th - 1) / th, nt = ntx * nty;
    int64_t* cnt = (int64_t*)calloc((size_t)nt + 1, sizeof(int64_t));
    if (!cnt) return -2;
    for (int64_t i = 0; i < n; ++i) {                      /* count pairs per tile */
        int64_t x0, x1, y0, y1;
        if (!star_roi(x[i], y[i], mag[i], W, H, R, &x0, &x1, &y0, &y1)) continue;
        for (int64_t ty = y0 / th; ty <= y1 / th; ++ty)
            for (int64_t tx = x0 / tw; tx <= x1 / tw; ++tx) cnt[ty * ntx + tx] += 1;
    }
    int64_t P = 0;
    for (int64_t t = 0; t < nt; ++t) { tile_off[t] = (uint32_t)P; P += cnt[t]; cnt[t] = 0; }
    tile_off[nt] = (uint32_t)P;
    if (P > ids_cap) { free(cnt); return -1; }
    for (int64_t i = 0; i < n; ++i) {                      /* fill in star order: stable */
        int64_t x0, x1, y0, y1;
        if (!star_roi(x[i], y[i], mag[i], W, H, R, &x0, &x1, &y0, &y1)) continue;
        for (int64_t ty = y0 / th; ty <= y1 / th; ++ty)
            for (int64_t tx = x0 / tw; tx <= x1 / tw; ++tx) {
                int64_t k = ty * ntx + tx;
                ids[tile_off[k] + cnt[k]] = (uint32_t)i;
                cnt[k] += 1;
            }
    }
    free(cnt);
    return P;
}

/* Output stage: gray value q = min(2^bits - 1, floor(v + 1/2)), v <= 0 or NaN -> 0 (reading R13).
 * floor(v + 1/2) is evaluated exactly as f + (v - f >= 1/2) with f = floor(v): v - f is exact for v >= 0, whereas
 * the rounded sum v + 0.5 can carry across an integer (e.g. v = 0.5 - 2^-54). */
void oracle_quantize(const double* v, int64_t npix, int32_t bits, void* out) {
    double qmax = bits == 8 ? 255.0 : 65535.0;
    for (int64_t i = 0; i < npix; ++i) {
        double q = 0.0;
        if (v[i] > 0.0) { double f = floor(v[i]); q = f + ((v[i] - f >= 0.5) ? 1.0 : 0.0); }  /* NaN -> 0 */
        if (q > qmax) q = qmax;
        if (bits == 8) ((uint8_t*)out)[i] = (uint8_t)q;
        else ((uint16_t*)out)[i] = (uint16_t)q;
    }
}
