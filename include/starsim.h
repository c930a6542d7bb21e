/*
 * include/starsim.h -- C ABI of libstarsim.so, the B200-native (sm_100a) star-image renderer.
 *
 * What it computes (C. Li et al., IPDPS-W 2012, Sec. II):
 *   Eq. 1  g(m) = A * 2.512^(-m)                       -- brightness from magnitude, A = `gain`
 *   Eq. 2  mu(x,y) = 1/(2 pi s^2) exp(-((x-X)^2+(y-Y)^2)/(2 s^2))   -- Gaussian PSF, s = `sigma`
 *   Eq. 3  phi(m,x,y) = g(m) * mu(x,y) for pixels (x,y) inside the star's ROI, summed over stars
 *   ROI: a square of side R = `roi` (Fig. 1, Fig. 5 loops PAPER.md:94-112): the R columns nearest to the
 *   star's x (ties at k+1/2 round up) times the R rows nearest to its y; pixels outside the image are dropped
 *   (PAPER.md:106, 134), nothing is renormalised.  Pixel (px,py) is sampled at integer (px,py); the image is
 *   row-major with y = row: out[py*width + px].  DESIGN.md "Readings" lists every such choice.
 *
 * Conventions for every entry point:
 *   - Array pointers marked (device) are CUDA device pointers on the ctx's device; (host) are host pointers.
 *   - The caller owns every input and output buffer.  The ctx owns its scratch (star records, tile lists, sort
 *     scratch, offsets); scratch grows geometrically, is reused across calls and is freed by starsim_destroy.
 *   - Calls are stream-ordered and asynchronous on `stream` (0 = legacy default stream); host-side validation is
 *     synchronous and happens before anything is enqueued.
 *   - A ctx is bound to one device and is not thread-safe: use one ctx per host thread / stream.
 *   - Return codes: STARSIM_OK, or a negative code.  On STARSIM_EINVAL nothing is enqueued and `out` is untouched.
 *     starsim_last_error() describes the most recent failure.
 *   - Per-star bad data is not an error: stars with a non-finite x, y or mag, or whose ROI misses the image (or the
 *     band), contribute nothing -- exactly as the oracle does.
 */
#ifndef STARSIM_H
#define STARSIM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct starsim_ctx starsim_ctx;
typedef struct CUstream_st* starsim_stream_t; /* == cudaStream_t */

enum {
  STARSIM_OK = 0,
  STARSIM_EINVAL = -1, /* an argument is out of range (list at each call)            */
  STARSIM_ENOMEM = -2, /* scratch growth failed (cudaMalloc)                          */
  STARSIM_ECUDA = -3,  /* a CUDA runtime error; text in starsim_last_error            */
  STARSIM_ENODEV = -4  /* the device is not an sm_100 (B200-class) GPU                */
};

/* Limits checked by every render call (EINVAL otherwise). */
#define STARSIM_MAX_DIM 32767      /* width, height in [1, 32767], width*height < 2^31 */
#define STARSIM_MAX_ROI 255        /* roi (R, the ROI side) in [1, 255]                 */

/* Create a context on CUDA device `cuda_device`.  Fails with ENODEV unless its compute capability is 10.x
 * (this library carries sm_100a code only).  *out is set to NULL on failure. */
int starsim_create(starsim_ctx** out, int cuda_device);

/* Destroy a context and free its scratch.  NULL-safe.  Synchronises the ctx's device first. */
void starsim_destroy(starsim_ctx* ctx);

/* Text of the last error on this ctx ("" if none).  Owned by the ctx, valid until its next call.  ctx may be NULL
 * (then a static description of the last create failure). */
const char* starsim_last_error(const starsim_ctx* ctx);

/* Render a full frame with the tiled path: per-star prep, binning of the (tile, star) pairs into
 * per-tile lists in star order (a stable counting sort, or atomic slots + a per-tile sort: starsim_set_binning),
 * then one register-accumulating tile kernel (starsim_set_tile_kernel),
 * free of atomics on the image, that writes every pixel once.  On a non-default stream the launches are captured
 * once into a CUDA graph and replayed while the arguments repeat (STARSIM_NO_GRAPH=1 disables this).
 *   x, y, mag  (device) float[n]: the star catalogue as SoA -- sub-pixel centre (image coordinates) and magnitude.
 *   n          number of stars, >= 0 (0 -> an all-zero image).  x, y, mag may be NULL iff n == 0.
 *   width, height   image size in pixels, each in [1, 32767], width*height < 2^31.
 *   sigma      PSF standard deviation delta of Eq. 2, finite and > 0.
 *   roi        ROI side R in pixels, [1, 255].
 *   gain       A of Eq. 1, finite and >= 0.
 *   out        (device) float[height*width], fully overwritten (0 where no star contributes); must not alias inputs.
 * Per-pixel accumulation is fp32 in star-index order, so the image is bitwise reproducible run to run.
 * Errors: EINVAL (ctx NULL, n < 0, n > 0 with a NULL x/y/mag, out NULL, sizes/sigma/roi/gain out of range),
 *         ENOMEM, ECUDA. */
int starsim_render(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                   int32_t width, int32_t height, float sigma, int32_t roi, float gain,
                   float* out, starsim_stream_t stream);

/* Render rows [row0, row0+rows) of the width x height frame into out_band (device) float[rows*width]: the
 * multi-GPU band decomposition.  Stars are routed to the band iff their clipped ROI rows
 * intersect it.  When row0 and rows are multiples of the tile height the band is bitwise equal to the same rows of
 * starsim_render.  Extra EINVAL: row0 < 0, rows < 1, row0 + rows > height. */
int starsim_render_band(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                        int32_t width, int32_t height, int32_t row0, int32_t rows,
                        float sigma, int32_t roi, float gain, float* out_band, starsim_stream_t stream);

/* Multi-GPU band exchange fused into the render (north star: bands assembled over NVLink 5 / NVSwitch; SURVEY.md
 * §8e): renders rows [row0, row0+rows) exactly like starsim_render_band, but the tile kernel's epilogue stores every
 * pixel of the band straight into each of the ndst full frames dsts[0..ndst), at row row0 + r of each -- the local
 * frame and the peer GPUs' frames mapped into this process (e.g. torch symmetric memory buffer pointers), so the
 * exchange overlaps the tiles still being rendered and no separate all-gather pass is needed.
 *   dsts  (host) array of ndst device pointers, each float[height*width] row-major; 1 <= ndst <= 8.
 * Same EINVAL cases as starsim_render_band, plus ndst outside [1, 8] or a NULL entry.  The library does not
 * synchronise with the peers: the caller orders the stores before any read of a frame (a cross-GPU barrier on the
 * stream, e.g. the symmetric-memory handle's barrier). */
int starsim_render_band_to(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                           int32_t width, int32_t height, int32_t row0, int32_t rows, float sigma, int32_t roi,
                           float gain, float* const* dsts, int32_t ndst, starsim_stream_t stream);

/* The tiled render with the output stage fused into its epilogue: every pixel
 * is written once as the gray value q = min(2^bits - 1, floor(v + 1/2)) (v <= 0 -> 0) of the same fp32 sum v that
 * starsim_render computes, so the result equals starsim_quantize(starsim_render(...)) bit for bit, with a quarter
 * (u8) or half (u16) of the image traffic and no separate pass.
 *   out  (device) uint8_t[height*width] if bits == 8, uint16_t[height*width] if bits == 16.
 * Same arguments and EINVAL cases as starsim_render, plus bits not 8 or 16. */
int starsim_render_gray(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                        int32_t width, int32_t height, float sigma, int32_t roi, float gain, int32_t bits,
                        void* out, starsim_stream_t stream);

/* PSF model of the renders that follow on this ctx (all of render, render_band, render_gray, render_atomic):
 *   STARSIM_PSF_POINT (default): Eq. 2 as the paper writes it, sampled at the pixel coordinate;
 *   STARSIM_PSF_INTEGRATED: Eq. 2 integrated over the pixel square [px-1/2, px+1/2] x
 *     [py-1/2, py+1/2], i.e. g(m) * P(px) * P(py) with P(p) = (erf((p+1/2-X)/(sqrt(2) s)) - erf((p-1/2-X)/(sqrt(2) s)))/2;
 *     same ROI, clipping and summation order.  Still separable, so the tiled path is unchanged but for the profiles.
 * EINVAL: ctx NULL or an unknown mode. */
#define STARSIM_PSF_POINT 0
#define STARSIM_PSF_INTEGRATED 1
int starsim_set_psf(starsim_ctx* ctx, int32_t mode);

/* ROI shape of the renders that follow on this ctx (reading R21):
 *   STARSIM_ROI_SQUARE (default): the R x R square of reading R5/R7 (Fig. 1 caption PAPER.md:19, Fig. 5);
 *   STARSIM_ROI_CIRCLE: the paper's literal "pixel circle" -- the pixels of that square whose centres lie
 *     in the circle inscribed in it: ROI row / column offsets (i, j) with (2j - (R-1))^2 + (2i - (R-1))^2 <= R^2,
 *     an exact integer test, then clipped to the image.  Supported by every render: the star-centric ones (atomic,
 *     lookup table) and the tiled ones (render, render_band, render_band_to, render_gray), which mask the circle per
 *     pixel in the tile kernel's walk -- k_tile_sb's for R <= 17 and k_tile_wide's for 27 <= R <= 65 (whatever
 *     starsim_set_tile_kernel says), k_tile's otherwise -- with the same profiles and the same
 *     deterministic order.
 * EINVAL: ctx NULL or an unknown shape. */
#define STARSIM_ROI_SQUARE 0
#define STARSIM_ROI_CIRCLE 1
int starsim_set_roi(starsim_ctx* ctx, int32_t shape);

/* Binning pipeline of the tiled renders that follow on this ctx.  Both produce the same CSR (each tile's list in
 * ascending star index, reading R18 of DESIGN.md), hence the same image bit for bit:
 *   STARSIM_BIN_AUTO (default): the deterministic counting sort (dbin.cu, no global atomics) when the frame or band
 *     has <= 2048 tiles and R <= 65, else the atomic-slot pipeline;
 *   STARSIM_BIN_ATOMIC: always the atomic-slot pipeline (per-tile counters, scatter, per-tile sort).
 * EINVAL: ctx NULL or an unknown mode. */
#define STARSIM_BIN_AUTO 0
#define STARSIM_BIN_ATOMIC 1
int starsim_set_binning(starsim_ctx* ctx, int32_t mode);

/* Tile-accumulation kernel of the tiled renders that follow on this ctx (render, render_band, render_band_to,
 * render_gray).  All compute Eqs. 2-3 per 128 x 64 tile in fp32 registers with the separable PSF
 * and write every pixel once; they differ in how a tile's star list is walked, hence in the (deterministic)
 * per-pixel summation order:
 *   STARSIM_TILE_AUTO (default): for R <= 17, STARSIM_TILE_WS on dense frames (expected list length per tile
 *     n (127 + R)(63 + R) / (width rows) >= 100, point PSF), else STARSIM_TILE_SB; for 27 <= R <= 65 k_tile_wide
 *     (sorted corner bins of the unclipped ROI origin over <= 5 bands x 9 strips, both roles in every warp); else
 *     the list kernel k_tile;
 *   STARSIM_TILE_LISTS: always the per-block entry-list kernel k_tile (the comparison / any R);
 *   STARSIM_TILE_SB: for R <= 17 k_tile_sb, sorted corner bins with both roles in every warp; for 27 <= R <= 65
 *     k_tile_wide; else k_tile;
 *   STARSIM_TILE_WS: for R <= 17 k_tile_ws, the warp-specialised sorted-corner-bin kernel (producer warps sort and
 *     evaluate profiles into a ring of shared-memory stages while consumer warps accumulate); for
 *     27 <= R <= 65 k_tile_wws, k_tile_wide's warp-specialised form; else k_tile.  SB and WS sum every pixel in the
 *     same order: the same image bit for bit;
 *   STARSIM_TILE_T8: for R <= 17 k_t8sort (every list segment sorted by ROI corner bin into a record array) then
 *     k_tile8 (8 x 8-pixel lane blocks, profile ring in shared memory, warp-specialised); for
 *     27 <= R <= 65 k_tile_wws; else k_tile.
 * Every kernel sums a tile list longer than L stars in L-star segments, each segment's sum added in list order
 * (reading R19), so a tile gives the same bits whether or not it was split across CTAs; L = 1024, and
 * L = 256 for 27 <= R <= 65 (a star there costs up to R^2 FMAs: heavy tiles spread over more CTAs).
 * EINVAL: ctx NULL or an unknown mode. */
#define STARSIM_TILE_AUTO 0
#define STARSIM_TILE_LISTS 1
#define STARSIM_TILE_SB 2
#define STARSIM_TILE_WS 3
#define STARSIM_TILE_T8 4
int starsim_set_tile_kernel(starsim_ctx* ctx, int32_t mode);

/* Band routing: of the catalogue x, y, mag (device, float[n]), the stars whose
 * ROI rows meet rows [row0, row0+rows) of a height-row frame -- first ROI row by reading R7 (the R rows nearest y,
 * ties at k+1/2 upward), exactly the binning's decision; non-finite y never routed -- are written in catalogue order
 * to x_out, y_out, mag_out (device, float[n] each, capacity n; must not alias the inputs), and their number to
 * *n_out (device uint32).  Two kernels (count per 4096-star block, then place), no host synchronisation.  A band
 * rendered from the routed catalogue is bitwise the band rendered from the whole catalogue.  Pair it with
 * starsim_set_star_count(ctx, n_out) to render the routed catalogue without reading the count back.
 * EINVAL: ctx NULL, n < 0 or >= 2^32, a NULL array with n > 0, n_out NULL, height outside [1, 32767], the band not
 * inside the frame, roi outside [1, 255]. */
int starsim_route_band(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n, int32_t height,
                       int32_t row0, int32_t rows, int32_t roi, float* x_out, float* y_out, float* mag_out,
                       uint32_t* n_out, starsim_stream_t stream);

/* Device-resident star count of the tiled renders that follow on this ctx (render, render_band, render_band_to,
 * render_gray): with n_dev (device uint32) set, a render's `n` is the capacity of x, y, mag and the kernels take the
 * first min(n, *n_dev) stars, reading *n_dev when they run (e.g. the n_out of starsim_route_band on the same
 * stream).  NULL (the default) restores plain `n`.  render_atomic / render_lut return EINVAL while it is set.
 * The pointer is kept, not copied: it must stay valid while set.  EINVAL: ctx NULL. */
int starsim_set_star_count(starsim_ctx* ctx, const uint32_t* n_dev);

/* The paper's own design, kept as the measured comparison (Fig. 6): zero the image, then one
 * warp per star adds g*mu into every ROI pixel with global fp32 reductions (red.global.add.f32).  Same arguments
 * and EINVAL cases as starsim_render.  The summation order is nondeterministic. */
int starsim_render_atomic(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                          int32_t width, int32_t height, float sigma, int32_t roi, float gain,
                          float* out, starsim_stream_t stream);

/* NEXT-4: the paper's adaptive simulator (Fig. 8), kept as a second measured comparison: the
 * intensity matrix of Eq. 2 over the R x R ROI for a star at the ROI's centre is tabulated once (the magnitude only
 * scales it: Eq. 1's s' times the one matrix is the paper's magnitude x ROI table), and every star adds s' times the
 * table into its ROI with global fp32 reductions.  Reading R20: each star is taken at the centre of its
 * ROI -- the R nearest pixels of R7, i.e. snapped to the nearest pixel centre for odd R -- so the result is exact
 * for stars on pixel centres and an approximation otherwise (that is the paper's design).  Same arguments and EINVAL
 * cases as starsim_render_atomic, plus roi > 63.  Honours starsim_set_psf.  Summation order nondeterministic. */
#define STARSIM_MAX_LUT_ROI 63
int starsim_render_lut(starsim_ctx* ctx, const float* x, const float* y, const float* mag, int64_t n,
                       int32_t width, int32_t height, float sigma, int32_t roi, float gain,
                       float* out, starsim_stream_t stream);

/* Upload the paper's AoS star records {float mag, posX, posY}[n] (Fig. 6 step 4) from host memory
 * `host_aos` (host, any alignment) and split them into the device SoA arrays x, y, mag (device, float[n] each).
 * The host->device copy goes through a ctx-owned staging buffer on `stream`; the call returns once the host
 * buffer may be reused.  EINVAL: n < 0, or n > 0 with a NULL pointer. */
int starsim_upload_aos(starsim_ctx* ctx, const void* host_aos, int64_t n,
                       float* x, float* y, float* mag, starsim_stream_t stream);

/* Output stage: q = min(2^bits - 1, floor(v + 1/2)) computed exactly, v <= 0 or NaN -> 0.
 *   img (device) float[npix]; out (device) uint8_t[npix] if bits == 8, uint16_t[npix] if bits == 16.
 * EINVAL: npix < 0, NULL pointers with npix > 0, bits not 8 or 16. */
int starsim_quantize(starsim_ctx* ctx, const float* img, int64_t npix, int32_t bits, void* out,
                     starsim_stream_t stream);

/* Introspection of the last starsim_render / starsim_render_band on this ctx (for the bit-exact binning tests):
 * synchronises that call's stream, then copies the CSR to host memory.
 *   *tile_w, *tile_h   tile size in pixels; tiles are numbered key = ty*ceil(width/tile_w) + tx over the frame
 *                      (over the band's rows for render_band, ty counted from row0).
 *   tile_off_host (host) uint32[off_cap]: CSR offsets, ntiles+1 entries are written if off_cap allows.
 *   ids_host      (host) uint32[ids_cap]: star indices, tile-major, star order inside a tile; P entries written.
 *   *n_pairs      P, the number of (tile, star) pairs.
 * EINVAL if no render happened yet or a capacity is too small (*n_pairs is still set). */
int starsim_get_bins(starsim_ctx* ctx, int32_t* tile_w, int32_t* tile_h,
                     uint32_t* tile_off_host, int64_t off_cap, uint32_t* ids_host, int64_t ids_cap,
                     int64_t* n_pairs);

/* Per-kernel device timing for roofline reporting.  When enabled, every launch of the library records CUDA events
 * on the launching stream around it; starsim_kernel_times() synchronises and returns, per kernel class, the summed
 * elapsed milliseconds and launch counts since the last reset.  Classes (index into the arrays):
 *   0 "prep": per-star prep + tile counts (k_dcount, k_prep); 1 "sort": list placement / sorting (k_dplace,
 *   k_sortlists, k_t8sort); 2 "csr": tile scans + scatter (k_dcolscan, k_scan*, k_scatter); 3 "tile": the tile
 *   kernel (k_tile, k_tile_sb, k_tile_ws, k_tile8, k_tile_wide, k_tile_wws); 4 "atomic": the star-centric renders (k_atomic, k_lut);
 *   5 memsets; 6 k_quantize; 7 k_split_aos; 8 "route": k_route_count + k_route_place.
 * While profiling is enabled, renders are launched directly (not through the captured CUDA graph) so that every
 * kernel can be bracketed; kernel durations are unaffected, only the launch gaps differ.
 * `ms` and `launches` must hold STARSIM_NUM_KCLASS entries.  enable != 0 turns recording on and resets. */
#define STARSIM_NUM_KCLASS 9
int starsim_profile(starsim_ctx* ctx, int enable);
int starsim_kernel_times(starsim_ctx* ctx, double* ms, int64_t* launches);

#ifdef __cplusplus
}
#endif
#endif /* STARSIM_H */
