// Internal definitions shared by the CUDA translation units of libstarsim.so (NOT part of the C ABI).
// Nothing here is shared with oracle/: the oracle is an independent fp64 program (task rule ③).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace starsim {

// Debug builds (-DSTARSIM_CHECKS, e.g. STARSIM_NVCC_EXTRA=-DSTARSIM_CHECKS): device-side bounds and invariant checks
// that trap, standing in for compute-sanitizer where it is unavailable; compiled out otherwise.
#ifdef STARSIM_CHECKS
#define SS_CHECK(c) \
  do {              \
    if (!(c)) __trap(); \
  } while (0)
#else
#define SS_CHECK(c) \
  do {              \
  } while (0)
#endif

// ---------------------------------------------------------------- tile geometry (DESIGN.md §Data layout)
// A tile is the unit of binning and of one k_tile CTA: TILE_W x TILE_H pixels.  Inside it, warp (wx, wy) owns the
// 64 x 16 block at columns 64*wx, rows 16*wy; the block is 8 strips of STRIP_W = 8 columns, one per group of 4 lanes.
constexpr int TILE_W = 128;
constexpr int TILE_H = 64;
constexpr int BAND_H = 16;                       // rows per warp band
constexpr int STRIP_W = 8;                       // columns per lane-group strip
constexpr int NBANDS = TILE_H / BAND_H;          // 4
constexpr int NSTRIPS = TILE_W / STRIP_W;        // 16
constexpr int TILE_WARPS = 8;                    // 2 (x) x 4 (bands)
constexpr int TILE_THREADS = TILE_WARPS * 32;
constexpr int CHUNK = TILE_THREADS;              // stars per chunk of a tile's list (one per thread)
constexpr int GY_CAP = 384;                      // band slots (16 floats: the row profile on one band) per chunk
constexpr int RCAP = 56;                         // strip slots (8 floats: the column profile on one strip) per strip
constexpr int LCAP = 32;                         // entries per (band, strip) list per chunk
constexpr int GX_PAIRS = 768;                    // (star, strip) pairs per chunk
constexpr int WS_MIN_PER_TILE = 100;            // STARSIM_TILE_AUTO picks tile_ws.cu from this expected list length
constexpr int SB_MAXR = 17;                      // tile_sb.cu: an ROI of side <= 17 spans <= 2 bands and <= 3 strips
constexpr int WIDE_MAXR = 65;                    // tile_wide.cu: 17 < R <= 65 (<= 5 bands and <= 9 strips)

// k_prep: one star per thread; per-tile counters CNT_STRIDE words apart (one 128-B line each, so that the
// atomics of different tiles never serialise on one L2 line)
constexpr int CNT_STRIDE = 32;
constexpr int PREP_THREADS = 256;
// dbin.cu (deterministic binning): frames / bands with at most DB_MAXT tiles and R <= DB_MAXR
constexpr int DB_MAXT = 2048;
constexpr int DB_MAXR = 65;                      // an ROI then overlaps at most 2 x 2 tiles
// k_scan_a / k_scan_b: SCAN_PER tiles per thread
constexpr int SCAN_THREADS = 256;
constexpr int SCAN_PER = 4;
constexpr int SCAN_TILES = SCAN_THREADS * SCAN_PER;
// k_sortlists: one tile list per CTA; lists of up to SORT_CAP ids stay in shared memory
constexpr int SORT_THREADS = 128;
constexpr int SORT_CAP = 2048;
constexpr int SORT_CHUNKS = SORT_CAP / SORT_THREADS;  // 32-item chunks per warp: SORT_CAP / (SORT_THREADS/32) / 32
constexpr int SORT_BITS = 8;
constexpr int SORT_RADIX = 1 << SORT_BITS;
constexpr int SORT_NB = 1024;                    // buckets of the range bucket sort

// Per-render header in device scratch, zeroed (with the tile counters) by one cudaMemsetAsync per render.
struct Header {
  uint32_t P;                          // number of (tile, star) pairs
  uint32_t nitems;                     // k_tile work items (written by k_scan)
  uint32_t nsplit;                     // tiles split into several items
  uint32_t next_item;                  // k_tile_sb: the next work item a persistent CTA takes (k_scan zeroes it)
  uint32_t next_seg;                   // k_t8sort: extra-segment slots of its bin-start table taken (zeroed likewise)
  uint32_t lite0;                      // first light item (whole tiles of <= LITE_MAX stars come last, plan.cuh)
  uint32_t pad[26];
};

// k_tile work item: stars [jb, je) of tile `tile`'s list; aux = ITEM_WHOLE, or (split index << 12 | part index) for
// one part of a tile whose list is longer than SPLIT_LEN (heavy tiles of clustered fields, SURVEY.md §7 hard part 5).
struct WorkItem {
  uint32_t tile, jb, je, aux;
};
constexpr uint32_t ITEM_WHOLE = 0xFFFFFFFFu;
// light tiles: a whole tile list of at most LITE_MAX stars (empty included).  The planner puts their items last
// (Header::lite0 on); with k_tile_sb they go to k_tile_lite instead (tile_sb.cu).
#ifndef SB_LITE_MAX
#define SB_LITE_MAX 32
#endif
constexpr int LITE_MAX = SB_LITE_MAX;
constexpr int SPARSE_MAX = 32768;            // catalogues of at most this many stars take the sparse path (AUTO)
#ifndef SPARSE_TESTS_OPT
#define SPARSE_TESTS_OPT (8 << 20)
#endif
constexpr int64_t SPARSE_TESTS = SPARSE_TESTS_OPT;  // ... when stars x tiles (the tile CTAs' star tests) is at most this
#ifndef LITE_AUTO_PER_TILE_OPT
#define LITE_AUTO_PER_TILE_OPT 16.0
#endif
constexpr double LITE_AUTO_PER_TILE = LITE_AUTO_PER_TILE_OPT;  // k_tile_lite is launched when the expected list per
                                                               // tile is <= this
constexpr int64_t LITE_AUTO_TILES = 1024;    // ... and the frame / band has at least this many tiles
constexpr int SPLIT_LEN = 1024;        // a tile list longer than this is split into parts of <= SPLIT_LEN stars
constexpr int PART_CAP = 2048;         // partial-tile buffers (128 x 64 fp32 each, 64 MB) available per render
#ifndef WIDE_SPLIT_OPT
#define WIDE_SPLIT_OPT 256
#endif
constexpr int WIDE_SPLIT = WIDE_SPLIT_OPT;  // the part / segment length for the wide-ROI kernels (FrameParams::split)

// Star record written by k_prep, read by k_scatter and k_tile: {x, y, s', lo_x | lo_y << 16}.
// s' = A * 2.512^-m / (2 pi sigma^2), evaluated in fp64 and rounded once to fp32.
struct __align__(16) StarRec {
  float x, y, s;
  uint32_t lo;  // (uint16)lo_x | (uint16)lo_y << 16 (two's complement int16 each); LO_CULLED if skipped
};
constexpr uint32_t LO_CULLED = 0x80008000u;
__device__ __forceinline__ int lo_x_of(uint32_t lo) { return (int)(int16_t)(lo & 0xFFFFu); }
__device__ __forceinline__ int lo_y_of(uint32_t lo) { return (int)(int16_t)(lo >> 16); }

constexpr int MAX_DST = 8;  // destinations of the fused band exchange (one per GPU of an 8-GPU box)

struct FrameParams {
  int32_t W, H;          // full frame
  int32_t row0, rows;    // band (row0 = 0, rows = H for a full frame)
  int32_t R;
  int32_t ntx, nty;      // tiles over the band
  int32_t vec;           // 1 if every 8-pixel run of an out row is aligned for one vector store
  int32_t vec32;         // fp32 image: 1 if every 8-pixel run is 32-B aligned (one 256-bit store, st.global.v8)
  int32_t obits;         // 0: fp32 image; 8 / 16: gray values quantised in the epilogue (u8 / u16 image)
  int32_t psf;           // 0: Eq. 2 point-sampled (the paper); 1: Eq. 2 integrated over the pixel square (NEXT-2)
  int32_t roi;           // 0: square ROI (reading R5); 1: the pixel circle inscribed in it (NEXT-3, reading R21)
  int32_t tile_impl;     // resolved by render_tiled: 1 the list kernel (tile.cu); 2 tile_sb.cu, 3 tile_ws.cu when R <= SB_MAXR (else tile.cu)
  int32_t bin_impl;      // 0: dbin.cu's deterministic binning when it applies; 1: always bin.cu's atomic-slot pipeline
  int32_t lite;          // 1: k_tile_sb takes items [0, lite0) and k_tile_lite the light items [lite0, nitems)
  int32_t ndst;          // > 0: the tile kernels store every pixel into dst[0..ndst) instead of `out` (fused band exchange)
  float* dst[MAX_DST];   // band origins (row0 of each destination frame) -- local and peer-mapped frames
  const uint32_t* n_dev; // starsim_set_star_count: the star count in device memory (n is then the capacity), or NULL
  int32_t split;         // part / segment length of long tile lists: SPLIT_LEN, or WIDE_SPLIT for k_tile_wide's ROIs
  float sk;              // sqrt(log2(e) / (2 sigma^2)):  exp(-d^2/(2 sigma^2)) = ex2(-(d * sk)^2)
  float kint;            // 1 / (sqrt(2) sigma): the erf argument scale of the integrated PSF
  double s_scale;        // A / (2 pi sigma^2), applied in fp64 before rounding s' to fp32
};

// The number of catalogue entries a kernel takes: n, or the device-resident count of a routed catalogue
// (starsim_route_band -> starsim_set_star_count), read when the kernel runs (no host round trip).
__device__ __forceinline__ int64_t frame_n(int64_t n, const FrameParams& fp) {
  if (!fp.n_dev) return n;
  const int64_t d = (int64_t)*fp.n_dev;
  return d < n ? d : n;
}

// Output stage: q = min(2^bits-1, floor(v + 1/2)), v <= 0 or NaN -> 0.  floor(v + 1/2) is taken
// exactly as f + (v - f >= 1/2), f = floorf(v) (v - f is exact in fp32 for v >= 0); the rounded v + 0.5f would carry
// across an integer for v = 0.49999997 (reading R13).
__device__ __forceinline__ uint32_t quant1(float v, float qmax) {
  float q = 0.f;
  if (v > 0.f) {
    const float f = floorf(v);
    q = f + ((v - f >= 0.5f) ? 1.f : 0.f);
    q = fminf(q, qmax);
  }
  return (uint32_t)q;
}

// NEXT-2: the 1-D pixel mass of the normalised Gaussian between the pixel edges ta < tb (in units of sqrt(2) sigma):
// Phi(tb) - Phi(ta), Phi(t) = erf(t)/2, from e = erfc(|t|) of each edge without cancellation.
__device__ __forceinline__ float edge_erfc(float t) { return erfcf(fabsf(t)); }
__device__ __forceinline__ float pix_mass(float ta, float ea, float tb, float eb) {
  if (ta >= 0.f) return 0.5f * (ea - eb);
  if (tb < 0.f) return 0.5f * (eb - ea);
  return 1.f - 0.5f * (ea + eb);
}

// NEXT-3 (reading R21): ROI pixel at row / column offsets (i, j) from the square ROI's first row / column lies in the
// circle inscribed in the R x R square iff (2j - (R-1))^2 + (2i - (R-1))^2 <= R^2 (integers: exact).
__device__ __forceinline__ bool in_roi_circle(int i, int j, int R) {
  const int u = 2 * j - (R - 1), v = 2 * i - (R - 1);
  return u * u + v * v <= R * R;
}

// MUFU.EX2 (2^x, flush-to-zero): the one SFU op per profile value.
__device__ __forceinline__ float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// First ROI column/row: the R integers nearest to c (ties at k+1/2 round up), lo = floor(c + 1 - R/2), evaluated
// exactly in fp32 (reading R7): f = floor(c) is exact, f + 0.5f is exact for |f| < 2^23, so the
// comparison decides floor(c + 1/2) without the rounding of the naive floorf(c + 1 - R/2).
__device__ __forceinline__ int roi_lo_exact(float c, int R) {
  float f = floorf(c);
  int fi = (int)f;
  if (R & 1) return fi + (c >= f + 0.5f ? 1 : 0) - (R - 1) / 2;
  return fi + 1 - R / 2;
}

}  // namespace starsim
