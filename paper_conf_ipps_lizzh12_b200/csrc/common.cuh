// Internal definitions shared by the CUDA translation units of libstarsim.so (NOT part of the C ABI).
// Nothing here is shared with oracle/: the oracle is an independent fp64 program (task rule ③).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace starsim {

// ---------------------------------------------------------------- tile geometry (DESIGN.md §Data layout)
constexpr int TILE_W = 32;   // tile width: one warp, 16 columns x 2 halves per lane
constexpr int TILE_H = 64;   // tile height: 32 rows of one parity per lane, in fp32 registers

// k_bin: BIN_THREADS threads x BIN_ITEMS stars per block
constexpr int BIN_THREADS = 256;
constexpr int BIN_ITEMS = 4;
constexpr int BIN_TILE = BIN_THREADS * BIN_ITEMS;
// k_radix: RAD_THREADS threads = 8 warps x RAD_CHUNKS chunks of 32 pairs per block; digits of <= 10 bits
constexpr int RAD_THREADS = 256;
constexpr int RAD_CHUNKS = 16;
constexpr int RAD_TILE = RAD_THREADS * RAD_CHUNKS;
constexpr int MAX_RADIX_BITS = 10;
constexpr int MAX_RADIX = 1 << MAX_RADIX_BITS;
// k_tile: 4 warps per block, one tile per warp
constexpr int TILE_WARPS = 4;

// Per-render header in device scratch, zeroed (with the look-back status arrays) by one cudaMemsetAsync per render.
struct Header {
  uint32_t ticket[4];                  // dynamic block ids: [0] k_bin, [1], [2] radix passes
  uint32_t P;                          // number of (tile, star) pairs
  uint32_t pad[11];
  uint32_t hist[2][MAX_RADIX];         // digit histograms of all keys for the (at most two) radix passes
};

// Star record written by k_count, read by k_scatter and k_tile: {x, y, s', lo_x | lo_y << 16}.
// s' = A * 2.512^-m / (2 pi sigma^2), evaluated in fp64 and rounded once to fp32.
struct __align__(16) StarRec {
  float x, y, s;
  uint32_t lo;  // (uint16)lo_x | (uint16)lo_y << 16 (two's complement int16 each); LO_CULLED if skipped
};
constexpr uint32_t LO_CULLED = 0x80008000u;
__device__ __forceinline__ int lo_x_of(uint32_t lo) { return (int)(int16_t)(lo & 0xFFFFu); }
__device__ __forceinline__ int lo_y_of(uint32_t lo) { return (int)(int16_t)(lo >> 16); }

struct FrameParams {
  int32_t W, H;          // full frame
  int32_t row0, rows;    // band (row0 = 0, rows = H for a full frame)
  int32_t R;
  int32_t ntx, nty;      // tiles over the band
  float kexp;            // -log2(e) / (2 sigma^2): exp(-d^2/(2 sigma^2)) = ex2(kexp * d^2)
  float sk;              // sqrt(log2(e) / (2 sigma^2)):  exp(-d^2/(2 sigma^2)) = ex2(-(d * sk)^2)
  double s_scale;        // A / (2 pi sigma^2), applied in fp64 before rounding s' to fp32
};

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
