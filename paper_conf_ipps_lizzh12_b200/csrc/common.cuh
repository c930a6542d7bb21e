// Internal definitions shared by the CUDA translation units of libstarsim.so (NOT part of the C ABI).
// Nothing here is shared with oracle/: the oracle is an independent fp64 program (task rule ③).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace starsim {

// ---------------------------------------------------------------- tile geometry (DESIGN.md §Data layout)
constexpr int TILE_W = 32;   // tile width  = one warp's 32 lanes, one column per lane
constexpr int TILE_H = 32;   // tile height = 32 fp32 accumulators per lane
constexpr int RADIX_BITS = 8;
constexpr int RADIX = 1 << RADIX_BITS;
constexpr int MAX_PASSES = 3;          // keys < 2^24 (ntiles <= 1024*1024 at 32767^2)

// k_bin: 256 threads x 8 stars
constexpr int BIN_THREADS = 256;
constexpr int BIN_ITEMS = 8;
constexpr int BIN_TILE = BIN_THREADS * BIN_ITEMS;
// k_radix: 256 threads = 8 warps x 16 chunks of 32 pairs
constexpr int RAD_THREADS = 256;
constexpr int RAD_CHUNKS = 16;
constexpr int RAD_TILE = RAD_THREADS * RAD_CHUNKS;
// k_tile: 4 warps per block, one 32x32 tile per warp
constexpr int TILE_WARPS = 4;

// Per-render header in device scratch, zeroed by one cudaMemsetAsync per render.
struct Header {
  uint32_t ticket[8];               // dynamic block ids: [0] k_bin, [1..3] radix passes
  uint32_t P;                       // number of (tile, star) pairs
  uint32_t pad[7];
  uint32_t hist[MAX_PASSES][RADIX]; // digit histograms of all keys, per radix pass
};

// Decoupled look-back status word: tag (30 bits) | flag (2 bits) | value (32 bits).  The tag is unique per
// (render, phase), so the status arrays are never cleared: a word with a stale tag reads as "not ready".
constexpr uint64_t FLAG_AGG = 1ull, FLAG_PREFIX = 2ull;
__device__ __forceinline__ uint64_t pack_status(uint32_t tag, uint64_t flag, uint32_t v) {
  return ((uint64_t)tag << 34) | (flag << 32) | (uint64_t)v;
}
__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// Exclusive prefix of `agg` over all blocks before `blk` for one counter (status[blk*stride]), publishing this
// block's aggregate then inclusive prefix.  Called by one thread per counter.
__device__ __forceinline__ uint32_t lookback(uint64_t* status, int64_t blk, int64_t stride, uint32_t tag,
                                             uint32_t agg) {
  if (blk == 0) {
    st_relaxed(status, pack_status(tag, FLAG_PREFIX, agg));
    return 0;
  }
  st_relaxed(status + blk * stride, pack_status(tag, FLAG_AGG, agg));
  uint32_t excl = 0;
  for (int64_t b = blk - 1; b >= 0; --b) {
    uint64_t w;
    do {
      w = ld_relaxed(status + b * stride);
    } while ((uint32_t)(w >> 34) != (tag & 0x3FFFFFFFu));
    excl += (uint32_t)w;
    if (((w >> 32) & 3ull) == FLAG_PREFIX) break;
  }
  st_relaxed(status + blk * stride, pack_status(tag, FLAG_PREFIX, excl + agg));
  return excl;
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

// Star record written by k_bin, read by k_tile: {x, y, s', lo_x | lo_y << 16}.
// s' = A * 2.512^-m / (2 pi sigma^2), evaluated in fp64 and rounded once to fp32.
struct __align__(16) StarRec {
  float x, y, s;
  uint32_t lo;  // (uint16)lo_x | (uint16)lo_y << 16 (two's complement int16 each)
};
__device__ __forceinline__ int lo_x_of(uint32_t lo) { return (int)(int16_t)(lo & 0xFFFFu); }
__device__ __forceinline__ int lo_y_of(uint32_t lo) { return (int)(int16_t)(lo >> 16); }

struct FrameParams {
  int32_t W, H;          // full frame
  int32_t row0, rows;    // band (row0 = 0, rows = H for a full frame)
  int32_t R;
  int32_t ntx, nty;      // tiles over the band
  float kexp;            // -log2(e) / (2 sigma^2): exp(-d^2/(2 sigma^2)) = ex2(kexp * d^2)
  double s_scale;        // A / (2 pi sigma^2), applied in fp64 before rounding s' to fp32
};

}  // namespace starsim
