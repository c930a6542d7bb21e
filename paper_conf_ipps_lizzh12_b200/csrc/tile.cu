// Tile accumulation (DESIGN.md §Path step a5).
//
// One warp owns one 32x32 tile.  Lane (c, h) = (lane & 15, lane >> 4) owns columns c and c+16 and the 16 rows of
// parity h (rows 2k+h), as 16 float2 register pairs acc[k] = (pixel(2k+h, c), pixel(2k+h, c+16)).  The tile's star
// list (CSR from the binning, star-index order) is walked in chunks of 32:
//   chunk phase (lane = star): load the star's id and record, clip its ROI to the tile, and evaluate its 1-D row
//     profile s' * exp(-(r-y)^2 / 2 sigma^2) (Eq. 2 is separable: a row factor times a column factor; Eq. 1's
//     brightness and the 1/(2 pi sigma^2) are in s') on the 16-row window that covers the ROI rows, split by parity,
//     into shared memory -- one MUFU.EX2 per value, every lane busy.
//   star phase (warp-uniform loop over the chunk): each lane evaluates the column profile at its two columns (one
//     MUFU.EX2 each, skipped for a half the ROI misses), loads the 8 row-profile values of its parity (2 x LDS.128),
//     and updates the 8 register pairs of the window with FFMA2: acc[k] += g[k] * (gx(c), gx(c+16)).  The window
//     start is warp-uniform (one jump into 16 specialised bodies), so rows outside the ROI cost nothing.
// Per-pixel accumulation is fp32 in star-index order; the tile is written once, coalesced.  No atomics.
#include "common.cuh"
#include "launch.h"

namespace starsim {

constexpr int CHUNK = 32;

template <int K>
__device__ __forceinline__ void fma_window8(float2 (&acc)[24], const float (&g)[8], float2 gx2) {
#pragma unroll
  for (int j = 0; j < 8; ++j) acc[K + j] = __ffma2_rn(make_float2(g[j], g[j]), gx2, acc[K + j]);
}

// NPAR = parity rows per lane per star: 8 for R <= 15 (16-row window), 16 for larger R (the whole tile).
template <int NPAR>
__global__ void __launch_bounds__(TILE_WARPS * 32) k_tile(const uint32_t* __restrict__ ids,
                                                          const uint32_t* __restrict__ tile_off,
                                                          const StarRec* __restrict__ rec, FrameParams fp,
                                                          float* __restrict__ out) {
  __shared__ __align__(16) float s_gy[TILE_WARPS][CHUNK][2 * NPAR];
  __shared__ __align__(8) float2 s_par[TILE_WARPS][CHUNK];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int c = lane & 15, h = lane >> 4;
  const int64_t t = (int64_t)blockIdx.x * TILE_WARPS + warp;
  if (t >= (int64_t)fp.ntx * fp.nty) return;
  const int tx = (int)(t % fp.ntx), ty = (int)(t / fp.ntx);
  const int X0 = tx * TILE_W;    // first column of the tile
  const int Y0 = ty * TILE_H;    // first row of the tile, relative to the band
  const int IY0 = fp.row0 + Y0;  // first image row of the tile
  const float fcA = (float)c, fcB = (float)(c + 16);
  const float kexp = fp.kexp;

  float2 acc[24];
#pragma unroll
  for (int i = 0; i < 24; ++i) acc[i] = make_float2(0.f, 0.f);

  const uint32_t j0 = tile_off[t], j1 = tile_off[t + 1];
  for (uint32_t base = j0; base < j1; base += CHUNK) {
    const int cnt = (int)min((uint32_t)CHUNK, j1 - base);
    // ---------------- chunk phase: lane = star
    if (lane < cnt) {
      const StarRec r = rec[ids[base + lane]];
      const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
      const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TILE_W - 1);
      const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, TILE_H - 1);
      const int k0 = NPAR == 8 ? (r0 >> 1) : 0;
      float* g = &s_gy[warp][lane][0];
#pragma unroll
      for (int hh = 0; hh < 2; ++hh)
#pragma unroll
        for (int j = 0; j < NPAR; ++j) {
          const int row = 2 * (k0 + j) + hh;
          const float dy = (float)(IY0 + row) - r.y;
          g[hh * NPAR + j] = (row >= r0 && row <= r1) ? r.s * ex2_approx(kexp * (dy * dy)) : 0.f;
        }
      s_par[warp][lane] = make_float2((float)X0 - r.x, __uint_as_float((uint32_t)c0 | ((uint32_t)c1 << 8) |
                                                                          ((uint32_t)k0 << 16)));
    }
    __syncwarp();
    // ---------------- star phase: warp-uniform loop
    for (int s = 0; s < cnt; ++s) {
      const float2 par = s_par[warp][s];
      const uint32_t pk = __float_as_uint(par.y);
      const int c0 = (int)(pk & 0xFF), c1 = (int)((pk >> 8) & 0xFF), k0 = (int)(pk >> 16);
      float gxA = 0.f, gxB = 0.f;
      if (c0 < 16) {
        const float d = fcA + par.x;
        gxA = ((unsigned)(c - c0) <= (unsigned)(c1 - c0)) ? ex2_approx(kexp * (d * d)) : 0.f;
      }
      if (c1 >= 16) {
        const float d = fcB + par.x;
        gxB = ((unsigned)(c + 16 - c0) <= (unsigned)(c1 - c0)) ? ex2_approx(kexp * (d * d)) : 0.f;
      }
      const float2 gx2 = make_float2(gxA, gxB);
      if (NPAR == 8) {
        const float4* g4 = reinterpret_cast<const float4*>(&s_gy[warp][s][h * 8]);
        const float4 u = g4[0], v = g4[1];
        const float g[8] = {u.x, u.y, u.z, u.w, v.x, v.y, v.z, v.w};
        switch (k0) {
#define STARSIM_CASE(i) \
  case i:               \
    fma_window8<i>(acc, g, gx2); \
    break;
          STARSIM_CASE(0) STARSIM_CASE(1) STARSIM_CASE(2) STARSIM_CASE(3) STARSIM_CASE(4) STARSIM_CASE(5)
          STARSIM_CASE(6) STARSIM_CASE(7) STARSIM_CASE(8) STARSIM_CASE(9) STARSIM_CASE(10) STARSIM_CASE(11)
          STARSIM_CASE(12) STARSIM_CASE(13) STARSIM_CASE(14) STARSIM_CASE(15)
#undef STARSIM_CASE
          default: break;
        }
      } else {
        const float4* g4 = reinterpret_cast<const float4*>(&s_gy[warp][s][h * 16]);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const float4 u = g4[q];
          acc[4 * q + 0] = __ffma2_rn(make_float2(u.x, u.x), gx2, acc[4 * q + 0]);
          acc[4 * q + 1] = __ffma2_rn(make_float2(u.y, u.y), gx2, acc[4 * q + 1]);
          acc[4 * q + 2] = __ffma2_rn(make_float2(u.z, u.z), gx2, acc[4 * q + 2]);
          acc[4 * q + 3] = __ffma2_rn(make_float2(u.w, u.w), gx2, acc[4 * q + 3]);
        }
      }
    }
    __syncwarp();
  }

  // ---------------- write the tile once: row 2k+h, columns X0+c and X0+c+16
  float* o = out + (int64_t)(Y0 + h) * fp.W + X0 + c;
  const bool okA = X0 + c < fp.W, okB = X0 + c + 16 < fp.W;
#pragma unroll
  for (int k = 0; k < 16; ++k) {
    if (Y0 + 2 * k + h < fp.rows) {
      if (okA) o[(int64_t)(2 * k) * fp.W] = acc[k].x;
      if (okB) o[(int64_t)(2 * k) * fp.W + 16] = acc[k].y;
    }
  }
}

void launch_tile(const uint32_t* ids, const uint32_t* tile_off, const StarRec* rec, const FrameParams& fp,
                 float* out, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  const unsigned blocks = (unsigned)((ntiles + TILE_WARPS - 1) / TILE_WARPS);
  if (fp.R <= 15)
    k_tile<8><<<blocks, TILE_WARPS * 32, 0, st>>>(ids, tile_off, rec, fp, out);
  else
    k_tile<16><<<blocks, TILE_WARPS * 32, 0, st>>>(ids, tile_off, rec, fp, out);
}

}  // namespace starsim
