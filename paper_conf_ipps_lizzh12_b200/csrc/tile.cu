// Tile accumulation (DESIGN.md §Path step a5): one warp owns one 32x32 tile of the image, one
// column per lane and the 32 rows of that column in fp32 registers.  It walks the tile's star list (CSR from the
// radix sort, star-index order) and, per star, evaluates the separable PSF of Eq. 2 -- a 1-D Gaussian column
// profile gx (one MUFU.EX2 per lane) times a 1-D row profile s'*gy (one MUFU.EX2 per row, staged through shared
// memory) -- and accumulates acc[r] += (s' gy[r]) * gx with FFMA2 over a row window that starts at the star's first
// row (warp-uniform jump table), so no work is spent on rows outside the ROI.  No atomics: every pixel is owned by
// exactly one lane and is written once, coalesced (128 B per row).
#include "common.cuh"
#include "launch.h"

namespace starsim {

template <int K, int NP>
__device__ __forceinline__ void fma_window(float2 (&acc)[24], const float2 (&g)[8], float2 gx2) {
#pragma unroll
  for (int j = 0; j < NP; ++j) acc[K + j] = __ffma2_rn(g[j], gx2, acc[K + j]);
}

// WIN = 16: R <= 15, rows processed in a 16-row window starting at the star's first (even-aligned) row.
// WIN = 32: any R, all 32 rows of the tile.
template <int WIN>
__global__ void __launch_bounds__(TILE_WARPS * 32) k_tile(const uint64_t* __restrict__ sorted,
                                                          const uint32_t* __restrict__ tile_off,
                                                          const StarRec* __restrict__ rec, FrameParams fp,
                                                          float* __restrict__ out) {
  __shared__ __align__(16) float s_g[TILE_WARPS][32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t t = (int64_t)blockIdx.x * TILE_WARPS + warp;
  if (t >= (int64_t)fp.ntx * fp.nty) return;
  const int tx = (int)(t % fp.ntx), ty = (int)(t / fp.ntx);
  const int X0 = tx * TILE_W;        // first column of the tile
  const int Y0 = ty * TILE_H;        // first row of the tile, relative to the band
  const int IY0 = fp.row0 + Y0;      // first image row of the tile
  const float fcol = (float)(X0 + lane);

  float2 acc[24];
#pragma unroll
  for (int i = 0; i < 24; ++i) acc[i] = make_float2(0.f, 0.f);

  const uint32_t j0 = tile_off[t], j1 = tile_off[t + 1];
  for (uint32_t j = j0; j < j1; ++j) {
    const uint32_t star = (uint32_t)sorted[j];
    const StarRec r = rec[star];
    const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
    const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TILE_W - 1);
    const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, TILE_H - 1);
    const float dx = fcol - r.x;
    const float gx = (lane >= c0 && lane <= c1) ? ex2_approx(fp.kexp * (dx * dx)) : 0.f;
    const int k0 = (WIN == 32) ? 0 : (r0 & ~1);
    if (lane < WIN) {
      const int rr = k0 + lane;
      const float dy = (float)(IY0 + rr) - r.y;
      s_g[warp][lane] = (rr >= r0 && rr <= r1) ? r.s * ex2_approx(fp.kexp * (dy * dy)) : 0.f;
    }
    __syncwarp();
    const float2 gx2 = make_float2(gx, gx);
    if (WIN == 32) {
      const float4* g4 = reinterpret_cast<const float4*>(&s_g[warp][0]);
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const float4 v = g4[q];
        acc[2 * q] = __ffma2_rn(make_float2(v.x, v.y), gx2, acc[2 * q]);
        acc[2 * q + 1] = __ffma2_rn(make_float2(v.z, v.w), gx2, acc[2 * q + 1]);
      }
    } else {
      float2 g[8];
      const float4* g4 = reinterpret_cast<const float4*>(&s_g[warp][0]);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const float4 v = g4[q];
        g[2 * q] = make_float2(v.x, v.y);
        g[2 * q + 1] = make_float2(v.z, v.w);
      }
      switch (k0 >> 1) {
#define STARSIM_CASE(i) \
  case i:               \
    fma_window<i, 8>(acc, g, gx2); \
    break;
        STARSIM_CASE(0) STARSIM_CASE(1) STARSIM_CASE(2) STARSIM_CASE(3) STARSIM_CASE(4) STARSIM_CASE(5)
        STARSIM_CASE(6) STARSIM_CASE(7) STARSIM_CASE(8) STARSIM_CASE(9) STARSIM_CASE(10) STARSIM_CASE(11)
        STARSIM_CASE(12) STARSIM_CASE(13) STARSIM_CASE(14) STARSIM_CASE(15)
#undef STARSIM_CASE
        default: break;
      }
    }
    __syncwarp();
  }

  // write the tile once: row r of the tile is 32 consecutive floats (128 B) -> one coalesced store per row
  const int col = X0 + lane;
  if (col < fp.W) {
    float* o = out + (int64_t)Y0 * fp.W + col;
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      const int rr = 2 * i;
      if (Y0 + rr < fp.rows) o[(int64_t)rr * fp.W] = acc[i].x;
      if (Y0 + rr + 1 < fp.rows) o[(int64_t)(rr + 1) * fp.W] = acc[i].y;
    }
  }
}

void launch_tile(const uint64_t* sorted, const uint32_t* tile_off, const StarRec* rec, const FrameParams& fp,
                 float* out, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  const unsigned blocks = (unsigned)((ntiles + TILE_WARPS - 1) / TILE_WARPS);
  if (fp.R <= 15)
    k_tile<16><<<blocks, TILE_WARPS * 32, 0, st>>>(sorted, tile_off, rec, fp, out);
  else
    k_tile<32><<<blocks, TILE_WARPS * 32, 0, st>>>(sorted, tile_off, rec, fp, out);
}

}  // namespace starsim
