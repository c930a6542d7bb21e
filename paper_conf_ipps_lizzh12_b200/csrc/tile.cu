// Tile accumulation (DESIGN.md §Path step a5).
//
// One warp owns one 32-wide x 64-tall tile.  Lane (c, h) = (lane & 15, lane >> 4) owns columns c and c+16 and the
// 32 rows of parity h (rows 2k+h), as 32 float2 register pairs acc[k] = (pixel(2k+h, c), pixel(2k+h, c+16)).  The
// tile's star list (CSR from the binning, star-index order) is walked in chunks of 32:
//   chunk phase (lane = star): load the star's id and record, clip its ROI to the tile, and evaluate its 1-D row
//     profile s' * exp(-(r-y)^2 / 2 sigma^2) (Eq. 2 is separable: a row factor times a column factor; Eq. 1's
//     brightness and the 1/(2 pi sigma^2) are in s') on the window of 2*NPAR rows that covers the ROI rows, split
//     by parity, into shared memory -- one MUFU.EX2 per value, every lane busy.
//   star phase: the chunk's stars are grouped by window start k0 (one ballot per k0), and each group runs a loop
//     whose body is specialised for its k0: every lane evaluates the column profile at its two columns (MUFU.EX2,
//     masked to the ROI columns by a 32-bit column mask), loads the NPAR row-profile values of its parity
//     (LDS.128) and updates the NPAR register pairs of the window with FFMA2: acc[k] += g[k] * (gx(c), gx(c+16)).
//     Rows outside the window cost nothing.
// The per-pixel order of the fp32 additions is (chunk, window start, star index) -- deterministic, and the same for
// a tile whatever the band decomposition.  The tile is written once, coalesced.  No atomics.
#include <type_traits>

#include "common.cuh"
#include "launch.h"

namespace starsim {

constexpr int CHUNK = 32;
constexpr int PROWS = TILE_H / 2;  // parity rows per lane

template <int KV, int KMAX, typename F>
__device__ __forceinline__ void for_each_window(F&& f) {
  f(std::integral_constant<int, KV>());
  if constexpr (KV < KMAX) for_each_window<KV + 1, KMAX>(f);
}

// NPAR = parity rows per lane per star (a window of 2*NPAR image rows whose start 2*k0 is clamped so that it stays
// inside the tile): 8 for R <= 15, 16 for R <= 31, 32 (the whole tile) beyond.
template <int NPAR>
__global__ void __launch_bounds__(TILE_WARPS * 32) k_tile(const uint32_t* __restrict__ ids,
                                                          const uint32_t* __restrict__ tile_off,
                                                          const StarRec* __restrict__ rec, FrameParams fp,
                                                          float* __restrict__ out) {
  constexpr int KMAX = PROWS - NPAR;
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
  // exp(-d^2 / 2 sigma^2) = 2^(-(d * sk)^2), sk = sqrt(log2(e) / (2 sigma^2)).  d = col - x is formed exactly
  // (tile-relative column minus the tile-relative star x, both exact in fp32) before the one scaling rounding.
  const float sk = fp.sk;
  const float fcA = (float)c, fcB = (float)(c + 16);
  const uint32_t mA = 1u << c, mB = 1u << (c + 16);

  float2 acc[PROWS];
#pragma unroll
  for (int i = 0; i < PROWS; ++i) acc[i] = make_float2(0.f, 0.f);

  const uint32_t j0 = tile_off[t], j1 = tile_off[t + 1];
  for (uint32_t base = j0; base < j1; base += CHUNK) {
    const int cnt = (int)min((uint32_t)CHUNK, j1 - base);
    // ---------------- chunk phase: lane = star
    int k0 = -1;
    if (lane < cnt) {
      const StarRec r = rec[ids[base + lane]];
      const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
      const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TILE_W - 1);
      const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, TILE_H - 1);
      k0 = min(r0 >> 1, KMAX);
      float* g = &s_gy[warp][lane][0];
      const float yr = r.y - (float)IY0;  // star y relative to the tile (exact)
#pragma unroll
      for (int hh = 0; hh < 2; ++hh)
#pragma unroll
        for (int j = 0; j < NPAR; ++j) {
          const int row = 2 * (k0 + j) + hh;
          const float d = ((float)row - yr) * sk;
          const float e = r.s * ex2_approx(-(d * d));
          g[hh * NPAR + j] = (row >= r0 && row <= r1) ? e : 0.f;
        }
      // the ROI's columns of this tile as a bit mask (c1 - c0 <= 31; 2u << 31 wraps to 0 -> all ones)
      const uint32_t bm = ((2u << (uint32_t)(c1 - c0)) - 1u) << c0;
      s_par[warp][lane] = make_float2(r.x - (float)X0, __uint_as_float(bm));
    }
    __syncwarp();
    // ---------------- star phase
    auto star = [&](int s, auto KW) {
      constexpr int K = decltype(KW)::value;
      const float2 par = s_par[warp][s];
      const uint32_t bm = __float_as_uint(par.y);
      const float dA = (fcA - par.x) * sk, dB = (fcB - par.x) * sk;
      const float eA = ex2_approx(-(dA * dA)), eB = ex2_approx(-(dB * dB));
      const float2 gx2 = make_float2((bm & mA) ? eA : 0.f, (bm & mB) ? eB : 0.f);
      const float4* g4 = reinterpret_cast<const float4*>(&s_gy[warp][s][h * NPAR]);
#pragma unroll
      for (int q = 0; q < NPAR / 4; ++q) {
        const float4 u = g4[q];
        acc[K + 4 * q + 0] = __ffma2_rn(make_float2(u.x, u.x), gx2, acc[K + 4 * q + 0]);
        acc[K + 4 * q + 1] = __ffma2_rn(make_float2(u.y, u.y), gx2, acc[K + 4 * q + 1]);
        acc[K + 4 * q + 2] = __ffma2_rn(make_float2(u.z, u.z), gx2, acc[K + 4 * q + 2]);
        acc[K + 4 * q + 3] = __ffma2_rn(make_float2(u.w, u.w), gx2, acc[K + 4 * q + 3]);
      }
    };
    // group the chunk's stars by window start: one ballot per k0, then a loop over that group's stars
    for_each_window<0, KMAX>([&](auto KW) {
      constexpr int K = decltype(KW)::value;
      uint32_t m = __ballot_sync(0xffffffffu, k0 == K);
      while (m) {
        const int s = __ffs(m) - 1;
        m &= m - 1;
        star(s, KW);
      }
    });
    __syncwarp();
  }

  // ---------------- write the tile once: row 2k+h, columns X0+c and X0+c+16
  float* o = out + (int64_t)(Y0 + h) * fp.W + X0 + c;
  const bool okA = X0 + c < fp.W, okB = X0 + c + 16 < fp.W;
#pragma unroll
  for (int k = 0; k < PROWS; ++k) {
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
  else if (fp.R <= 31)
    k_tile<16><<<blocks, TILE_WARPS * 32, 0, st>>>(ids, tile_off, rec, fp, out);
  else
    k_tile<PROWS><<<blocks, TILE_WARPS * 32, 0, st>>>(ids, tile_off, rec, fp, out);
}

}  // namespace starsim
