// Band routing: the stars whose ROI rows meet the band [row0, row0 + rows),
// compacted in catalogue order into x_out / y_out / mag_out, their number written to device memory.  A band rendered
// from the routed catalogue has the same tile lists, in the same relative order, as the band rendered from the whole
// catalogue (the binning clips every star to the band and keeps star order), so the image is the same bit for bit.
//
//   k_route_count    CTA b: the number of routed stars among [b RT_CTA, (b+1) RT_CTA)        -> blk[b]
//   k_route_place    CTA b: its output offset (sum of blk[0..b)), then its routed stars in order (warp ballots +
//                    one block scan per round of RT_THREADS stars); the last CTA writes the total to *n_out.
//
// The routing rule is the first ROI row of reading R7 (roi_lo_exact, the same decision the binning takes) against
// the band rows; a non-finite y is never routed (the binning culls it anyway, reading R11).  Only y decides: stars
// with a non-finite x or magnitude, or an ROI outside the columns, are routed and culled later by the binning.
#include "common.cuh"
#include "launch.h"

namespace starsim {

constexpr int RT_THREADS = 256;
constexpr int RT_PER = 16;
constexpr int RT_CTA = RT_THREADS * RT_PER;  // stars per CTA
constexpr int RT_WARPS = RT_THREADS / 32;

__device__ __forceinline__ bool routed(float y, int row0, int rows, int R) {
  // pre-filter (also rejects NaN / inf): outside it the ROI rows cannot meet the band, inside it the ints are exact
  if (!(y > (float)(row0 - R - 2) && y < (float)(row0 + rows + R + 2))) return false;
  const int ly = roi_lo_exact(y, R);
  return ly <= row0 + rows - 1 && ly + R - 1 >= row0;
}

__device__ __forceinline__ uint32_t block_sum(uint32_t v, uint32_t* s_w) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) s_w[warp] = v;
  __syncthreads();
  uint32_t t = 0u;
#pragma unroll
  for (int w = 0; w < RT_WARPS; ++w) t += s_w[w];
  __syncthreads();
  return t;
}

__global__ void __launch_bounds__(RT_THREADS) k_route_count(const float* __restrict__ Y, int64_t n, int32_t row0,
                                                            int32_t rows, int32_t R, uint32_t* __restrict__ blk) {
  __shared__ uint32_t s_w[RT_WARPS];
  const int64_t i0 = (int64_t)blockIdx.x * RT_CTA + threadIdx.x;
  float ys[RT_PER];
#pragma unroll
  for (int k = 0; k < RT_PER; ++k) {
    const int64_t i = i0 + (int64_t)k * RT_THREADS;
    ys[k] = i < n ? __ldg(&Y[i]) : __int_as_float(0x7fc00000);  // NaN: not routed
  }
  uint32_t c = 0u;
#pragma unroll
  for (int k = 0; k < RT_PER; ++k) c += routed(ys[k], row0, rows, R) ? 1u : 0u;
  c = block_sum(c, s_w);
  if (threadIdx.x == 0) blk[blockIdx.x] = c;
}

__global__ void __launch_bounds__(RT_THREADS) k_route_place(const float* __restrict__ X, const float* __restrict__ Y,
                                                            const float* __restrict__ M, int64_t n, int32_t row0,
                                                            int32_t rows, int32_t R,
                                                            const uint32_t* __restrict__ blk, float* __restrict__ Xo,
                                                            float* __restrict__ Yo, float* __restrict__ Mo,
                                                            uint32_t* __restrict__ n_out) {
  __shared__ uint32_t s_w[RT_WARPS];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, b = blockIdx.x;
  const int64_t i0 = (int64_t)b * RT_CTA + tid;
  float ys[RT_PER];
#pragma unroll
  for (int k = 0; k < RT_PER; ++k) {
    const int64_t i = i0 + (int64_t)k * RT_THREADS;
    ys[k] = i < n ? __ldg(&Y[i]) : __int_as_float(0x7fc00000);
  }
  // this CTA's first output position: the routed stars of the CTAs before it
  uint32_t pre = 0u;
  for (int j = tid; j < b; j += RT_THREADS) pre += __ldg(&blk[j]);
  uint32_t base = block_sum(pre, s_w);
  const uint32_t lt = (1u << lane) - 1u;
#pragma unroll
  for (int k = 0; k < RT_PER; ++k) {
    const bool f = routed(ys[k], row0, rows, R);
    const uint32_t bal = __ballot_sync(0xffffffffu, f);
    if (lane == 0) s_w[warp] = __popc(bal);
    __syncthreads();
    uint32_t wpre = 0u, tot = 0u;
#pragma unroll
    for (int w = 0; w < RT_WARPS; ++w) {
      const uint32_t c = s_w[w];
      wpre += w < warp ? c : 0u;
      tot += c;
    }
    if (f) {
      const int64_t i = i0 + (int64_t)k * RT_THREADS;
      const uint32_t o = base + wpre + __popc(bal & lt);
      Xo[o] = __ldg(&X[i]);
      Yo[o] = ys[k];
      Mo[o] = __ldg(&M[i]);
    }
    base += tot;
    __syncthreads();
  }
  if (b == gridDim.x - 1 && tid == 0) *n_out = base;
}

size_t route_blocks(int64_t n) { return (size_t)((n + RT_CTA - 1) / RT_CTA); }

void launch_route(const float* x, const float* y, const float* m, int64_t n, int32_t row0, int32_t rows, int32_t R,
                  uint32_t* blk, float* xo, float* yo, float* mo, uint32_t* n_out, cudaStream_t st) {
  const unsigned nb = (unsigned)route_blocks(n);
  if (nb == 0) {
    cudaMemsetAsync(n_out, 0, sizeof(uint32_t), st);
    return;
  }
  k_route_count<<<nb, RT_THREADS, 0, st>>>(y, n, row0, rows, R, blk);
  k_route_place<<<nb, RT_THREADS, 0, st>>>(x, y, m, n, row0, rows, R, blk, xo, yo, mo, n_out);
}

}  // namespace starsim
