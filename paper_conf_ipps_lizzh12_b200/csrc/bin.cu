// Binning of the catalogue into 32x32 image tiles (DESIGN.md §Path steps a1-a4):
//   k_count   a1: per-star prep (validity, s' in fp64, exact ROI origin, clip) + counting of the (tile, star) pairs
//             per tile key with global atomics; the last block to finish scans the counts into the CSR offsets.
//   k_scatter a3: every star writes its index into each overlapped tile's segment (slot from an atomic cursor) --
//             a one-digit (radix 2^keybits) counting sort by tile key.
//   k_segsort a4: restores star-index order inside every tile segment (bitonic in shared memory; heavy segments by
//             a warp merge sort through global scratch), so the CSR is unique and the per-pixel summation order of
//             k_tile is the paper's star order -- bitwise reproducible and identical across band decompositions.
// All sm_100a CUDA, no library calls.
#include <algorithm>

#include "common.cuh"
#include "launch.h"

namespace starsim {

// Clipped ROI of a record against the frame columns and the band rows; false if culled or empty.
__device__ __forceinline__ bool clip_roi(const FrameParams& fp, uint32_t lo, int& cx0, int& cx1, int& cy0, int& cy1) {
  if (lo == LO_CULLED) return false;
  const int lx = lo_x_of(lo), ly = lo_y_of(lo);
  cx0 = max(lx, 0);
  cx1 = min(lx + fp.R - 1, fp.W - 1);
  cy0 = max(ly, fp.row0);
  cy1 = min(ly + fp.R - 1, fp.row0 + fp.rows - 1);
  return cx0 <= cx1 && cy0 <= cy1;
}

// ---------------------------------------------------------------------------------------------------------------
// k_count -- step a1 + tile counting.  One thread per star.
//   reject non-finite x, y, mag (reading R11); s' = A 2.512^-m / (2 pi sigma^2) in fp64 (Eq. 1 with the
//   1/(2 pi sigma^2) of Eq. 2 folded in), rounded once to fp32; exact ROI origin (reading R7); clip to the image
//   columns and the band rows; count one pair per overlapped tile.  The last block scans the per-tile counts into
//   tile_off[0..ntiles] and leaves cnt[t] = tile_off[t] as the scatter cursor.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(SCAN_THREADS) k_count(const float* __restrict__ X, const float* __restrict__ Y,
                                                        const float* __restrict__ M, int64_t n, FrameParams fp,
                                                        StarRec* __restrict__ rec, uint32_t* cnt, Header* hdr,
                                                        uint32_t* __restrict__ tile_off, uint32_t ntiles) {
  __shared__ uint32_t s_warp[SCAN_THREADS / 32];
  __shared__ uint32_t s_max[SCAN_THREADS / 32];
  __shared__ bool s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t i = (int64_t)blockIdx.x * SCAN_THREADS + tid;
  if (i < n) {
    const float x = X[i], y = Y[i], m = M[i];
    const float R = (float)fp.R;
    bool ok = isfinite(x) && isfinite(y) && isfinite(m);
    // pre-filter far-off stars (keeps the int conversions exact); the exact test is the clip below
    ok = ok && x > -R - 2.f && x < (float)fp.W + R + 2.f && y > (float)fp.row0 - R - 2.f &&
         y < (float)(fp.row0 + fp.rows) + R + 2.f;
    StarRec r;
    r.x = x;
    r.y = y;
    r.s = 0.f;
    r.lo = LO_CULLED;
    int cx0, cx1, cy0, cy1;
    if (ok) {
      const int lx = roi_lo_exact(x, fp.R), ly = roi_lo_exact(y, fp.R);
      r.lo = ((uint32_t)(uint16_t)(int16_t)lx) | ((uint32_t)(uint16_t)(int16_t)ly << 16);
      if (clip_roi(fp, r.lo, cx0, cx1, cy0, cy1)) {
        r.s = (float)(fp.s_scale * exp2(-(double)m * 1.3288364642295399628));  // 2.512^-m, Eq. 1
        const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
        const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
        for (int ty = ty0; ty <= ty1; ++ty)
          for (int tx = tx0; tx <= tx1; ++tx) atomicAdd(&cnt[ty * fp.ntx + tx], 1u);
      } else {
        r.lo = LO_CULLED;
      }
    }
    rec[i] = r;
  }

  // ---- the last block to finish turns counts into CSR offsets (threadFenceReduction pattern)
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    s_last = atomicAdd(&hdr->done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const uint32_t per = (ntiles + SCAN_THREADS - 1) / SCAN_THREADS;
  const uint32_t b0 = min(ntiles, tid * per), b1 = min(ntiles, b0 + per);
  uint32_t sum = 0, mx = 0;
  for (uint32_t t = b0; t < b1; ++t) {
    const uint32_t c = __ldcg(&cnt[t]);
    sum += c;
    mx = max(mx, c);
  }
  uint32_t incl = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if (lane == 31) s_warp[warp] = incl;
  if (lane == 0) s_max[warp] = mx;
  __syncthreads();
  if (tid == 0) {
    uint32_t run = 0, m2 = 0;
    for (int w = 0; w < SCAN_THREADS / 32; ++w) {
      const uint32_t v = s_warp[w];
      s_warp[w] = run;
      run += v;
      m2 = max(m2, s_max[w]);
    }
    hdr->P = run;
    hdr->max_seg = m2;
    tile_off[ntiles] = run;
  }
  __syncthreads();
  uint32_t off = s_warp[warp] + incl - sum;
  for (uint32_t t = b0; t < b1; ++t) {
    const uint32_t c = __ldcg(&cnt[t]);
    tile_off[t] = off;
    cnt[t] = off;  // scatter cursor
    off += c;
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_scatter -- step a3: one thread per star, its index into every overlapped tile's segment.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_scatter(const StarRec* __restrict__ rec, int64_t n, FrameParams fp,
                                                 uint32_t* cursor, uint32_t* __restrict__ ids) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  int cx0, cx1, cy0, cy1;
  if (!clip_roi(fp, rec[i].lo, cx0, cx1, cy0, cy1)) return;
  const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
  const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
  for (int ty = ty0; ty <= ty1; ++ty)
    for (int tx = tx0; tx <= tx1; ++tx) ids[atomicAdd(&cursor[ty * fp.ntx + tx], 1u)] = (uint32_t)i;
}

// ---------------------------------------------------------------------------------------------------------------
// k_segsort -- step a4: sort every tile segment by star index.  One warp per tile.
// ---------------------------------------------------------------------------------------------------------------
__device__ void warp_bitonic_smem(uint32_t* s, int p2, int lane) {
  for (int k = 2; k <= p2; k <<= 1)
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = lane; i < p2; i += 32) {
        const int ixj = i ^ j;
        if (ixj > i) {
          const uint32_t a = s[i], b = s[ixj];
          const bool up = (i & k) == 0;
          if ((a > b) == up) {
            s[i] = b;
            s[ixj] = a;
          }
        }
      }
      __syncwarp();
    }
}

__device__ __forceinline__ uint32_t lower_bound_g(const uint32_t* a, uint32_t len, uint32_t v) {
  uint32_t lo = 0, hi = len;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

__global__ void __launch_bounds__(SORT_WARPS * 32) k_segsort(uint32_t* __restrict__ ids, uint32_t* __restrict__ scratch,
                                                            const uint32_t* __restrict__ tile_off, uint32_t ntiles) {
  __shared__ uint32_t s_buf[SORT_WARPS][SORT_MAX];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t t = (int64_t)blockIdx.x * SORT_WARPS + warp;
  if (t >= ntiles) return;
  const uint32_t a = tile_off[t], L = tile_off[t + 1] - a;
  if (L <= 1) return;
  uint32_t* s = s_buf[warp];
  uint32_t* seg = ids + a;
  // runs of SORT_MAX sorted in shared memory (one run unless the tile is heavy)
  for (uint32_t r0 = 0; r0 < L; r0 += SORT_MAX) {
    const uint32_t len = min((uint32_t)SORT_MAX, L - r0);
    int p2 = 32;
    while ((uint32_t)p2 < len) p2 <<= 1;
    for (int i = lane; i < p2; i += 32) s[i] = (uint32_t)i < len ? seg[r0 + i] : 0xFFFFFFFFu;
    __syncwarp();
    warp_bitonic_smem(s, p2, lane);
    for (uint32_t i = lane; i < len; i += 32) seg[r0 + i] = s[i];
    __syncwarp();
  }
  if (L <= SORT_MAX) return;
  // heavy tile: bottom-up merge of the sorted runs through global scratch (ids are unique: rank = lower bound)
  uint32_t* src = seg;
  uint32_t* dst = scratch + a;
  for (uint32_t w = SORT_MAX; w < L; w <<= 1) {
    for (uint32_t lo = 0; lo < L; lo += 2 * w) {
      const uint32_t mid = min(lo + w, L), hi = min(lo + 2 * w, L);
      for (uint32_t i = lo + lane; i < mid; i += 32)
        dst[i + lower_bound_g(src + mid, hi - mid, src[i])] = src[i];
      for (uint32_t j = mid + lane; j < hi; j += 32)
        dst[lo + (j - mid) + lower_bound_g(src + lo, mid - lo, src[j])] = src[j];
    }
    __syncwarp();
    uint32_t* tmp = src;
    src = dst;
    dst = tmp;
  }
  if (src != seg) {
    for (uint32_t i = lane; i < L; i += 32) seg[i] = src[i];
    __syncwarp();
  }
}

// ---------------------------------------------------------------------------------------------------------------
void launch_count(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                  uint32_t* cnt, Header* hdr, uint32_t* tile_off, uint32_t ntiles, cudaStream_t st) {
  const int64_t nblk = std::max<int64_t>(1, (n + SCAN_THREADS - 1) / SCAN_THREADS);
  k_count<<<(unsigned)nblk, SCAN_THREADS, 0, st>>>(x, y, m, n, fp, rec, cnt, hdr, tile_off, ntiles);
}

void launch_scatter(const StarRec* rec, int64_t n, const FrameParams& fp, uint32_t* cursor, uint32_t* ids,
                    cudaStream_t st) {
  if (n <= 0) return;
  k_scatter<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(rec, n, fp, cursor, ids);
}

void launch_segsort(uint32_t* ids, uint32_t* scratch, const uint32_t* tile_off, uint32_t ntiles, cudaStream_t st) {
  k_segsort<<<(ntiles + SORT_WARPS - 1) / SORT_WARPS, SORT_WARPS * 32, 0, st>>>(ids, scratch, tile_off, ntiles);
}

}  // namespace starsim
