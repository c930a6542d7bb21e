// Binning of the catalogue into 32x32 image tiles (DESIGN.md §Path steps a1-a4):
//   k_count   a1: per-star prep (validity, s' in fp64, exact ROI origin, clip) + counting of the (tile, star) pairs
//             per tile key with global atomics (the return value is the pair's slot); the last block to finish
//             scans the counts into the CSR offsets.
//   k_scatter a3: every star writes its index into each overlapped tile's segment at the slot k_count took --
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
//   columns and the band rows; one atomic increment per overlapped tile, whose return value is the pair's slot in
//   that tile's segment (kept in slots[i*tps + k], k = the tile's row-major index in the star's tile range).
//   The last block scans the per-tile counts into tile_off[0..ntiles].
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(CNT_THREADS) k_count(const float* __restrict__ X, const float* __restrict__ Y,
                                                       const float* __restrict__ M, int64_t n, FrameParams fp,
                                                       StarRec* __restrict__ rec, uint32_t* cnt,
                                                       uint32_t* __restrict__ slots, int tps, Header* hdr,
                                                       uint32_t* __restrict__ tile_off, uint32_t ntiles) {
  __shared__ uint32_t s_warp[CNT_THREADS / 32];
  __shared__ uint32_t s_max[CNT_THREADS / 32];
  __shared__ bool s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t i = (int64_t)blockIdx.x * CNT_THREADS + tid;
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
        uint32_t* sl = slots + i * tps;
        if (tps == 4) {  // R <= 33: at most 2 x 2 tiles -- issue the (independent) atomics together
          const int key = ty0 * fp.ntx + tx0;
          const bool bx = tx1 > tx0, by = ty1 > ty0;
          uint32_t a = atomicAdd(&cnt[key], 1u), b = 0, c = 0, d = 0;
          if (bx) b = atomicAdd(&cnt[key + 1], 1u);
          if (by) c = atomicAdd(&cnt[key + fp.ntx], 1u);
          if (bx && by) d = atomicAdd(&cnt[key + fp.ntx + 1], 1u);
          // slot order = row-major over the star's tile range
          reinterpret_cast<uint4*>(sl)[0] = bx ? make_uint4(a, b, c, d) : make_uint4(a, c, 0u, 0u);
        } else {
          int k = 0;
          for (int ty = ty0; ty <= ty1; ++ty)
            for (int tx = tx0; tx <= tx1; ++tx) sl[k++] = atomicAdd(&cnt[ty * fp.ntx + tx], 1u);
        }
      } else {
        r.lo = LO_CULLED;
      }
    }
    rec[i] = r;
  }

  // ---- the last block to finish turns counts into CSR offsets (threadFenceReduction pattern).  It scans the
  // counts in chunks of CNT_THREADS * SCAN_V tiles; each thread loads its SCAN_V consecutive counts at once.
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    s_last = atomicAdd(&hdr->done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  uint32_t carry = 0, mx = 0;
  for (uint32_t cb = 0; cb < ntiles; cb += CNT_THREADS * SCAN_V) {
    const uint32_t b0 = cb + (uint32_t)tid * SCAN_V;
    uint32_t v[SCAN_V];
    if (b0 + SCAN_V <= ntiles) {
      const uint4* p = reinterpret_cast<const uint4*>(cnt + b0);  // cnt is 16-B aligned (after the 64-B header)
#pragma unroll
      for (int q = 0; q < SCAN_V / 4; ++q) {
        const uint4 u = __ldcg(p + q);
        v[4 * q] = u.x; v[4 * q + 1] = u.y; v[4 * q + 2] = u.z; v[4 * q + 3] = u.w;
      }
    } else {
#pragma unroll
      for (int e = 0; e < SCAN_V; ++e) v[e] = b0 + e < ntiles ? __ldcg(cnt + b0 + e) : 0u;
    }
    uint32_t sum = 0;
#pragma unroll
    for (int e = 0; e < SCAN_V; ++e) { sum += v[e]; mx = max(mx, v[e]); }
    uint32_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += u;
    }
    if (lane == 31) s_warp[warp] = incl;
    __syncthreads();
    if (tid < 32) {
      uint32_t w = tid < CNT_THREADS / 32 ? s_warp[tid] : 0u, wi = w;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t u = __shfl_up_sync(0xffffffffu, wi, o);
        if (lane >= o) wi += u;
      }
      if (tid < CNT_THREADS / 32) s_warp[tid] = wi - w;   // exclusive prefix of the warp totals
      if (tid == 31) s_max[0] = wi;                        // chunk total
    }
    __syncthreads();
    uint32_t off = carry + s_warp[warp] + incl - sum;
    if (b0 + SCAN_V <= ntiles) {
      uint4* q4 = reinterpret_cast<uint4*>(tile_off + b0);
      uint32_t o[SCAN_V];
#pragma unroll
      for (int e = 0; e < SCAN_V; ++e) { o[e] = off; off += v[e]; }
#pragma unroll
      for (int q = 0; q < SCAN_V / 4; ++q) q4[q] = make_uint4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
    } else {
#pragma unroll
      for (int e = 0; e < SCAN_V; ++e)
        if (b0 + e < ntiles) { tile_off[b0 + e] = off; off += v[e]; }
    }
    carry += s_max[0];
    __syncthreads();
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if (lane == 0) s_warp[warp] = mx;
  __syncthreads();
  if (tid == 0) {
    uint32_t m2 = 0;
    for (int w = 0; w < CNT_THREADS / 32; ++w) m2 = max(m2, s_warp[w]);
    hdr->P = carry;
    hdr->max_seg = m2;
    tile_off[ntiles] = carry;
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_scatter -- step a3: one thread per star writes its index at tile_off[key] + slot for each overlapped tile.
// No atomics: the slots were taken in k_count.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_scatter(const StarRec* __restrict__ rec, int64_t n, FrameParams fp,
                                                 const uint32_t* __restrict__ slots, int tps,
                                                 const uint32_t* __restrict__ tile_off, uint32_t* __restrict__ ids) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  int cx0, cx1, cy0, cy1;
  if (!clip_roi(fp, rec[i].lo, cx0, cx1, cy0, cy1)) return;
  const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
  const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
  const uint32_t* sl = slots + i * tps;
  if (tps == 4) {
    const uint4 s4 = reinterpret_cast<const uint4*>(sl)[0];
    const int key = ty0 * fp.ntx + tx0;
    const bool bx = tx1 > tx0, by = ty1 > ty0;
    ids[tile_off[key] + s4.x] = (uint32_t)i;
    if (bx) ids[tile_off[key + 1] + s4.y] = (uint32_t)i;
    if (by) ids[tile_off[key + fp.ntx] + (bx ? s4.z : s4.y)] = (uint32_t)i;
    if (bx && by) ids[tile_off[key + fp.ntx + 1] + s4.w] = (uint32_t)i;
  } else {
    int k = 0;
    for (int ty = ty0; ty <= ty1; ++ty)
      for (int tx = tx0; tx <= tx1; ++tx) ids[tile_off[ty * fp.ntx + tx] + sl[k++]] = (uint32_t)i;
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_segsort -- step a4: sort every tile segment by star index.  One warp per tile: segments of <= 256 entries in
// registers (bitonic network, E entries per lane, cross-lane stages by SHFL.BFLY), <= SORT_MAX in shared memory,
// longer ones as sorted runs merged through global scratch.
// ---------------------------------------------------------------------------------------------------------------
template <int E>
__device__ __forceinline__ void warp_bitonic_regs(uint32_t (&v)[E], int lane) {
  constexpr int N = 32 * E;
#pragma unroll
  for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      if (j >= E) {  // partner in lane ^ (j / E), same slot
        const int lm = j / E;
        const bool lower = (lane & lm) == 0;
        const bool up = k >= E ? ((lane * E) & k) == 0 : true;
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const bool upe = k >= E ? up : (((lane * E + e) & k) == 0);
          const uint32_t o = __shfl_xor_sync(0xffffffffu, v[e], lm);
          v[e] = (lower == upe) ? min(v[e], o) : max(v[e], o);
        }
      } else {  // partner in the same lane
#pragma unroll
        for (int e = 0; e < E; ++e) {
          if ((e & j) == 0) {
            const int p = e | j;
            const bool up = ((lane * E + e) & k) == 0;
            const uint32_t a = v[e], b = v[p];
            v[e] = up ? min(a, b) : max(a, b);
            v[p] = up ? max(a, b) : min(a, b);
          }
        }
      }
    }
  }
}

template <int E>
__device__ __forceinline__ void sort_small(uint32_t* seg, uint32_t L, int lane) {
  uint32_t v[E];
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const uint32_t idx = (uint32_t)(lane * E + e);
    v[e] = idx < L ? seg[idx] : 0xFFFFFFFFu;
  }
  warp_bitonic_regs<E>(v, lane);
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const uint32_t idx = (uint32_t)(lane * E + e);
    if (idx < L) seg[idx] = v[e];
  }
}

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
  if (L <= 32) { sort_small<1>(seg, L, lane); return; }
  if (L <= 64) { sort_small<2>(seg, L, lane); return; }
  if (L <= 128) { sort_small<4>(seg, L, lane); return; }
  if (L <= 256) { sort_small<8>(seg, L, lane); return; }
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
                  uint32_t* cnt, uint32_t* slots, int tps, Header* hdr, uint32_t* tile_off, uint32_t ntiles,
                  cudaStream_t st) {
  const int64_t nblk = std::max<int64_t>(1, (n + CNT_THREADS - 1) / CNT_THREADS);
  k_count<<<(unsigned)nblk, CNT_THREADS, 0, st>>>(x, y, m, n, fp, rec, cnt, slots, tps, hdr, tile_off, ntiles);
}

void launch_scatter(const StarRec* rec, int64_t n, const FrameParams& fp, const uint32_t* slots, int tps,
                    const uint32_t* tile_off, uint32_t* ids, cudaStream_t st) {
  if (n <= 0) return;
  k_scatter<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(rec, n, fp, slots, tps, tile_off, ids);
}

void launch_segsort(uint32_t* ids, uint32_t* scratch, const uint32_t* tile_off, uint32_t ntiles, cudaStream_t st) {
  k_segsort<<<(ntiles + SORT_WARPS - 1) / SORT_WARPS, SORT_WARPS * 32, 0, st>>>(ids, scratch, tile_off, ntiles);
}

}  // namespace starsim
