// Binning: per-star prep + scan + emit of (tile, star) pairs (k_bin), stable LSD radix sort (k_radix), CSR tile
// offsets (k_offsets).  DESIGN.md §Path steps a1-a4.  All sm_100a CUDA, no library calls.
#include <algorithm>

#include "common.cuh"
#include "launch.h"

namespace starsim {

// ---------------------------------------------------------------------------------------------------------------
// k_bin -- one pass over the catalogue (step a1 + a2 + a3 + the radix histograms):
//   per star: reject non-finite x, y, mag (reading R11); s' = A 2.512^-m / (2 pi sigma^2) in fp64 (Eq. 1 with the
//   1/(2 pi sigma^2) of Eq. 2 folded in); exact ROI origin (reading R7); clip to the image columns and the band rows;
//   count the 32x32 tiles the clipped ROI overlaps; single-pass exclusive scan of the counts over stars (decoupled
//   look-back across blocks); emit the star's pairs (key = ty*ntx + tx, value = star index) in star order, tiles
//   row-major; histogram the radix digits of every key.
// Layout: 256 threads x 8 stars, striped loads (coalesced), blocked scan through shared memory.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(BIN_THREADS) k_bin(const float* __restrict__ X, const float* __restrict__ Y,
                                                     const float* __restrict__ M, int64_t n, FrameParams fp,
                                                     StarRec* __restrict__ rec, uint64_t* __restrict__ pairs,
                                                     Header* hdr, uint64_t* status, uint32_t tag, int passes) {
  __shared__ uint32_t s_cnt[BIN_TILE];
  __shared__ uint32_t s_hist[MAX_PASSES][RADIX];
  __shared__ uint32_t s_warp[BIN_THREADS / 32];
  __shared__ uint32_t s_base;
  __shared__ int64_t s_blk;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_blk = atomicAdd(&hdr->ticket[0], 1u);
  for (int i = tid; i < MAX_PASSES * RADIX; i += BIN_THREADS) (&s_hist[0][0])[i] = 0;
  __syncthreads();
  const int64_t blk = s_blk;
  const int64_t base = blk * BIN_TILE;

  // ---- a1: per-star prep (striped: star base + k*256 + tid)
  uint32_t cnts[BIN_ITEMS];      // tiles per star
  uint16_t tr[BIN_ITEMS][4];     // its tile range tx0, tx1, ty0, ty1
#pragma unroll
  for (int k = 0; k < BIN_ITEMS; ++k) {
    const int64_t i = base + k * BIN_THREADS + tid;
    uint32_t cnt = 0;
    if (i < n) {
      const float x = X[i], y = Y[i], m = M[i];
      const float R = (float)fp.R;
      bool ok = isfinite(x) && isfinite(y) && isfinite(m);
      // pre-filter far-off stars (keeps the int conversions exact); the exact test is the clip below
      ok = ok && x > -R - 2.f && x < (float)fp.W + R + 2.f && y > (float)fp.row0 - R - 2.f &&
           y < (float)(fp.row0 + fp.rows) + R + 2.f;
      int lx = 0, ly = 0, cx0 = 0, cx1 = -1, cy0 = 0, cy1 = -1;
      if (ok) {
        lx = roi_lo_exact(x, fp.R);
        ly = roi_lo_exact(y, fp.R);
        cx0 = max(lx, 0);
        cx1 = min(lx + fp.R - 1, fp.W - 1);
        cy0 = max(ly, fp.row0);
        cy1 = min(ly + fp.R - 1, fp.row0 + fp.rows - 1);
        ok = cx0 <= cx1 && cy0 <= cy1;
      }
      StarRec r;
      r.x = x;
      r.y = y;
      r.s = ok ? (float)(fp.s_scale * pow(2.512, -(double)m)) : 0.f;
      r.lo = ((uint32_t)(uint16_t)(int16_t)lx) | ((uint32_t)(uint16_t)(int16_t)ly << 16);
      rec[i] = r;
      if (ok) {
        const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
        const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
        tr[k][0] = (uint16_t)tx0; tr[k][1] = (uint16_t)tx1; tr[k][2] = (uint16_t)ty0; tr[k][3] = (uint16_t)ty1;
        cnt = (uint32_t)((tx1 - tx0 + 1) * (ty1 - ty0 + 1));
      }
    }
    cnts[k] = cnt;
    s_cnt[k * BIN_THREADS + tid] = cnt;
  }
  __syncthreads();

  // ---- a2: block-wide exclusive scan in star order (thread t owns stars t*8 .. t*8+7 of the block)
  uint32_t v[BIN_ITEMS], tsum = 0;
#pragma unroll
  for (int j = 0; j < BIN_ITEMS; ++j) { v[j] = s_cnt[tid * BIN_ITEMS + j]; tsum += v[j]; }
  uint32_t incl = tsum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += t;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (tid == 0) {
    uint32_t run = 0;
    for (int w = 0; w < BIN_THREADS / 32; ++w) { uint32_t t = s_warp[w]; s_warp[w] = run; run += t; }
    // cross-block decoupled look-back: exclusive prefix of this block
    const uint32_t excl = lookback(status, blk, 1, tag, run);
    s_base = excl;
    const int64_t nblk = (n + BIN_TILE - 1) / BIN_TILE;
    if (blk == nblk - 1) hdr->P = excl + run;
  }
  __syncthreads();
  {
    uint32_t off = s_base + s_warp[warp] + incl - tsum;
#pragma unroll
    for (int j = 0; j < BIN_ITEMS; ++j) { s_cnt[tid * BIN_ITEMS + j] = off; off += v[j]; }
  }
  __syncthreads();

  // ---- a3: emit pairs in star order; histogram every pass's digit
#pragma unroll
  for (int k = 0; k < BIN_ITEMS; ++k) {
    if (cnts[k] == 0) continue;
    const int64_t i = base + k * BIN_THREADS + tid;
    uint32_t o = s_cnt[k * BIN_THREADS + tid];
    for (int ty = tr[k][2]; ty <= tr[k][3]; ++ty)
      for (int tx = tr[k][0]; tx <= tr[k][1]; ++tx) {
        const uint32_t key = (uint32_t)ty * (uint32_t)fp.ntx + (uint32_t)tx;
        pairs[o++] = ((uint64_t)key << 32) | (uint64_t)(uint32_t)i;
        for (int p = 0; p < passes; ++p) atomicAdd(&s_hist[p][(key >> (p * RADIX_BITS)) & (RADIX - 1)], 1u);
      }
  }
  __syncthreads();
  for (int p = 0; p < passes; ++p) {
    const uint32_t c = s_hist[p][tid];
    if (c) atomicAdd(&hdr->hist[p][tid], c);
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_radix -- one stable LSD pass on digit (key >> shift) & 255 (step a4).  Onesweep structure: the digit
// histogram over all keys comes from k_bin; each block ranks its 4096 pairs stably (warp match_any + per-warp digit
// counters in shared memory), looks back across blocks per digit, and scatters.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(RAD_THREADS) k_radix(const uint64_t* __restrict__ in, uint64_t* __restrict__ out,
                                                       Header* hdr, int pass, uint64_t* status, uint32_t tag) {
  __shared__ uint32_t s_wcnt[RAD_THREADS / 32][RADIX];
  __shared__ uint32_t s_base[RADIX];
  __shared__ uint32_t s_warp[RAD_THREADS / 32];
  __shared__ int64_t s_blk;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t P = hdr->P;
  const int64_t nblk = ((int64_t)P + RAD_TILE - 1) / RAD_TILE;
  if (tid == 0) s_blk = atomicAdd(&hdr->ticket[1 + pass], 1u);
  for (int i = tid; i < (RAD_THREADS / 32) * RADIX; i += RAD_THREADS) (&s_wcnt[0][0])[i] = 0;
  __syncthreads();
  const int64_t blk = s_blk;
  if (blk >= nblk) return;
  const int shift = pass * RADIX_BITS;
  const int64_t wbase = blk * RAD_TILE + (int64_t)warp * (RAD_CHUNKS * 32);
  const uint32_t lt = (1u << lane) - 1u;

  uint64_t item[RAD_CHUNKS];
  uint32_t rank[RAD_CHUNKS];
#pragma unroll
  for (int c = 0; c < RAD_CHUNKS; ++c) {
    const int64_t j = wbase + c * 32 + lane;
    const bool valid = j < (int64_t)P;
    item[c] = valid ? in[j] : ~0ull;
    const uint32_t d = valid ? (uint32_t)(item[c] >> (32 + shift)) & (RADIX - 1) : 0x100u;
    const uint32_t peers = __match_any_sync(0xffffffffu, d);
    uint32_t before = 0;
    if (valid) before = s_wcnt[warp][d];
    __syncwarp();
    rank[c] = before + __popc(peers & lt);
    if (valid && (__ffs(peers) - 1) == lane) s_wcnt[warp][d] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();

  // thread tid = digit d: exclusive scan over warps, block count, global digit start, look-back
  const int d = tid;
  uint32_t run = 0;
#pragma unroll
  for (int w = 0; w < RAD_THREADS / 32; ++w) { const uint32_t t = s_wcnt[w][d]; s_wcnt[w][d] = run; run += t; }
  // exclusive scan of the global histogram -> start of digit d
  const uint32_t h = hdr->hist[pass][d];
  uint32_t incl = h;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += t;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (int w = 0; w < warp; ++w) wpre += s_warp[w];
  const uint32_t gstart = wpre + incl - h;
  const uint32_t excl = lookback(status + d, blk, RADIX, tag, run);
  s_base[d] = gstart + excl;
  __syncthreads();

#pragma unroll
  for (int c = 0; c < RAD_CHUNKS; ++c) {
    const int64_t j = wbase + c * 32 + lane;
    if (j < (int64_t)P) {
      const uint32_t dd = (uint32_t)(item[c] >> (32 + shift)) & (RADIX - 1);
      out[s_base[dd] + s_wcnt[warp][dd] + rank[c]] = item[c];
    }
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_offsets -- CSR: tile_off[t] = first sorted position with key >= t (t in [0, ntiles]).
// ---------------------------------------------------------------------------------------------------------------
__global__ void k_offsets(const uint64_t* __restrict__ sorted, const Header* __restrict__ hdr, uint32_t ntiles,
                          uint32_t* __restrict__ tile_off) {
  const uint32_t P = hdr->P;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (P == 0) {
    for (int64_t t = t0; t <= ntiles; t += stride) tile_off[t] = 0;
    return;
  }
  for (int64_t p = t0; p < P; p += stride) {
    const int64_t k = (int64_t)(sorted[p] >> 32);
    const int64_t kp = p ? (int64_t)(sorted[p - 1] >> 32) : -1;
    for (int64_t t = kp + 1; t <= k; ++t) tile_off[t] = (uint32_t)p;
    if (p == (int64_t)P - 1)
      for (int64_t t = k + 1; t <= ntiles; ++t) tile_off[t] = P;
  }
}

// ---------------------------------------------------------------------------------------------------------------
void launch_bin(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                uint64_t* pairs, Header* hdr, uint64_t* status, uint32_t tag, int passes, cudaStream_t st) {
  const int64_t nblk = (n + BIN_TILE - 1) / BIN_TILE;
  if (nblk == 0) return;
  k_bin<<<(unsigned)nblk, BIN_THREADS, 0, st>>>(x, y, m, n, fp, rec, pairs, hdr, status, tag, passes);
}

void launch_radix(const uint64_t* in, uint64_t* out, Header* hdr, int pass, uint64_t* status, uint32_t tag,
                  int64_t pmax, cudaStream_t st) {
  const int64_t nblk = (pmax + RAD_TILE - 1) / RAD_TILE;
  if (nblk == 0) return;
  k_radix<<<(unsigned)nblk, RAD_THREADS, 0, st>>>(in, out, hdr, pass, status, tag);
}

void launch_offsets(const uint64_t* sorted, const Header* hdr, uint32_t ntiles, uint32_t* tile_off, int64_t pmax,
                    int num_sms, cudaStream_t st) {
  int64_t want = (std::max<int64_t>(pmax, (int64_t)ntiles + 1) + 255) / 256;
  const int64_t cap = (int64_t)num_sms * 8;
  if (want > cap) want = cap;
  if (want < 1) want = 1;
  k_offsets<<<(unsigned)want, 256, 0, st>>>(sorted, hdr, ntiles, tile_off);
}

}  // namespace starsim
