// Binning of the catalogue into image tiles (DESIGN.md §Path steps a1-a4), atomic-free:
//   k_bin      a1+a2+a3: per-star prep (validity, s' in fp64, exact ROI origin, clip, tiles overlapped), a
//              single-pass exclusive scan of the per-star tile counts over the catalogue (decoupled look-back),
//              emission of one (tile key, star index) pair per overlapped tile in star order, and the radix-digit
//              histograms of all keys.
//   k_radix    a4: one stable LSD pass of a hand-written onesweep radix sort on the tile key: per block, stable
//              ranking of 4096 pairs (warp ballots + per-warp digit counters), a decoupled look-back per digit across
//              blocks, and a scatter staged through shared memory so every digit run is written contiguously.
//   k_offsets  CSR: tile_off[t] = first sorted position with key >= t; ids[] = the sorted star indices.
// Stability of every pass keeps star-index order inside each tile, so the CSR is unique (bit-exact against the
// oracle's definition) and the per-pixel summation order in k_tile is the paper's star order.
#include <algorithm>

#include "common.cuh"
#include "launch.h"

namespace starsim {

// ---------------------------------------------------------------------------------------------------------------
// decoupled look-back (status word: flag in the high 32 bits, 1 = block aggregate, 2 = inclusive prefix; the status
// arrays are zeroed before every render)
// ---------------------------------------------------------------------------------------------------------------
__device__ __forceinline__ void st_status(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_status(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
constexpr unsigned long long ST_AGG = 1ull << 32, ST_PREFIX = 2ull << 32;

// Warp-parallel look-back by a full warp: exclusive prefix of block `blk` (status[blk*stride] holds this block's
// word).  Publishes the aggregate first, then the inclusive prefix.  Returns the exclusive prefix on every lane.
__device__ __forceinline__ uint32_t warp_lookback(unsigned long long* status, int64_t blk, int64_t stride,
                                                  uint32_t agg, int lane) {
  if (blk == 0) {
    if (lane == 0) st_status(status, ST_PREFIX | agg);
    return 0;
  }
  if (lane == 0) st_status(status + blk * stride, ST_AGG | agg);
  uint32_t excl = 0;
  int64_t b = blk - 1 - lane;  // this lane's predecessor in the current window of 32
  while (true) {
    unsigned long long w = 0;
    if (b >= 0) {
      do {
        w = ld_status(status + b * stride);
      } while ((w >> 32) == 0);
    }
    const uint32_t is_prefix = __ballot_sync(0xffffffffu, b >= 0 && (w >> 32) == 2);
    // lanes up to and including the nearest prefix contribute (lane 0 is the nearest predecessor)
    const uint32_t upto = is_prefix ? ((2u << (__ffs(is_prefix) - 1)) - 1u) : 0xffffffffu;
    uint32_t v = (((upto >> lane) & 1u) && b >= 0) ? (uint32_t)w : 0u;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    excl += v;
    if (is_prefix) break;
    b -= 32;
    if (__shfl_sync(0xffffffffu, b, 0) < 0) break;  // walked past block 0 (its word is a prefix, so not reached)
  }
  if (lane == 0) st_status(status + blk * stride, ST_PREFIX | (excl + agg));
  return excl;
}

// Clipped ROI of a star against the frame columns and the band rows; false if empty.
__device__ __forceinline__ bool clip_roi(const FrameParams& fp, int lx, int ly, int& cx0, int& cx1, int& cy0,
                                         int& cy1) {
  cx0 = max(lx, 0);
  cx1 = min(lx + fp.R - 1, fp.W - 1);
  cy0 = max(ly, fp.row0);
  cy1 = min(ly + fp.R - 1, fp.row0 + fp.rows - 1);
  return cx0 <= cx1 && cy0 <= cy1;
}

// ---------------------------------------------------------------------------------------------------------------
// k_bin -- steps a1 (prep), a2 (scan of tile counts over stars), a3 (emit pairs), digit histograms.
//   per star: reject non-finite x, y, mag (reading R11); s' = A 2.512^-m / (2 pi sigma^2) in fp64 (Eq. 1 with the
//   1/(2 pi sigma^2) of Eq. 2 folded in), rounded once to fp32; exact ROI origin (reading R7); clip to the image
//   columns and the band rows; the tiles the clipped ROI overlaps.
// Layout: BIN_THREADS threads x BIN_ITEMS stars, striped loads (coalesced), blocked scan through shared memory.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(BIN_THREADS) k_bin(const float* __restrict__ X, const float* __restrict__ Y,
                                                     const float* __restrict__ M, int64_t n, FrameParams fp,
                                                     StarRec* __restrict__ rec, uint64_t* __restrict__ pairs,
                                                     Header* hdr, unsigned long long* status, int bits0, int bits1) {
  __shared__ uint32_t s_cnt[BIN_TILE];
  __shared__ uint32_t s_h0[MAX_RADIX], s_h1[MAX_RADIX];
  __shared__ uint32_t s_warp[BIN_THREADS / 32];
  __shared__ uint32_t s_base;
  __shared__ int64_t s_blk;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nb0 = 1 << bits0, nb1 = 1 << bits1;
  if (tid == 0) s_blk = atomicAdd(&hdr->ticket[0], 1u);
  for (int i = tid; i < MAX_RADIX; i += BIN_THREADS) s_h0[i] = s_h1[i] = 0;
  __syncthreads();
  const int64_t blk = s_blk;
  const int64_t base = blk * BIN_TILE;

  // ---- a1: per-star prep (striped: star base + k*BIN_THREADS + tid)
  uint32_t cnts[BIN_ITEMS];
  uint32_t trx[BIN_ITEMS], try_[BIN_ITEMS];  // tx0 | tx1 << 16, ty0 | ty1 << 16
#pragma unroll
  for (int k = 0; k < BIN_ITEMS; ++k) {
    const int64_t i = base + k * BIN_THREADS + tid;
    uint32_t cnt = 0;
    trx[k] = try_[k] = 0;
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
        if (clip_roi(fp, lx, ly, cx0, cx1, cy0, cy1)) {
          r.lo = ((uint32_t)(uint16_t)(int16_t)lx) | ((uint32_t)(uint16_t)(int16_t)ly << 16);
          r.s = (float)(fp.s_scale * exp2(-(double)m * 1.3288364642295399628));  // 2.512^-m, Eq. 1
          const uint32_t tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
          const uint32_t ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
          trx[k] = tx0 | (tx1 << 16);
          try_[k] = ty0 | (ty1 << 16);
          cnt = (tx1 - tx0 + 1) * (ty1 - ty0 + 1);
        }
      }
      rec[i] = r;
    }
    cnts[k] = cnt;
    s_cnt[k * BIN_THREADS + tid] = cnt;
  }
  __syncthreads();

  // ---- a2: block-wide exclusive scan in star order (thread t owns stars t*BIN_ITEMS ... of the block)
  uint32_t v[BIN_ITEMS], tsum = 0;
#pragma unroll
  for (int j = 0; j < BIN_ITEMS; ++j) {
    v[j] = s_cnt[tid * BIN_ITEMS + j];
    tsum += v[j];
  }
  uint32_t incl = tsum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += t;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const uint32_t w = lane < BIN_THREADS / 32 ? s_warp[lane] : 0u;
    uint32_t wi = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, wi, o);
      if (lane >= o) wi += t;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, wi, 31);
    if (lane < BIN_THREADS / 32) s_warp[lane] = wi - w;
    const uint32_t excl = warp_lookback(status, blk, 1, total, lane);
    if (lane == 0) {
      s_base = excl;
      const int64_t nblk = (n + BIN_TILE - 1) / BIN_TILE;
      if (blk == nblk - 1) hdr->P = excl + total;
    }
  }
  __syncthreads();
  {
    uint32_t off = s_base + s_warp[warp] + incl - tsum;
#pragma unroll
    for (int j = 0; j < BIN_ITEMS; ++j) {
      s_cnt[tid * BIN_ITEMS + j] = off;
      off += v[j];
    }
  }
  __syncthreads();

  // ---- a3: emit pairs in star order, tiles row-major; histogram the digits of every key
  const uint32_t m0 = (uint32_t)nb0 - 1u, m1 = (uint32_t)nb1 - 1u;
#pragma unroll
  for (int k = 0; k < BIN_ITEMS; ++k) {
    if (cnts[k] == 0) continue;
    const int64_t i = base + k * BIN_THREADS + tid;
    uint32_t o = s_cnt[k * BIN_THREADS + tid];
    for (uint32_t ty = try_[k] & 0xFFFFu; ty <= (try_[k] >> 16); ++ty)
      for (uint32_t tx = trx[k] & 0xFFFFu; tx <= (trx[k] >> 16); ++tx) {
        const uint32_t key = ty * (uint32_t)fp.ntx + tx;
        pairs[o++] = ((uint64_t)key << 32) | (uint64_t)(uint32_t)i;
        atomicAdd(&s_h0[key & m0], 1u);
        if (bits1) atomicAdd(&s_h1[(key >> bits0) & m1], 1u);
      }
  }
  __syncthreads();
  for (int d = tid; d < nb0; d += BIN_THREADS)
    if (s_h0[d]) atomicAdd(&hdr->hist[0][d], s_h0[d]);
  if (bits1)
    for (int d = tid; d < nb1; d += BIN_THREADS)
      if (s_h1[d]) atomicAdd(&hdr->hist[1][d], s_h1[d]);
}

// ---------------------------------------------------------------------------------------------------------------
// k_radix -- one stable LSD pass on digit (key >> shift) & (2^BITS - 1).
// ---------------------------------------------------------------------------------------------------------------
template <int BITS>
__global__ void __launch_bounds__(RAD_THREADS) k_radix(const uint64_t* __restrict__ in, uint64_t* __restrict__ out,
                                                       Header* hdr, int pass, int shift,
                                                       unsigned long long* status) {
  constexpr int NB = 1 << BITS;
  constexpr int NW = RAD_THREADS / 32;
  constexpr int PER = (NB + RAD_THREADS - 1) / RAD_THREADS;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  uint64_t* s_items = reinterpret_cast<uint64_t*>(smem_raw);          // RAD_TILE pairs in block digit order
  uint32_t* s_wcnt = reinterpret_cast<uint32_t*>(s_items + RAD_TILE);  // NW x NB per-warp digit counters
  uint32_t* s_lstart = s_wcnt + NW * NB;                               // NB: block-local digit start
  uint32_t* s_goff = s_lstart + NB;                                    // NB: global position of the digit run
  __shared__ uint32_t s_warp[NW];
  __shared__ int64_t s_blk;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t P = hdr->P;
  const int64_t nblk = ((int64_t)P + RAD_TILE - 1) / RAD_TILE;
  if (tid == 0) s_blk = atomicAdd(&hdr->ticket[1 + pass], 1u);
  for (int i = tid; i < NW * NB; i += RAD_THREADS) s_wcnt[i] = 0;
  __syncthreads();
  const int64_t blk = s_blk;
  if (blk >= nblk) return;
  const int64_t wbase = blk * RAD_TILE + (int64_t)warp * (RAD_CHUNKS * 32);
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t* wc = s_wcnt + warp * NB;

  // ---- stable rank within the warp's 32*RAD_CHUNKS pairs (chunks in order, lanes in order)
  uint64_t item[RAD_CHUNKS];
  uint32_t rank[RAD_CHUNKS];
#pragma unroll
  for (int c = 0; c < RAD_CHUNKS; ++c) {
    const int64_t j = wbase + c * 32 + lane;
    item[c] = j < (int64_t)P ? in[j] : 0ull;
  }
#pragma unroll
  for (int c = 0; c < RAD_CHUNKS; ++c) {
    const int64_t j = wbase + c * 32 + lane;
    const bool valid = j < (int64_t)P;
    const uint32_t d = (uint32_t)(item[c] >> (32 + shift)) & (NB - 1);
    uint32_t peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < BITS; ++b) {
      const uint32_t vb = __ballot_sync(0xffffffffu, (d >> b) & 1u);
      peers &= ((d >> b) & 1u) ? vb : ~vb;
    }
    const uint32_t before = valid ? wc[d] : 0u;
    __syncwarp();
    rank[c] = before + __popc(peers & lt);
    if (valid && (__ffs(peers) - 1) == lane) wc[d] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();

  // ---- per digit: offsets of the warps inside the block and the block count
  for (int d = tid; d < NB; d += RAD_THREADS) {
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
      const uint32_t t = s_wcnt[w * NB + d];
      s_wcnt[w * NB + d] = run;
      run += t;
    }
    s_goff[d] = run;  // block count, temporarily
  }
  __syncthreads();
  // ---- block-local digit starts (exclusive scan of the block counts) and global digit starts
  uint32_t bcnt[PER], gh[PER];
  {
    uint32_t sum = 0, gsum = 0;
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      const int d = tid * PER + e;
      bcnt[e] = d < NB ? s_goff[d] : 0u;
      gh[e] = d < NB ? hdr->hist[pass][d] : 0u;
      sum += bcnt[e];
      gsum += gh[e];
    }
    // two block-wide exclusive scans (block counts, global histogram) with one pair of barriers
    uint32_t incl = sum, gincl = gsum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      const uint32_t g = __shfl_up_sync(0xffffffffu, gincl, o);
      if (lane >= o) {
        incl += t;
        gincl += g;
      }
    }
    __shared__ uint32_t s_gwarp[NW];
    if (lane == 31) {
      s_warp[warp] = incl;
      s_gwarp[warp] = gincl;
    }
    __syncthreads();
    uint32_t wpre = 0, gpre = 0;
    for (int w = 0; w < warp; ++w) {
      wpre += s_warp[w];
      gpre += s_gwarp[w];
    }
    uint32_t off = wpre + incl - sum, goff = gpre + gincl - gsum;
#pragma unroll
    for (int e = 0; e < PER; ++e) {
      const int d = tid * PER + e;
      if (d < NB) {
        s_lstart[d] = off;
        // per-digit decoupled look-back across blocks (the predecessors publish their aggregates early)
        const uint32_t bc = bcnt[e];
        uint32_t excl = 0;
        unsigned long long* st = status + d;
        if (blk == 0) {
          st_status(st, ST_PREFIX | bc);
        } else {
          st_status(st + blk * NB, ST_AGG | bc);
          for (int64_t b = blk - 1; b >= 0; --b) {
            unsigned long long w;
            do {
              w = ld_status(st + b * NB);
            } while ((w >> 32) == 0);
            excl += (uint32_t)w;
            if ((w >> 32) == 2) break;
          }
          st_status(st + blk * NB, ST_PREFIX | (excl + bc));
        }
        s_goff[d] = goff + excl;
      }
      off += bcnt[e];
      goff += gh[e];
    }
  }
  __syncthreads();

  // ---- stage the block's pairs in digit order in shared memory, then write each digit run contiguously
#pragma unroll
  for (int c = 0; c < RAD_CHUNKS; ++c) {
    const int64_t j = wbase + c * 32 + lane;
    if (j < (int64_t)P) {
      const uint32_t d = (uint32_t)(item[c] >> (32 + shift)) & (NB - 1);
      s_items[s_lstart[d] + s_wcnt[warp * NB + d] + rank[c]] = item[c];
    }
  }
  __syncthreads();
  const int cntb = (int)min((int64_t)RAD_TILE, (int64_t)P - blk * RAD_TILE);
  for (int i = tid; i < cntb; i += RAD_THREADS) {
    const uint64_t it = s_items[i];
    const uint32_t d = (uint32_t)(it >> (32 + shift)) & (NB - 1);
    out[s_goff[d] + (uint32_t)i - s_lstart[d]] = it;
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_offsets -- CSR: tile_off[t] = first sorted position with key >= t (t in [0, ntiles]); ids[p] = star index of
// sorted pair p.
// ---------------------------------------------------------------------------------------------------------------
__global__ void k_offsets(const uint64_t* __restrict__ sorted, const Header* __restrict__ hdr, uint32_t ntiles,
                          uint32_t* __restrict__ tile_off, uint32_t* __restrict__ ids) {
  const uint32_t P = hdr->P;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (P == 0) {
    for (int64_t t = t0; t <= ntiles; t += stride) tile_off[t] = 0;
    return;
  }
  for (int64_t p = t0; p < P; p += stride) {
    const uint64_t it = sorted[p];
    ids[p] = (uint32_t)it;
    const int64_t k = (int64_t)(it >> 32);
    const int64_t kp = p ? (int64_t)(sorted[p - 1] >> 32) : -1;
    for (int64_t t = kp + 1; t <= k; ++t) tile_off[t] = (uint32_t)p;
    if (p == (int64_t)P - 1)
      for (int64_t t = k + 1; t <= ntiles; ++t) tile_off[t] = P;
  }
}

// ---------------------------------------------------------------------------------------------------------------
void launch_bin(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                uint64_t* pairs, Header* hdr, unsigned long long* status, int bits0, int bits1, cudaStream_t st) {
  const int64_t nblk = (n + BIN_TILE - 1) / BIN_TILE;
  if (nblk == 0) return;
  k_bin<<<(unsigned)nblk, BIN_THREADS, 0, st>>>(x, y, m, n, fp, rec, pairs, hdr, status, bits0, bits1);
}

template <int BITS>
static size_t radix_smem() {
  return sizeof(uint64_t) * RAD_TILE + sizeof(uint32_t) * ((RAD_THREADS / 32) * (1 << BITS) + 2 * (1 << BITS));
}

template <int BITS>
static void launch_radix_t(const uint64_t* in, uint64_t* out, Header* hdr, int pass, int shift,
                           unsigned long long* status, int64_t nblk, cudaStream_t st) {
  k_radix<BITS><<<(unsigned)nblk, RAD_THREADS, radix_smem<BITS>(), st>>>(in, out, hdr, pass, shift, status);
}

template <int BITS>
static void set_radix_smem() {
  cudaFuncSetAttribute(k_radix<BITS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)radix_smem<BITS>());
  if constexpr (BITS < MAX_RADIX_BITS) set_radix_smem<BITS + 1>();
}

// Per-process kernel attributes (dynamic shared memory above 48 KB); called by starsim_create.
void init_kernels() { set_radix_smem<1>(); }

void launch_radix(const uint64_t* in, uint64_t* out, Header* hdr, int pass, int shift, int bits,
                  unsigned long long* status, int64_t pmax, cudaStream_t st) {
  const int64_t nblk = (pmax + RAD_TILE - 1) / RAD_TILE;
  if (nblk == 0) return;
  switch (bits) {
    case 1: launch_radix_t<1>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 2: launch_radix_t<2>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 3: launch_radix_t<3>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 4: launch_radix_t<4>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 5: launch_radix_t<5>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 6: launch_radix_t<6>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 7: launch_radix_t<7>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 8: launch_radix_t<8>(in, out, hdr, pass, shift, status, nblk, st); break;
    case 9: launch_radix_t<9>(in, out, hdr, pass, shift, status, nblk, st); break;
    default: launch_radix_t<10>(in, out, hdr, pass, shift, status, nblk, st); break;
  }
}

void launch_offsets(const uint64_t* sorted, const Header* hdr, uint32_t ntiles, uint32_t* tile_off, uint32_t* ids,
                    int64_t pmax, int num_sms, cudaStream_t st) {
  int64_t want = (std::max<int64_t>(pmax, (int64_t)ntiles + 1) + 255) / 256;
  const int64_t cap = (int64_t)num_sms * 8;
  if (want > cap) want = cap;
  if (want < 1) want = 1;
  k_offsets<<<(unsigned)want, 256, 0, st>>>(sorted, hdr, ntiles, tile_off, ids);
}

}  // namespace starsim
