// Binning of the catalogue into image tiles (DESIGN.md §Path steps a1-a4).
//   k_prep       a1: per star -- validity, s' in fp64, exact ROI origin, clip to the frame columns and band rows; the
//                tiles its clipped ROI overlaps (row-major), and for each one a slot in that tile's list from an
//                atomic counter (one ATOMG per (tile, star) pair).  Writes the 16-B star record.
//   k_scan_a/b   a2: exclusive scan of the per-tile counts -> tile_off[ntiles+1], P; and k_tile's work list
//                (heavy tiles split into parts).
//   k_scatter    a3: ids[tile_off[tile] + slot] = star for every pair.
//   k_sortlists  a4: sort every tile's list ascending (LSD radix on the star index in shared memory, 8-bit digits,
//                stable warp-ballot ranking); lists longer than SORT_CAP are sorted in SORT_CAP chunks through a
//                global ping-pong buffer.
// The atomics fix only which slot a star takes; the per-tile sort makes the CSR unique -- star-index order inside
// each tile, bit-exact against the oracle's definition -- so k_tile's per-pixel summation order is deterministic.
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "plan.cuh"
#include "prep.cuh"

namespace starsim {

// ---------------------------------------------------------------------------------------------------------------
// k_prep -- step a1.  Per star: reject non-finite x, y, mag (reading R11); s' = A 2.512^-m / (2 pi sigma^2) in fp64
// (Eq. 1 with the 1/(2 pi sigma^2) of Eq. 2 folded in), rounded once to fp32; exact ROI origin (reading R7); clip;
// one slot per overlapped tile.  slots[i*tps + k] is the slot in the k-th overlapped tile (row-major).
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(PREP_THREADS) k_prep(const float* __restrict__ X, const float* __restrict__ Y,
                                                       const float* __restrict__ M, int64_t n, FrameParams fp,
                                                       StarRec* __restrict__ rec, uint32_t* __restrict__ cnt,
                                                       uint32_t* __restrict__ slots, int tps) {
  const int64_t i = (int64_t)blockIdx.x * PREP_THREADS + threadIdx.x;
  if (i >= frame_n(n, fp)) return;
  int cx0, cx1, cy0, cy1;
  const StarRec r = prep_star(X[i], Y[i], M[i], fp, cx0, cx1, cy0, cy1);
  if (r.lo != LO_CULLED) {
    const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
    const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
    uint32_t* sl = slots + i * tps;
    int k = 0;
    for (int ty = ty0; ty <= ty1; ++ty)
      for (int tx = tx0; tx <= tx1; ++tx) sl[k++] = atomicAdd(&cnt[(int64_t)(ty * fp.ntx + tx) * CNT_STRIDE], 1u);
  }
  rec[i] = r;
}

// ---------------------------------------------------------------------------------------------------------------
// k_scan -- step a2 and k_tile's work list, one CTA of 1024 threads, each a contiguous run of tiles:
//   tile_off[t] = sum of cnt[0..t), tile_off[ntiles] = P;
//   a tile whose list is longer than SPLIT_LEN becomes ceil(len / SPLIT_LEN) work items over consecutive star ranges
//   (its parts), every other tile one item; parts come first (the heavy work starts first).  The split depends only
//   on the tile's own list, so it is the same for any band decomposition.  If the parts would need more than
//   `part_cap` partial buffers, nothing is split.
// ---------------------------------------------------------------------------------------------------------------
// Two kernels, SCAN_TILES tiles per CTA (SCAN_PER per thread): k_scan_a writes each CTA's sums (pairs, parts, split
// tiles); k_scan_b re-reduces the sums of the CTAs before it and of all CTAs (a few hundred at most), scans its own
// tiles and writes tile_off and the work items.
// block-wide exclusive scan of uint4 (SCAN_THREADS threads); *total receives the block sum
__device__ __forceinline__ uint4 block_excl_scan4(uint4 v, uint4* s_w, uint4* total) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint4 incl = warp_incl_scan4(v, lane);
  if (lane == 31) s_w[warp] = incl;
  __syncthreads();
  uint4 pre = make_uint4(0, 0, 0, 0), tot = make_uint4(0, 0, 0, 0);
#pragma unroll
  for (int w = 0; w < SCAN_THREADS / 32; ++w) {
    const uint4 u = s_w[w];
    if (w < warp) pre = add4(pre, u);
    tot = add4(tot, u);
  }
  __syncthreads();
  *total = tot;
  return sub4(add4(pre, incl), v);
}

__device__ __forceinline__ void load_counts(const uint32_t* cnt, int64_t ntiles, int64_t t0, uint32_t* c, uint4& sum,
                                            uint32_t split) {
  sum = make_uint4(0, 0, 0, 0);
#pragma unroll
  for (int k = 0; k < SCAN_PER; ++k) c[k] = t0 + k < ntiles ? __ldcg(&cnt[(t0 + k) * CNT_STRIDE]) : 0u;
#pragma unroll
  for (int k = 0; k < SCAN_PER; ++k) sum = add4(sum, t0 + k < ntiles ? tile_counts(c[k], split) : make_uint4(0, 0, 0, 0));
}

__global__ void __launch_bounds__(SCAN_THREADS) k_scan_a(const uint32_t* __restrict__ cnt, int64_t ntiles,
                                                         uint4* __restrict__ partial, int plan) {
  __shared__ uint4 s_w[SCAN_THREADS / 32];
  const int64_t t0 = (int64_t)blockIdx.x * SCAN_TILES + (int64_t)threadIdx.x * SCAN_PER;
  uint32_t c[SCAN_PER];
  uint4 sum, tot;
  load_counts(cnt, ntiles, t0, c, sum, plan_split(plan));
  block_excl_scan4(sum, s_w, &tot);
  if (threadIdx.x == 0) partial[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(SCAN_THREADS) k_scan_b(const uint32_t* __restrict__ cnt, int64_t ntiles,
                                                         const uint4* __restrict__ partial, int nblk,
                                                         uint32_t* __restrict__ tile_off, Header* hdr,
                                                         WorkItem* __restrict__ items,
                                                         uint2* __restrict__ split_tab, int plan,
                                                         uint32_t* __restrict__ done) {
  __shared__ uint4 s_w[SCAN_THREADS / 32];
  const int tid = threadIdx.x;
  const int part_cap = plan_cap(plan);
  const uint32_t split = plan_split(plan);
  // sums of the CTAs before this one, and of all CTAs
  uint4 before = make_uint4(0, 0, 0, 0), all = make_uint4(0, 0, 0, 0);
  for (int k = tid; k < nblk; k += SCAN_THREADS) {
    const uint4 u = partial[k];
    if (k < (int)blockIdx.x) before = add4(before, u);
    all = add4(all, u);
  }
  uint4 tb, ta;
  block_excl_scan4(before, s_w, &tb);
  block_excl_scan4(all, s_w, &ta);
  const bool split_on = ta.y <= (uint32_t)part_cap;
  const uint32_t nparts = split_on ? ta.y : 0u, nsplit = split_on ? ta.z : 0u;
  const uint32_t lite0 = nparts + (uint32_t)ntiles - nsplit - ta.w;
  if (blockIdx.x == 0 && tid == 0) plan_header(hdr, tile_off, ntiles, ta, part_cap);
  const int64_t t0 = (int64_t)blockIdx.x * SCAN_TILES + (int64_t)tid * SCAN_PER;
  uint32_t c[SCAN_PER];
  uint4 sum, tot;
  load_counts(cnt, ntiles, t0, c, sum, split);
  const uint4 ex = add4(tb, block_excl_scan4(sum, s_w, &tot));
  uint32_t run = ex.x, pb = ex.y, si = ex.z, li = ex.w;
#pragma unroll
  for (int k = 0; k < SCAN_PER; ++k) {
    const int64_t t = t0 + k;
    if (t >= ntiles) break;
    plan_tile((uint32_t)t, c[k], run, pb, si, li, nparts, lite0, split_on, tile_off, items, split_tab, done, split);
  }
}

// k_scan_one: the same as k_scan_a + k_scan_b in a single CTA of SCAN1_THREADS threads (SCAN_PER tiles each), for
// frames / bands of at most SCAN1_TILES tiles: one launch instead of two.
constexpr int SCAN1_THREADS = 1024;
constexpr int SCAN1_TILES = SCAN1_THREADS * SCAN_PER;

__global__ void __launch_bounds__(SCAN1_THREADS) k_scan_one(const uint32_t* __restrict__ cnt, int64_t ntiles,
                                                             uint32_t* __restrict__ tile_off, Header* hdr,
                                                             WorkItem* __restrict__ items,
                                                             uint2* __restrict__ split_tab, int plan,
                                                             uint32_t* __restrict__ done) {
  const int part_cap = plan_cap(plan);
  const uint32_t split = plan_split(plan);
  __shared__ uint4 s_w[SCAN1_THREADS / 32];
  __shared__ uint4 s_tot;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t t0 = (int64_t)tid * SCAN_PER;
  uint32_t c[SCAN_PER];
  uint4 sum;
  load_counts(cnt, ntiles, t0, c, sum, split);
  const uint4 incl = warp_incl_scan4(sum, lane);
  if (lane == 31) s_w[warp] = incl;
  __syncthreads();
  if (warp == 0) {  // exclusive scan of the warp sums in place; the total
    const uint4 v = s_w[lane];
    const uint4 wi = warp_incl_scan4(v, lane);
    __syncwarp();
    s_w[lane] = sub4(wi, v);
    if (lane == 31) s_tot = wi;
  }
  __syncthreads();
  const uint4 pre = s_w[warp], ta = s_tot;
  const bool split_on = ta.y <= (uint32_t)part_cap;
  const uint32_t nparts = split_on ? ta.y : 0u, nsplit = split_on ? ta.z : 0u;
  const uint32_t lite0 = nparts + (uint32_t)ntiles - nsplit - ta.w;
  if (tid == 0) plan_header(hdr, tile_off, ntiles, ta, part_cap);
  const uint4 ex = sub4(add4(pre, incl), sum);
  uint32_t run = ex.x, pb = ex.y, si = ex.z, li = ex.w;
#pragma unroll
  for (int k = 0; k < SCAN_PER; ++k) {
    const int64_t t = t0 + k;
    if (t >= ntiles) break;
    plan_tile((uint32_t)t, c[k], run, pb, si, li, nparts, lite0, split_on, tile_off, items, split_tab, done, split);
  }
}

// ---------------------------------------------------------------------------------------------------------------
// k_scatter -- step a3: every (tile, star) pair to its slot.
// ---------------------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(PREP_THREADS) k_scatter(const StarRec* __restrict__ rec, int64_t n, FrameParams fp,
                                                          const uint32_t* __restrict__ slots, int tps,
                                                          const uint32_t* __restrict__ tile_off,
                                                          uint32_t* __restrict__ ids) {
  const int64_t i = (int64_t)blockIdx.x * PREP_THREADS + threadIdx.x;
  if (i >= frame_n(n, fp)) return;
  const uint32_t lo = rec[i].lo;
  if (lo == LO_CULLED) return;
  int cx0, cx1, cy0, cy1;
  clip_roi(fp, lo_x_of(lo), lo_y_of(lo), cx0, cx1, cy0, cy1);
  const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
  const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
  const uint32_t* sl = slots + i * tps;
  int k = 0;
  for (int ty = ty0; ty <= ty1; ++ty)
    for (int tx = tx0; tx <= tx1; ++tx) {
      const int t = ty * fp.ntx + tx;
      ids[tile_off[t] + sl[k++]] = (uint32_t)i;
    }
}

// ---------------------------------------------------------------------------------------------------------------
// k_sortlists -- step a4.  One CTA per tile.  One LSD pass over digit (v >> shift) & 255 of `len` values in `in`
// (shared memory) -> `out` (shared or global, at out[dbase[d] + rank]): each warp ranks its contiguous slice of
// SORT_CHUNKS x 32 values stably (ballots over the digit bits, per-warp digit counters), then digits are laid out
// warp-major inside each digit.  `gbase` (optional) offsets every digit run; `dcount` returns the per-digit counts.
// ---------------------------------------------------------------------------------------------------------------
struct SortSmem {
  uint32_t wcnt[SORT_THREADS / 32][SORT_RADIX];
  uint32_t dstart[SORT_RADIX];
  uint32_t wsum[SORT_THREADS / 32];
};

__device__ void sort_pass(const uint32_t* in, int len, int shift, uint32_t* out, const uint32_t* gbase,
                          uint32_t* dcount, SortSmem& sm) {
  constexpr int NW = SORT_THREADS / 32;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  for (int i = tid; i < NW * SORT_RADIX; i += SORT_THREADS) (&sm.wcnt[0][0])[i] = 0;
  __syncthreads();
  // warp slice: [w0, w1), processed in 32-value chunks in order
  const int per = ((len + NW - 1) / NW + 31) & ~31;
  const int w0 = min(warp * per, len), w1 = min(w0 + per, len);
  uint32_t* wc = sm.wcnt[warp];
  uint32_t rank[SORT_CHUNKS];
#pragma unroll
  for (int c = 0; c < SORT_CHUNKS; ++c) {
    const int j = w0 + c * 32 + lane;
    rank[c] = 0;
    if (w0 + c * 32 >= w1) continue;  // warp-uniform
    const bool valid = j < w1;
    const uint32_t d = valid ? (in[j] >> shift) & (SORT_RADIX - 1) : 0u;
    uint32_t peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
    for (int b = 0; b < SORT_BITS; ++b) {
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
  // per digit: warp offsets inside the digit run, digit totals; then the exclusive scan over digits (DPT contiguous
  // digits per thread)
  constexpr int DPT = SORT_RADIX / SORT_THREADS;
  uint32_t dtot[DPT], tot = 0;
#pragma unroll
  for (int k = 0; k < DPT; ++k) {
    const int d = tid * DPT + k;
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
      const uint32_t t = sm.wcnt[w][d];
      sm.wcnt[w][d] = run;
      run += t;
    }
    if (dcount) dcount[d] = run;
    dtot[k] = run;
    tot += run;
  }
  uint32_t incl = tot;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  if (lane == 31) sm.wsum[warp] = incl;
  __syncthreads();
  {
    uint32_t pre = incl - tot;
    for (int w = 0; w < warp; ++w) pre += sm.wsum[w];
#pragma unroll
    for (int k = 0; k < DPT; ++k) {
      const int d = tid * DPT + k;
      sm.dstart[d] = pre + (gbase ? gbase[d] : 0u);
      pre += dtot[k];
    }
  }
  __syncthreads();
#pragma unroll
  for (int c = 0; c < SORT_CHUNKS; ++c) {
    const int j = w0 + c * 32 + lane;
    if (j < w1) {
      const uint32_t v = in[j];
      const uint32_t d = (v >> shift) & (SORT_RADIX - 1);
      out[sm.dstart[d] + sm.wcnt[warp][d] + rank[c]] = v;
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(SORT_THREADS) k_sortlists(uint32_t* __restrict__ ids,
                                                            uint32_t* __restrict__ tmp,
                                                            const uint32_t* __restrict__ tile_off, int passes) {
  __shared__ __align__(16) uint32_t s_a[SORT_CAP];
  __shared__ __align__(16) uint32_t s_b[SORT_CAP];
  __shared__ SortSmem sm;
  __shared__ uint32_t s_gbase[SORT_RADIX], s_cnt[SORT_RADIX];
  __shared__ uint32_t s_bcnt[SORT_NB];
  __shared__ uint32_t s_red[2][SORT_THREADS / 32];
  __shared__ int s_fallback;
  const int64_t t = blockIdx.x;
  const uint32_t j0 = tile_off[t], j1 = tile_off[t + 1];
  const int len = (int)(j1 - j0);
  if (len <= 1) return;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t* g = ids + j0;
  if (len <= SORT_CAP) {
    // bucket sort on the id range: bucket = (v - min) >> sh with at most SORT_NB buckets; the atomics only decide
    // the order inside a bucket, which the per-bucket insertion sort then fixes.  Buckets hold ~len/SORT_NB ids for
    // any list whose ids spread over their range; a skewed list (a bucket > 32) falls back to the LSD radix sort.
    uint32_t mn = 0xffffffffu, mx = 0u;
    for (int i = tid; i < len; i += SORT_THREADS) {
      const uint32_t v = g[i];
      s_a[i] = v;
      mn = min(mn, v);
      mx = max(mx, v);
    }
    for (int i = tid; i < SORT_NB; i += SORT_THREADS) s_bcnt[i] = 0;
    mn = __reduce_min_sync(0xffffffffu, mn);
    mx = __reduce_max_sync(0xffffffffu, mx);
    if (lane == 0) {
      s_red[0][warp] = mn;
      s_red[1][warp] = mx;
    }
    if (tid == 0) s_fallback = 0;
    __syncthreads();
    mn = s_red[0][0];
    mx = s_red[1][0];
#pragma unroll
    for (int w = 1; w < SORT_THREADS / 32; ++w) {
      mn = min(mn, s_red[0][w]);
      mx = max(mx, s_red[1][w]);
    }
    int sh = 0;
    while (((mx - mn) >> sh) >= (uint32_t)SORT_NB) ++sh;
    // histogram; the slot an atomic returns is kept in s_r (aliases the radix counters, unused on this path)
    uint16_t* s_r = reinterpret_cast<uint16_t*>(&sm.wcnt[0][0]);
    static_assert(sizeof(sm.wcnt) >= SORT_CAP * sizeof(uint16_t), "s_r alias");
    for (int i = tid; i < len; i += SORT_THREADS) s_r[i] = (uint16_t)atomicAdd(&s_bcnt[(s_a[i] - mn) >> sh], 1u);
    __syncthreads();
    // exclusive scan of the bucket counts (SORT_NB / SORT_THREADS per thread, contiguous)
    constexpr int PB = SORT_NB / SORT_THREADS;
    uint32_t c[PB], sum = 0;
#pragma unroll
    for (int k = 0; k < PB; ++k) {
      c[k] = s_bcnt[tid * PB + k];
      sum += c[k];
    }
    uint32_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    if (lane == 31) sm.wsum[warp] = incl;
    __syncthreads();
    uint32_t run = incl - sum;
    for (int w = 0; w < warp; ++w) run += sm.wsum[w];
    uint32_t start[PB];
    bool skew = false;
#pragma unroll
    for (int k = 0; k < PB; ++k) {
      start[k] = run;
      s_bcnt[tid * PB + k] = run;  // bucket start
      run += c[k];
      skew |= c[k] > 32;
    }
    if (skew) s_fallback = 1;
    __syncthreads();
    if (!s_fallback) {
      for (int i = tid; i < len; i += SORT_THREADS) {
        const uint32_t v = s_a[i];
        s_b[s_bcnt[(v - mn) >> sh] + s_r[i]] = v;
      }
      __syncthreads();
      // insertion sort inside every bucket
#pragma unroll
      for (int k = 0; k < PB; ++k) {
        uint32_t* a = s_b + start[k];
        const int n = (int)c[k];
        for (int x = 1; x < n; ++x) {
          const uint32_t v = a[x];
          int y = x - 1;
          while (y >= 0 && a[y] > v) {
            a[y + 1] = a[y];
            --y;
          }
          a[y + 1] = v;
        }
      }
      __syncthreads();
      for (int i = tid; i < len; i += SORT_THREADS) g[i] = s_b[i];
      return;
    }
    // skewed list: LSD radix sort in shared memory (s_a still holds the list)
    uint32_t *src = s_a, *dst2 = s_b;
    for (int p = 0; p < passes; ++p) {
      sort_pass(src, len, p * SORT_BITS, dst2, nullptr, nullptr, sm);
      uint32_t* sw = src;
      src = dst2;
      dst2 = sw;
    }
    for (int i = tid; i < len; i += SORT_THREADS) g[i] = src[i];
    return;
  }
  // long list: each pass streams SORT_CAP chunks in order; digit runs are placed with running global bases
  uint32_t *src = g, *dst = tmp + j0;
  for (int p = 0; p < passes; ++p) {
    const int shift = p * SORT_BITS;
    for (int i = tid; i < SORT_RADIX; i += SORT_THREADS) s_cnt[i] = 0;
    __syncthreads();
    for (int i = tid; i < len; i += SORT_THREADS) atomicAdd(&s_cnt[(src[i] >> shift) & (SORT_RADIX - 1)], 1u);
    __syncthreads();
    if (tid == 0) {
      uint32_t run = 0;
      for (int d = 0; d < SORT_RADIX; ++d) {
        s_gbase[d] = run;
        run += s_cnt[d];
      }
    }
    __syncthreads();
    // dstart of sort_pass is relative to the chunk; out[] must be the run base + position inside the digit run
    for (int c0 = 0; c0 < len; c0 += SORT_CAP) {
      const int cl = min(SORT_CAP, len - c0);
      for (int i = tid; i < cl; i += SORT_THREADS) s_a[i] = src[c0 + i];
      __syncthreads();
      sort_pass(s_a, cl, shift, s_b, nullptr, s_cnt, sm);  // chunk sorted into s_b, per-digit counts in s_cnt
      // s_b holds the chunk grouped by digit; copy every digit run to dst at the running base
      for (int i = tid; i < cl; i += SORT_THREADS) {
        const uint32_t v = s_b[i];
        const uint32_t d = (v >> shift) & (SORT_RADIX - 1);
        dst[s_gbase[d] + (uint32_t)i - sm.dstart[d]] = v;
      }
      __syncthreads();
      for (int d = tid; d < SORT_RADIX; d += SORT_THREADS) s_gbase[d] += s_cnt[d];
      __syncthreads();
    }
    uint32_t* sw = src;
    src = dst;
    dst = sw;
  }
  if (src != g) {
    for (int i = tid; i < len; i += SORT_THREADS) g[i] = src[i];
  }
}

// ---------------------------------------------------------------------------------------------------------------
void launch_prep(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                 uint32_t* cnt, uint32_t* slots, int tps, cudaStream_t st) {
  if (n <= 0) return;
  k_prep<<<(unsigned)((n + PREP_THREADS - 1) / PREP_THREADS), PREP_THREADS, 0, st>>>(x, y, m, n, fp, rec, cnt, slots,
                                                                                     tps);
}

int scan_launches(int64_t ntiles) { return ntiles <= SCAN1_TILES ? 1 : 2; }

void launch_scan(const uint32_t* cnt, int64_t ntiles, uint32_t* tile_off, Header* hdr, WorkItem* items,
                 uint2* split_tab, int plan, void* partial, uint32_t* done, cudaStream_t st) {
  if (ntiles <= SCAN1_TILES) {
    k_scan_one<<<1, SCAN1_THREADS, 0, st>>>(cnt, ntiles, tile_off, hdr, items, split_tab, plan, done);
    return;
  }
  const int nblk = (int)((ntiles + SCAN_TILES - 1) / SCAN_TILES);
  k_scan_a<<<nblk, SCAN_THREADS, 0, st>>>(cnt, ntiles, (uint4*)partial, plan);
  k_scan_b<<<nblk, SCAN_THREADS, 0, st>>>(cnt, ntiles, (const uint4*)partial, nblk, tile_off, hdr, items, split_tab,
                                         plan, done);
}

void launch_scatter(const StarRec* rec, int64_t n, const FrameParams& fp, const uint32_t* slots, int tps,
                    const uint32_t* tile_off, uint32_t* ids, cudaStream_t st) {
  if (n <= 0) return;
  k_scatter<<<(unsigned)((n + PREP_THREADS - 1) / PREP_THREADS), PREP_THREADS, 0, st>>>(rec, n, fp, slots, tps,
                                                                                        tile_off, ids);
}

void launch_sortlists(uint32_t* ids, uint32_t* tmp, const uint32_t* tile_off, int64_t ntiles, int64_t n,
                      cudaStream_t st) {
  if (n <= 1 || ntiles <= 0) return;
  int bits = 0;
  while (bits < 32 && ((uint64_t)(n - 1) >> bits) != 0) ++bits;
  const int passes = std::max(1, (bits + SORT_BITS - 1) / SORT_BITS);
  k_sortlists<<<(unsigned)ntiles, SORT_THREADS, 0, st>>>(ids, tmp, tile_off, passes);
}

void init_kernels() {
  init_tile_kernel();
  init_tile_sb_kernel();
  init_tile_ws_kernel();
  init_tile_wide_kernel();
  init_tile8_kernel();
  init_dbin_kernels();
}

}  // namespace starsim
