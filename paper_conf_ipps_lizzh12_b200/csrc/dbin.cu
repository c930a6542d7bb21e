// Deterministic binning: a stable counting sort of the (tile, star)
// pairs by tile, with no global atomics and no per-tile sort.  Used when the frame (or band) has at most DB_MAXT
// tiles and an ROI overlaps at most 2 x 2 tiles (R <= 65); bin.cu's atomic-slot pipeline covers the rest.
//
//   k_dcount     a1 + counts: CTA c takes stars [c*blk, (c+1)*blk) (blk = DB_CTA, or 1,024 for catalogues of at most
//                DB_SMALL_N stars: dbin_block); per star the record of step a1
//                (prep_star); per tile the number of pairs of the CTA (shared-memory atomics -- counts do not depend
//                on order) -> row c of the block-major count matrix C[c][tile] (coalesced).
//   k_dcolscan   per 8-tile column block: the rows staged in shared memory, exclusive scan of every tile's column
//                C[0..nCTA)[tile] in CTA order (in place) and the tile's total -> cnt[tile].
//   k_dplace     step a2 first on every CTA of the grid (each scans the tile totals; CTA c writes tile_off and the
//                work items of the tiles t = c mod gridDim -- no scan launch between the two; the grid has at least
//                ntiles / 256 CTAs), then CTA c's pairs are grouped by tile in shared memory (slots from
//                shared-memory atomics, in arbitrary order); a pair's rank in its group is the number of the group's
//                stars with a smaller index, and it goes to tile_off[t] + C[c][t] + rank: every tile list holds its
//                stars in ascending star index -- the unique CSR (reading R18), bit-exact, with no sort pass over the
//                lists and no atomics on global memory.  (Groups are (4096-star block, tile) pairs: a few stars each.)
//   k_dsmall     a catalogue of at most DB_CTA stars: all of the above in one CTA and one launch.
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "plan.cuh"
#include "prep.cuh"

namespace starsim {

constexpr int DB_CTA = 4096;                     // stars per CTA (one column of the count matrix)
constexpr int DC_THREADS = 1024;                 // k_dcount: DB_CTA / DC_THREADS stars per thread
constexpr int DC_PER = DB_CTA / DC_THREADS;
#ifndef DP_THREADS_OPT
#define DP_THREADS_OPT 1024
#endif
constexpr int DP_THREADS = DP_THREADS_OPT;        // k_dplace
#ifndef DP_MINB_OPT
#define DP_MINB_OPT (2048 / DP_THREADS_OPT)
#endif
#ifndef DC_MINB_OPT
#define DC_MINB_OPT 2
#endif
constexpr int DP_MINB = DP_MINB_OPT;              // CTAs per SM (all 245 CTAs of a 1M-star frame resident)
constexpr int DP_WARPS = DP_THREADS / 32;
constexpr int DP_KEYS = DB_CTA * 4;              // at most 2 x 2 tiles per star
constexpr int DP_SPT = DB_CTA / DP_THREADS;      // stars per thread (strided by DP_THREADS)
constexpr int DCS_THREADS = 256;

// CTAs that hold stars (at least one: CTA 0 plans the tiles of an empty routed catalogue)
// Stars per CTA (one row of the count matrix): DB_CTA, or DB_CTA_SMALL for catalogues of at most DB_SMALL_N stars
// (4x the CTAs: a small catalogue's binning is the per-CTA latency of a few CTAs).  A function of
// the catalogue capacity n only, the same for every kernel of a render.
constexpr int DB_CTA_SMALL = DC_THREADS;
#ifndef DB_SMALL_N_OPT
#define DB_SMALL_N_OPT 262144
#endif
constexpr int64_t DB_SMALL_N = DB_SMALL_N_OPT;
__host__ __device__ __forceinline__ int dbin_block(int64_t n) { return n <= DB_SMALL_N ? DB_CTA_SMALL : DB_CTA; }
__device__ __forceinline__ int dbin_live_ctas(int64_t n, int blk) { return n > 0 ? (int)((n + blk - 1) / blk) : 1; }
static_assert(DB_MAXT <= 65536 && DB_CTA <= 65536, "tile ids, slots and star indices are 16-bit in k_dplace");
static_assert(DP_WARPS <= 32, "dp_block_scan scans the warp sums with one warp");

// A star's tile box, packed: first tile t0 | dx << 16 | dy << 17 (it also covers t0 + 1 if dx, t0 + ntx if dy,
// t0 + ntx + 1 if both); DP_NONE if the star is culled.  Written by k_dcount, read by k_dplace.
constexpr uint32_t DP_NONE = 0xFFFFFFFFu;

template <int SPT>  // stars per thread: the CTA's block is DC_THREADS * SPT stars
__global__ void __launch_bounds__(DC_THREADS, DC_MINB_OPT) k_dcount(const float* __restrict__ X, const float* __restrict__ Y,
                                                       const float* __restrict__ M, int64_t n, FrameParams fp,
                                                       StarRec* __restrict__ rec, uint32_t* __restrict__ codes,
                                                       uint32_t* __restrict__ C,
                                                       int nCTA, int ntiles) {
  __shared__ uint32_t cnt[DB_MAXT];
  const int tid = threadIdx.x, cta = blockIdx.x;
  n = frame_n(n, fp);
  if (cta >= dbin_live_ctas(n, DC_THREADS * SPT)) return;  // beyond a routed catalogue's count: k_dcolscan skips it
  for (int t = tid; t < ntiles; t += DC_THREADS) cnt[t] = 0u;
  // all loads of the thread's stars first (one memory latency, not DC_PER)
  const int64_t i0 = (int64_t)cta * (DC_THREADS * SPT) + tid;
  float xs[SPT], ys[SPT], ms[SPT];
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int64_t i = i0 + (int64_t)k * DC_THREADS;
    const bool in = i < n;
    xs[k] = in ? __ldg(&X[i]) : 0.f;
    ys[k] = in ? __ldg(&Y[i]) : 0.f;
    ms[k] = in ? __ldg(&M[i]) : 0.f;
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int64_t i = i0 + (int64_t)k * DC_THREADS;
    if (i >= n) break;
    int cx0, cx1, cy0, cy1;
    const StarRec r = prep_star(xs[k], ys[k], ms[k], fp, cx0, cx1, cy0, cy1);
    rec[i] = r;
    uint32_t code = DP_NONE;
    if (r.lo != LO_CULLED) {
      const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
      const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
      for (int ty = ty0; ty <= ty1; ++ty)
        for (int tx = tx0; tx <= tx1; ++tx) atomicAdd(&cnt[ty * fp.ntx + tx], 1u);
      code = (uint32_t)(ty0 * fp.ntx + tx0) | (uint32_t)(tx1 - tx0) << 16 | (uint32_t)(ty1 - ty0) << 17;
    }
    codes[i] = code;  // the star's tile box for k_dplace (one coalesced word instead of a record gather)
  }
  __syncthreads();
  for (int t = tid; t < ntiles; t += DC_THREADS) C[(int64_t)cta * ntiles + t] = cnt[t];  // CTA-major row
}

// C is CTA-major: C[cta][t] (row stride ntiles), so k_dcount's and k_dplace's accesses to their own CTA's row are
// coalesced.  k_dcolscan takes DCS_TILES tiles per CTA, one per warp: lane l sums rows 8 l .. 8 l + 7 of its tile's
// column in registers, one warp scan of the lane sums per DCS_ROWS rows (carried), the exclusive prefixes written back
// in place, then the tile totals (round 1's one-warp-scan-per-32-rows chain was latency-bound: 10 us at T).
constexpr int DCS_TILES = 8;   // one tile per warp
constexpr int DCS_ROWS = 256;
constexpr int DCS_RPL = DCS_ROWS / 32;  // rows per lane
__global__ void __launch_bounds__(DCS_THREADS) k_dcolscan(uint32_t* __restrict__ C, int nCTA_cap, int ntiles,
                                                         uint32_t* __restrict__ cnt, int cstride, int64_t n,
                                                         const uint32_t* __restrict__ n_dev, int blk) {
  static_assert(DCS_THREADS == 32 * DCS_TILES, "one warp per tile");
  static_assert(DCS_ROWS == 32 * DCS_RPL, "a lane holds DCS_RPL consecutive rows");
  // warp w: tile t0 + w; lane l: rows 8 l .. 8 l + 7 of each DCS_ROWS-row block, summed serially in registers, then
  // one warp scan of the lane sums (a single dependent scan per block instead of one per 32 rows)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int t = blockIdx.x * DCS_TILES + warp;
  const int nCTA = (n_dev && n > 0) ? dbin_live_ctas(n < (int64_t)*n_dev ? n : (int64_t)*n_dev, blk) : nCTA_cap;
  if (t >= ntiles) return;  // warp-uniform (no block barrier below)
  uint32_t carry = 0;
  for (int r0 = 0; r0 < nCTA; r0 += DCS_ROWS) {
    uint32_t v[DCS_RPL];
    const int rb = r0 + DCS_RPL * lane;
#pragma unroll
    for (int i = 0; i < DCS_RPL; ++i) v[i] = rb + i < nCTA ? C[(int64_t)(rb + i) * ntiles + t] : 0u;  // (L1: the
    // 8 warps read the 8 words of one sector per row)
    uint32_t sum = 0;
#pragma unroll
    for (int i = 0; i < DCS_RPL; ++i) sum += v[i];
    uint32_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += u;
    }
    uint32_t run = carry + incl - sum;
#pragma unroll
    for (int i = 0; i < DCS_RPL; ++i) {
      if (rb + i < nCTA) C[(int64_t)(rb + i) * ntiles + t] = run;
      run += v[i];
    }
    carry += __shfl_sync(0xffffffffu, incl, 31);
  }
  if (lane == 0) cnt[(int64_t)t * cstride] = carry;
}

// block-wide exclusive scan of one value per thread (DP_THREADS); returns the prefix, *total the sum
__device__ __forceinline__ uint32_t dp_block_scan(uint32_t v, uint32_t* s_w, uint32_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t incl = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += u;
  }
  if (lane == 31) s_w[warp] = incl;
  __syncthreads();
  if (warp == 0) {  // exclusive scan of the DP_WARPS (= 32) warp sums; the total in slot DP_WARPS
    const uint32_t u = lane < DP_WARPS ? s_w[lane] : 0u;
    uint32_t wi = u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, wi, o);
      if (lane >= o) wi += t;
    }
    __syncwarp();
    if (lane < DP_WARPS) s_w[lane] = wi - u;
    if (lane == 31) s_w[DP_WARPS] = wi;
  }
  __syncthreads();
  const uint32_t pre = s_w[warp];
  *total = s_w[DP_WARPS];
  __syncthreads();
  return pre + incl - v;
}

struct DpSmem {
  uint32_t toff[DB_MAXT];        // step a2, computed by every CTA: the first list position of every tile
  uint4 s_w4[DP_WARPS];
  uint4 s_tot;
  uint32_t gstart[DB_MAXT + 1];  // per tile: pairs of the CTA, then the first position of the tile's group
  uint32_t cur[DB_MAXT];         // per tile: next free slot of its group; then the tile list position of the group
  uint16_t arr[DP_KEYS];          // the CTA's star indices grouped by tile (in arbitrary order inside a group)
  uint32_t s_w[DP_WARPS + 1];
  uint32_t bmap[DP_WARPS][DB_CTA / 32];  // per warp: a large group's members as a bitmap of star indices
  uint32_t nbig;                         // the tiles of the large groups
  uint16_t big[DP_KEYS / 32];
};
constexpr uint32_t DP_BIG = 32;  // groups of more pairs are placed through a bitmap, not the rank loop
static_assert(DP_KEYS / (DP_BIG + 1) < DP_KEYS / 32, "the large-group list holds every large group");

// tiles of a packed box (0 if the star is culled) and its e-th tile, e < box_n (row-major order inside the box)
__device__ __forceinline__ int box_n(uint32_t code) {
  return code == DP_NONE ? 0 : (1 + (int)((code >> 16) & 1u)) << (int)((code >> 17) & 1u);
}
__device__ __forceinline__ int box_tile(uint32_t code, int e, int ntx) {
  const int dx = (int)((code >> 16) & 1u);
  const int ex = e & dx, ey = e >> dx;
  return (int)(code & 0xFFFFu) + ey * ntx + ex;
}

// Step a2 inside k_dplace (no separate scan launch): every CTA scans the DB_MAXT tile totals k_dcolscan wrote (2 per
// thread) into S.toff, and CTA c writes tile_off, the work items, the split table and the header for the tiles
// t = c mod nCTA -- the same values k_scan_one computes (plan_tile).
template <bool SMEM_CNT = false>  // counts in shared memory (k_dsmall) instead of k_dcolscan's global totals
__device__ __forceinline__ void dp_scan_tiles(DpSmem& S, const uint32_t* __restrict__ cnt, int ntiles, int nCTA,
                                              uint32_t* __restrict__ tile_off, Header* hdr,
                                              WorkItem* __restrict__ items, uint2* __restrict__ split_tab,
                                              int plan, uint32_t* __restrict__ done) {
  const int part_cap = plan_cap(plan);
  const uint32_t split = plan_split(plan);
  constexpr int TPT = DB_MAXT / DP_THREADS;
  static_assert(TPT * DP_THREADS == DB_MAXT, "tiles per thread");
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, cta = blockIdx.x;
  uint32_t c[TPT];
  uint4 sum = make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
  for (int k = 0; k < TPT; ++k) {
    const int t = tid * TPT + k;
    c[k] = t < ntiles ? (SMEM_CNT ? cnt[t] : __ldcg(&cnt[t])) : 0u;  // dense totals (k_dcolscan, cstride 1)
    if (t < ntiles) sum = add4(sum, tile_counts(c[k], split));
  }
  const uint4 incl = warp_incl_scan4(sum, lane);
  if (lane == 31) S.s_w4[warp] = incl;
  __syncthreads();
  if (warp == 0) {  // exclusive scan of the warp sums; the total
    const uint4 v = lane < DP_WARPS ? S.s_w4[lane] : make_uint4(0u, 0u, 0u, 0u);
    const uint4 wi = warp_incl_scan4(v, lane);
    __syncwarp();
    if (lane < DP_WARPS) S.s_w4[lane] = sub4(wi, v);
    if (lane == 31) S.s_tot = wi;
  }
  __syncthreads();
  const uint4 pre = S.s_w4[warp];
  const uint4 ta = S.s_tot;
  const bool split_on = ta.y <= (uint32_t)part_cap;
  const uint32_t nparts = split_on ? ta.y : 0u, nsplit = split_on ? ta.z : 0u;
  const uint32_t lite0 = nparts + (uint32_t)ntiles - nsplit - ta.w;
  const uint4 ex = sub4(add4(pre, incl), sum);
  uint32_t run = ex.x, pb = ex.y, si = ex.z, li = ex.w;
  if (cta == 0 && tid == 0) plan_header(hdr, tile_off, ntiles, ta, part_cap);
#pragma unroll
  for (int k = 0; k < TPT; ++k) {
    const int t = tid * TPT + k;
    if (t >= ntiles) break;
    S.toff[t] = run;
    if (t % nCTA == cta) {
      plan_tile((uint32_t)t, c[k], run, pb, si, li, nparts, lite0, split_on, tile_off, items, split_tab, done, split);
    } else {  // the same prefix updates as plan_tile
      const uint4 u = tile_counts(c[k], split);
      run += u.x;
      pb += split_on ? u.y : 0u;
      si += split_on ? u.z : 0u;
      li += u.w;
    }
  }
  __syncthreads();
}

// Steps a3-a4 of k_dplace for the CTA's stars (codes in registers, star i = blockIdx.x DB_CTA + tid + k DP_THREADS):
// group the pairs by tile in shared memory, rank each in its group by star index, write it to
// tile_off[t] + C[t][cta] + rank (C == nullptr: a single CTA, every group starts at its tile's list start).
template <int SPT>
__device__ __forceinline__ void dp_place(DpSmem& S, const uint32_t (&code)[SPT], const FrameParams& fp,
                                         const uint32_t* __restrict__ C, int nCTA, int ntiles,
                                         uint32_t* __restrict__ ids) {
  const int tid = threadIdx.x, cta = blockIdx.x;
  const int64_t c0 = (int64_t)cta * (DP_THREADS * SPT);
  for (int t = tid; t <= ntiles; t += DP_THREADS) S.gstart[t] = 0u;
  if (tid == 0) S.nbig = 0u;
  __syncthreads();
  // group sizes
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int nb = box_n(code[k]);
    for (int e = 0; e < nb; ++e) atomicAdd(&S.gstart[box_tile(code[k], e, fp.ntx)], 1u);
  }
  __syncthreads();
  // exclusive scan of the group sizes (TPT consecutive tiles per thread)
  {
    constexpr int TPT = (DB_MAXT + DP_THREADS - 1) / DP_THREADS;
    uint32_t c[TPT], sum = 0;
#pragma unroll
    for (int k = 0; k < TPT; ++k) {
      const int t = tid * TPT + k;
      c[k] = t < ntiles ? S.gstart[t] : 0u;
      sum += c[k];
    }
    uint32_t tot;
    uint32_t run = dp_block_scan(sum, S.s_w, &tot);
#pragma unroll
    for (int k = 0; k < TPT; ++k) {
      const int t = tid * TPT + k;
      if (t < ntiles) {
        S.gstart[t] = run;
        S.cur[t] = run;
        if (c[k] > DP_BIG) {
          const uint32_t bi = atomicAdd(&S.nbig, 1u);
          SS_CHECK(bi < (uint32_t)(DP_KEYS / 32));
          S.big[bi] = (uint16_t)t;
        }
      }
      run += c[k];
    }
    if (tid == 0) S.gstart[ntiles] = tot;
  }
  __syncthreads();
  // group the star indices by tile (arbitrary order inside a group)
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int nb = box_n(code[k]);
    for (int e = 0; e < nb; ++e)
      S.arr[atomicAdd(&S.cur[box_tile(code[k], e, fp.ntx)], 1u)] = (uint16_t)(tid + k * DP_THREADS);
  }
  __syncthreads();
  // first list position of every group: tile_off[t] + (pairs of tile t in the CTAs before)
  for (int t = tid; t < ntiles; t += DP_THREADS) S.cur[t] = S.toff[t] + (C ? __ldcg(&C[(int64_t)cta * ntiles + t]) : 0u);
  __syncthreads();
  // a pair's rank in its group = the group's stars with a smaller index (groups of at most DP_BIG pairs: the common
  // case of uniform fields)
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const uint32_t idx = (uint32_t)(tid + k * DP_THREADS);
    const int nb = box_n(code[k]);
    for (int e = 0; e < nb; ++e) {
      const int t = box_tile(code[k], e, fp.ntx);
      const uint32_t g0 = S.gstart[t], g1 = S.gstart[t + 1];
      if (g1 - g0 > DP_BIG) continue;
      uint32_t rank = 0;
      for (uint32_t u = g0; u < g1; ++u) rank += S.arr[u] < idx ? 1u : 0u;
      ids[S.cur[t] + rank] = (uint32_t)c0 + idx;
    }
  }
  // larger groups (clustered fields: the rank loop would cost O(group^2)): one warp per group sets the members' bits
  // in a bitmap of the CTA's star indices, then writes the set bits in ascending order (a warp scan of the per-lane
  // counts) -- the same ascending-index list
  const int lane = tid & 31, warp = tid >> 5;
  uint32_t* bm = S.bmap[warp];
  for (uint32_t b = (uint32_t)warp; b < S.nbig; b += DP_WARPS) {
    const int t = S.big[b];
    const uint32_t g0 = S.gstart[t], g1 = S.gstart[t + 1];
    constexpr int WPL = DB_CTA / 32 / 32;  // bitmap words per lane
#pragma unroll
    for (int w = 0; w < WPL; ++w) bm[lane * WPL + w] = 0u;
    __syncwarp();
    for (uint32_t u = g0 + lane; u < g1; u += 32) {
      const uint32_t v = S.arr[u];
      atomicOr(&bm[v >> 5], 1u << (v & 31u));
    }
    __syncwarp();
    uint32_t cntl = 0;
#pragma unroll
    for (int w = 0; w < WPL; ++w) cntl += __popc(bm[lane * WPL + w]);
    uint32_t incl = cntl;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t q = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += q;
    }
    uint32_t pos = S.cur[t] + incl - cntl;
    SS_CHECK(__shfl_sync(0xffffffffu, incl, 31) == g1 - g0);  // every member's bit set once
#pragma unroll 1
    for (int w = 0; w < WPL; ++w) {
      uint32_t m = bm[lane * WPL + w];
      while (m) {
        const int b = __ffs(m) - 1;
        m &= m - 1u;
        ids[pos++] = (uint32_t)c0 + (uint32_t)((lane * WPL + w) * 32 + b);
      }
    }
    __syncwarp();
  }
}

template <int SPT>
__global__ void __launch_bounds__(DP_THREADS, DP_MINB) k_dplace(const uint32_t* __restrict__ codes, int64_t n, FrameParams fp,
                                                       const uint32_t* __restrict__ C, int nCTA, int ntiles,
                                                       const uint32_t* __restrict__ cnt, uint32_t* __restrict__ tile_off,
                                                       Header* hdr, WorkItem* __restrict__ items,
                                                       uint2* __restrict__ split_tab, int part_cap,
                                                       uint32_t* __restrict__ done, uint32_t* __restrict__ ids) {
  static_assert(TILE_W == 128 && TILE_H == 64, "tile boxes span at most 2 x 2 tiles for R <= DB_MAXR");
  extern __shared__ __align__(16) unsigned char dsm_raw[];
  DpSmem& S = *reinterpret_cast<DpSmem*>(dsm_raw);
  const int tid = threadIdx.x, cta = blockIdx.x;
  const int64_t c0 = (int64_t)cta * (DP_THREADS * SPT);
  n = frame_n(n, fp);
  // step a2 is spread over every CTA of the grid (CTA c plans the tiles t = c mod gridDim.x; the grid has at least
  // ntiles / 256 CTAs, so a sparse frame's plan is not one CTA's serial work); only the CTAs that hold stars go on
  dp_scan_tiles(S, cnt, ntiles, (int)gridDim.x, tile_off, hdr, items, split_tab, part_cap, done);
  if (cta >= dbin_live_ctas(n, DP_THREADS * SPT)) return;
  uint32_t code[SPT];
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int64_t i = c0 + tid + k * DP_THREADS;
    code[k] = i < n ? __ldg(&codes[i]) : DP_NONE;
  }
  dp_place<SPT>(S, code, fp, C, nCTA, ntiles, ids);
}

// k_dsmall: a catalogue of at most DB_CTA stars binned by ONE CTA in one launch -- k_dcount's step a1 and counts
// (shared-memory atomics), step a2 over the counts in shared memory (dp_scan_tiles: the CTA plans every tile), and
// k_dplace's grouping and ranking with no count matrix (one CTA: every group starts at its tile's list start).  The
// same records, CSR and plan as the three-kernel path, bit for bit; for small frames the launches and the count
// matrix round trip were the cost.
__global__ void __launch_bounds__(DP_THREADS, 1) k_dsmall(const float* __restrict__ X, const float* __restrict__ Y,
                                                          const float* __restrict__ M, int64_t n, FrameParams fp,
                                                          StarRec* __restrict__ rec, int ntiles,
                                                          uint32_t* __restrict__ tile_off, Header* hdr,
                                                          WorkItem* __restrict__ items, uint2* __restrict__ split_tab,
                                                          int part_cap, uint32_t* __restrict__ done,
                                                          uint32_t* __restrict__ ids) {
  static_assert(DP_THREADS == DC_THREADS && DP_SPT == DC_PER, "k_dcount's star-to-thread map");
  extern __shared__ __align__(16) unsigned char dsm_raw[];
  DpSmem& S = *reinterpret_cast<DpSmem*>(dsm_raw);
  const int tid = threadIdx.x;
  n = frame_n(n, fp);
  for (int t = tid; t < ntiles; t += DP_THREADS) S.cur[t] = 0u;  // the tile counts
  float xs[DP_SPT], ys[DP_SPT], ms[DP_SPT];
#pragma unroll
  for (int k = 0; k < DP_SPT; ++k) {
    const int64_t i = tid + (int64_t)k * DP_THREADS;
    const bool in = i < n;
    xs[k] = in ? __ldg(&X[i]) : 0.f;
    ys[k] = in ? __ldg(&Y[i]) : 0.f;
    ms[k] = in ? __ldg(&M[i]) : 0.f;
  }
  __syncthreads();
  uint32_t code[DP_SPT];
#pragma unroll
  for (int k = 0; k < DP_SPT; ++k) {
    const int64_t i = tid + (int64_t)k * DP_THREADS;
    code[k] = DP_NONE;
    if (i >= n) continue;
    int cx0, cx1, cy0, cy1;
    const StarRec r = prep_star(xs[k], ys[k], ms[k], fp, cx0, cx1, cy0, cy1);
    rec[i] = r;
    if (r.lo != LO_CULLED) {
      const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
      const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
      for (int ty = ty0; ty <= ty1; ++ty)
        for (int tx = tx0; tx <= tx1; ++tx) atomicAdd(&S.cur[ty * fp.ntx + tx], 1u);
      code[k] = (uint32_t)(ty0 * fp.ntx + tx0) | (uint32_t)(tx1 - tx0) << 16 | (uint32_t)(ty1 - ty0) << 17;
    }
  }
  __syncthreads();
  dp_scan_tiles<true>(S, S.cur, ntiles, 1, tile_off, hdr, items, split_tab, part_cap, done);
  dp_place<DP_SPT>(S, code, fp, nullptr, 1, ntiles, ids);
}


// ---------------------------------------------------------------------------------------------------------------
// k_dfused: k_dcount, k_dcolscan and k_dplace in ONE cooperative launch (every CTA resident: the driver refuses the
// launch otherwise), separated by two grid barriers -- no launch gaps, and each CTA keeps its stars' tile boxes in
// registers from the count to the placement.  Same records, count matrix, plan and CSR, bit for bit.
//   phase 1 (CTA c < live): step a1 + the CTA's pair counts -> row c of C;
//   barrier;
//   phase 2: 32-tile column blocks b = c, c + gridDim, ...: the live rows staged in shared memory, every tile's
//            column scanned (exclusive, in place) and its total -> cnt;
//   barrier;
//   phase 3: step a2 (every CTA, the tiles t = c mod gridDim) and, for the live CTAs, the placement.
// The barrier counter is zeroed by a memset node before every launch (api.cu), so no state survives a frame.
// ---------------------------------------------------------------------------------------------------------------
constexpr int DF_ROWS = 256;
struct DfSmem {
  union {
    uint32_t cnt[DB_MAXT];
    uint32_t sm[DF_ROWS][33];
    DpSmem dp;
  };
};

__device__ __forceinline__ void grid_barrier(uint32_t* bar, uint32_t target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(bar, 1u);
    uint32_t v;
    do {
      asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
    } while (v < target);
  }
  __syncthreads();
}

__global__ void __launch_bounds__(DP_THREADS, 2) k_dfused(const float* __restrict__ X, const float* __restrict__ Y,
                                                          const float* __restrict__ M, int64_t n, FrameParams fp,
                                                          StarRec* __restrict__ rec, uint32_t* __restrict__ C,
                                                          uint32_t* __restrict__ cntg, int ntiles,
                                                          uint32_t* __restrict__ tile_off, Header* hdr,
                                                          WorkItem* __restrict__ items, uint2* __restrict__ split_tab,
                                                          int part_cap, uint32_t* __restrict__ done,
                                                          uint32_t* __restrict__ ids, uint32_t* bar) {
  static_assert(DP_THREADS == DC_THREADS && DP_SPT == DC_PER, "k_dcount's star-to-thread map");
  static_assert(DP_THREADS == 1024, "phase 2: 32 warps, one per tile of a 32-tile block");
  extern __shared__ __align__(16) unsigned char dsm_raw[];
  DfSmem& F = *reinterpret_cast<DfSmem*>(dsm_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, cta = blockIdx.x;
  const uint32_t nC = gridDim.x;
  n = frame_n(n, fp);
  const int live = dbin_live_ctas(n, DB_CTA);
  // ---- phase 1 (k_dcount)
  uint32_t code[DP_SPT];
#pragma unroll
  for (int k = 0; k < DP_SPT; ++k) code[k] = DP_NONE;
  if (cta < live) {
    for (int t = tid; t < ntiles; t += DP_THREADS) F.cnt[t] = 0u;
    const int64_t i0 = (int64_t)cta * DB_CTA + tid;
    float xs[DP_SPT], ys[DP_SPT], ms[DP_SPT];
#pragma unroll
    for (int k = 0; k < DP_SPT; ++k) {
      const int64_t i = i0 + (int64_t)k * DP_THREADS;
      const bool in = i < n;
      xs[k] = in ? __ldg(&X[i]) : 0.f;
      ys[k] = in ? __ldg(&Y[i]) : 0.f;
      ms[k] = in ? __ldg(&M[i]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < DP_SPT; ++k) {
      const int64_t i = i0 + (int64_t)k * DP_THREADS;
      if (i >= n) break;
      int cx0, cx1, cy0, cy1;
      const StarRec r = prep_star(xs[k], ys[k], ms[k], fp, cx0, cx1, cy0, cy1);
      rec[i] = r;
      if (r.lo != LO_CULLED) {
        const int tx0 = cx0 / TILE_W, tx1 = cx1 / TILE_W;
        const int ty0 = (cy0 - fp.row0) / TILE_H, ty1 = (cy1 - fp.row0) / TILE_H;
        for (int ty = ty0; ty <= ty1; ++ty)
          for (int tx = tx0; tx <= tx1; ++tx) atomicAdd(&F.cnt[ty * fp.ntx + tx], 1u);
        code[k] = (uint32_t)(ty0 * fp.ntx + tx0) | (uint32_t)(tx1 - tx0) << 16 | (uint32_t)(ty1 - ty0) << 17;
      }
    }
    __syncthreads();
    for (int t = tid; t < ntiles; t += DP_THREADS) C[(int64_t)cta * ntiles + t] = F.cnt[t];
  }
  grid_barrier(bar, nC);
  // ---- phase 2 (k_dcolscan): 32-tile column blocks, warp w = tile t0 + w, lane l = rows l + 32 k
  for (int t0 = cta * 32; t0 < ntiles; t0 += (int)nC * 32) {
    const bool tin = t0 + lane < ntiles;
    uint32_t carry = 0;
    for (int r0 = 0; r0 < live; r0 += DF_ROWS) {
      const int rows = min(DF_ROWS, live - r0);
#pragma unroll
      for (int i = 0; i < DF_ROWS / 32; ++i) {
        const int r = warp + 32 * i;
        if (r < rows) F.sm[r][lane] = tin ? __ldcg(&C[(int64_t)(r0 + r) * ntiles + t0 + lane]) : 0u;
      }
      __syncthreads();
      for (int k = 0; k < DF_ROWS / 32 && 32 * k < rows; ++k) {
        const int r = 32 * k + lane;
        const uint32_t v = r < rows ? F.sm[r][warp] : 0u;
        uint32_t incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
          if (lane >= o) incl += u;
        }
        if (r < rows) F.sm[r][warp] = carry + incl - v;
        carry += __shfl_sync(0xffffffffu, incl, 31);
      }
      __syncthreads();
#pragma unroll
      for (int i = 0; i < DF_ROWS / 32; ++i) {
        const int r = warp + 32 * i;
        if (r < rows && tin) C[(int64_t)(r0 + r) * ntiles + t0 + lane] = F.sm[r][lane];
      }
      __syncthreads();
    }
    if (lane == 0 && t0 + warp < ntiles) cntg[t0 + warp] = carry;
  }
  grid_barrier(bar, 2u * nC);
  // ---- phase 3 (k_dplace)
  dp_scan_tiles(F.dp, cntg, ntiles, (int)nC, tile_off, hdr, items, split_tab, part_cap, done);
  if (cta >= live) return;
  dp_place<DP_SPT>(F.dp, code, fp, C, (int)nC, ntiles, ids);
}

size_t dbin_smem(int) { return sizeof(DpSmem); }

int dbin_ctas(int64_t n) { return (int)((n + dbin_block(n) - 1) / dbin_block(n)); }
bool dfused_block_ok(int64_t n) { return dbin_block(n) == DB_CTA; }  // k_dfused bins DB_CTA-star blocks only

void init_dbin_kernels() {
  cudaFuncSetAttribute(k_dplace<DP_SPT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(DpSmem));
  cudaFuncSetAttribute(k_dplace<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(DpSmem));
  cudaFuncSetAttribute(k_dsmall, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(DpSmem));
  cudaFuncSetAttribute(k_dfused, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(DfSmem));
}

bool dsmall_ok(int64_t n) { return n <= DB_CTA; }

// the largest co-resident k_dfused grid on this device (0: none); the fused binning applies when the catalogue's
// CTAs fit it (and the cooperative launch re-checks)
int dfused_max_grid(int num_sms) {
  int nb = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_dfused, DP_THREADS, sizeof(DfSmem)) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return nb * num_sms;
}

cudaError_t launch_dfused(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp,
                          StarRec* rec, uint32_t* C, uint32_t* cnt, int ntiles, uint32_t* tile_off, Header* hdr,
                          WorkItem* items, uint2* split_tab, int part_cap, uint32_t* done, uint32_t* ids,
                          uint32_t* bar, cudaStream_t st) {
  cudaMemsetAsync(bar, 0, sizeof(uint32_t), st);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)((n + DB_CTA - 1) / DB_CTA));
  cfg.blockDim = dim3(DP_THREADS);
  cfg.dynamicSmemBytes = sizeof(DfSmem);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_dfused, x, y, m, n, fp, rec, C, cnt, ntiles, tile_off, hdr, items, split_tab,
                            part_cap, done, ids, bar);
}

void launch_dsmall(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                   int ntiles, uint32_t* tile_off, Header* hdr, WorkItem* items, uint2* split_tab, int part_cap,
                   uint32_t* done, uint32_t* ids, cudaStream_t st) {
  k_dsmall<<<1, DP_THREADS, sizeof(DpSmem), st>>>(x, y, m, n, fp, rec, ntiles, tile_off, hdr, items, split_tab,
                                                  part_cap, done, ids);
}

void launch_dcount(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                   uint32_t* codes, uint32_t* C, int ntiles, cudaStream_t st) {
  const int nc = dbin_ctas(n);
  if (nc <= 0) return;
  if (dbin_block(n) == DB_CTA)
    k_dcount<DC_PER><<<nc, DC_THREADS, 0, st>>>(x, y, m, n, fp, rec, codes, C, nc, ntiles);
  else
    k_dcount<1><<<nc, DC_THREADS, 0, st>>>(x, y, m, n, fp, rec, codes, C, nc, ntiles);
}

void launch_dcolscan(uint32_t* C, int64_t n, int ntiles, uint32_t* cnt, int cstride, const uint32_t* n_dev,
                     cudaStream_t st) {
  k_dcolscan<<<(ntiles + DCS_TILES - 1) / DCS_TILES, DCS_THREADS, 0, st>>>(C, dbin_ctas(n), ntiles, cnt, cstride, n,
                                                                           n_dev, dbin_block(n));
}

void launch_dplace(const uint32_t* codes, int64_t n, const FrameParams& fp, const uint32_t* C, int ntiles,
                   const uint32_t* cnt, uint32_t* tile_off, Header* hdr, WorkItem* items, uint2* split_tab,
                   int part_cap, uint32_t* done, uint32_t* ids, cudaStream_t st) {
  const int nc = dbin_ctas(n);
  const int grid = std::max(nc, (ntiles + 255) / 256);  // planning CTAs (k_dplace)
  if (nc <= 0) return;
  auto* k = dbin_block(n) == DB_CTA ? k_dplace<DP_SPT> : k_dplace<1>;
  k<<<grid, DP_THREADS, sizeof(DpSmem), st>>>(codes, n, fp, C, nc, ntiles, cnt, tile_off, hdr, items, split_tab,
                                              part_cap, done, ids);
}

}  // namespace starsim
