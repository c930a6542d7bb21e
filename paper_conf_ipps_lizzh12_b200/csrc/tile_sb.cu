// Tile accumulation with sorted corner bins (DESIGN.md §The tile kernel) -- the kernel for
// R <= SB_MAXR (every BASELINE config except the wide-ROI end of the C4 sweep, which uses tile.cu).
//
// Same contract, tile geometry, lane layout and epilogue as tile.cu (tile_common.cuh): one CTA renders one 128 x 64
// tile (or one part of a split heavy tile) from its CSR star list, accumulating Eq. 3's sum of separable Eq. 2 terms
// [s' gy(r)] * gx(c) in fp32 registers, and writes every pixel once.  What differs is how a chunk of up to 256 stars
// is prepared and walked:
//
//   sort   (thread = star): the star's ROI clipped to the tile starts in band b0 = r0/16 and strip q0 = c0/8 (its
//          "corner bin", 4 x 16 bins).  A stable counting sort by corner bin (warp match + per-warp histogram + one
//          scan) gives the star its sorted index j.  For R <= 17 the ROI spans at most 2 bands and 3 strips, so the
//          stars that can touch the block (B, Q) of lane group q are exactly those with corner bins
//          (B-1, Q-2..Q) and (B, Q-2..Q): two contiguous ranges of the sorted order.  No per-block lists are built.
//   prep   (thread = star): its row profile s' gy on its two bands b0, b0+1 (16-float band slots in the [hq][i]
//          order the lanes read) and its column profile gx on strips q0..q0+2 (8-float strip slots in a ring of
//          4 indexed by Q & 3), zero outside the ROI, at fixed places of sorted star j: one MUFU.EX2 per value.
//   accumulate (warp): lane group q walks its two ranges (band slot 1 for the corner band B-1, band slot 0 for B),
//          padded with an all-zero slot to the warp's longest walk; a step is three LDS.128 (4 row factors, 8 column
//          factors) and 16 FFMA2.  Stars of a range that do not reach the block read all-zero slots (exact zeros).
//
// Bank conflicts: strip slot of strip Q sits at ring position Q & 3 with its two 16-B halves swapped when bit 2 of
// Q is set, so the 8 lane groups of a warp always hit 8 distinct bank quads; band slot k of star j sits in the half
// (j ^ k) & 1 of the star's 128 B, spreading the groups of a warp over both halves.
//
// Summation order of a pixel: range 1 then range 2, each in sorted order (corner bin, then the tile list's star
// order) -- deterministic, and a function of the tile's own list only, so band renders stay bitwise equal to the
// frame (reading R12).  No atomics on the image.
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "prep.cuh"
#include "tile_common.cuh"

namespace starsim {

#ifdef STARSIM_SB_TIMING
// per-phase SM cycles summed over warps (debug builds only): sort, scan, profiles, wait, accumulate, chunks
__device__ unsigned long long g_sb_prof[6];
#define SB_T(v) const long long v = clock64()
#define SB_ACC(k, d) if (lane == 0) atomicAdd(&g_sb_prof[k], (unsigned long long)(d))
#else
#define SB_T(v)
#define SB_ACC(k, d)
#endif

// corner bins: band key 0..4 (0 = the ROI comes in over the tile's top edge, else 1 + band) x strip key 0..16 (0 =
// it comes in over the left edge, else 1 + strip), band-major
constexpr int SB_NSK = NSTRIPS + 1;
constexpr int SB_NBIN = (NBANDS + 1) * SB_NSK;  // 85
constexpr int SB_CHUNK = CHUNK;             // stars per chunk (<= TILE_THREADS; 192 with 4 CTAs/SM measured slower: spills)
#ifndef SB_MINB_OPT
#define SB_MINB_OPT 2
#endif
constexpr int SB_MINB = SB_MINB_OPT;         // CTAs per SM: 2 (128 registers, no spills; 3 CTAs at 80 registers spilled and measured 4-20 % slower, profiles/r2_ab_minb.txt)
constexpr int SB_MINB_CIRC = 2;             // the circle variant: 2 CTAs per SM, registers for its per-pixel mask
constexpr uint32_t SB_ZJ = SB_CHUNK;        // the all-zero slot

struct SbSmem {
  float gy[(SB_CHUNK + 1) * 32];    // sorted star j: two 16-float band slots, slot k at j*32 + ((j ^ k) & 1) * 16
  float gx[(SB_CHUNK + 1) * 32];    // sorted star j: ring of four 8-float strip slots, strip Q at j*32 + (Q & 3) * 8
  uint32_t hist[TILE_WARPS][SB_NBIN];      // per warp: stars of each corner bin
  uint32_t binoff[TILE_WARPS][SB_NBIN];    // per warp, per bin: stars of the bin in the warps before
  uint32_t binstart[SB_NBIN + 1];          // exclusive scan of the bin totals (bin-major)
  uint32_t lo2[SB_CHUNK + 1];              // CIRC: sorted star j's ROI origin (tile-relative, int16 x | int16 y << 16)
};

// NEXT-3 in the tiled path (CIRC): the walk masks every ROI pixel outside the pixel circle of reading R21 --
// (2 (col - lo_x) - (R-1))^2 + (2 (row - lo_y) - (R-1))^2 <= R^2 per (row, column) of the lane's 4 x 8 block, with
// the star's ROI origin read from its slot.  The profiles, slots and summation order are unchanged.
template <bool INTEG, bool CIRC>
__global__ void __launch_bounds__(TILE_THREADS, CIRC ? SB_MINB_CIRC : SB_MINB) k_tile_sb(const uint32_t* __restrict__ ids,
                                                             const StarRec* __restrict__ rec, FrameParams fp,
                                                             void* __restrict__ out_,
                                                             const WorkItem* __restrict__ items,
                                                             const uint2* __restrict__ split_tab,
                                                             float* __restrict__ part_buf,
                                                             uint32_t* __restrict__ done, Header* hdr, float* __restrict__ seg_scratch) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  SbSmem& S = *reinterpret_cast<SbSmem*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  // exp(-d^2 / 2 sigma^2) = 2^(-(d * sk)^2); d = pixel - centre is formed exactly (tile-relative integer minus the
  // tile-relative centre, both exact in fp32) before the one scaling rounding.
  const float sk = fp.sk;

  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base = (uint32_t)__cvta_generic_to_shared(S.gy) + 16u * hq;
  const uint32_t gx_base = (uint32_t)__cvta_generic_to_shared(S.gx) + 32u * (Q & 3);
  // the strip halves of lanes with swz = 1 are stored swapped: those lanes load columns 4-7 first and hold them in
  // acc[i][0..1] until the epilogue swaps them back (so both loads use the same address + an immediate offset)
  __shared__ int s_last;
  if (tid < 32) {
    S.gy[SB_ZJ * 32 + tid] = 0.f;
    S.gx[SB_ZJ * 32 + tid] = 0.f;
  }

  // Persistent CTAs (SB_MINB per SM): item blockIdx.x first, then items from a counter k_scan zeroed (parts of heavy
  // tiles come first).  The next item's index is fetched when an item starts, its WorkItem when the first chunk's
  // profiles are done, its first star ids before the last chunk's accumulation and its records after it: the
  // latency of starting a tile hides behind the previous tile's work.
  __shared__ uint32_t s_next;
  // with k_tile_lite (fp.lite) this kernel takes the items before the light ones
  const uint32_t nitems = fp.lite ? __ldcg(&hdr->lite0) : __ldcg(&hdr->nitems);
  uint32_t item = blockIdx.x;
  if (item >= nitems) return;
  WorkItem wi = items[item];
  StarRec rnext = {};
  if (tid < SB_CHUNK && wi.jb + tid < wi.je) rnext = rec[ids[wi.jb + tid]];
  for (;;) {
  uint32_t nxt = 0;
  if (tid == 0) nxt = atomicAdd(&hdr->next_item, 1u) + gridDim.x;
  uint32_t item_n = 0xFFFFFFFFu, nid0 = 0;
  WorkItem wn = {0u, 0u, 0u, 0u};
  bool fetched = false;
  const int tx = (int)(wi.tile % (uint32_t)fp.ntx), ty = (int)(wi.tile / (uint32_t)fp.ntx);
  const int X0 = tx * TILE_W;    // first column of the tile
  const int Y0 = ty * TILE_H;    // first row of the tile, relative to the band
  const int IY0 = fp.row0 + Y0;  // first image row of the tile
  const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
  float2 acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);

  const uint32_t j1 = wi.je;
  static_assert(SPLIT_LEN % SB_CHUNK == 0, "segments are whole chunks");
  uint32_t segs_done = 0;  // SPLIT_LEN segments of this item already in the scratch (tile_common.cuh)
  for (uint32_t base = wi.jb; base < j1; base += SB_CHUNK) {
    // ======================= sort: thread = star (base + tid) of the tile's list
    const int nvalid = (int)min((uint32_t)SB_CHUNK, j1 - base);
    const StarRec r = rnext;
    int c0 = 0, c1 = -1, r0 = 0, r1 = -1;
    uint32_t key = SB_NBIN, lo2 = 0u;
    if (tid < nvalid) {
      const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
      lo2 = (uint32_t)(lx & 0xFFFF) | (uint32_t)ly << 16;
      c0 = max(lx, 0);
      c1 = min(lx + fp.R - 1, TWe - 1);
      r0 = max(ly, 0);
      r1 = min(ly + fp.R - 1, THe - 1);
      if (c0 <= c1 && r0 <= r1) key = (uint32_t)((ly < 0 ? 0 : 1 + (r0 >> 4)) * SB_NSK + (lx < 0 ? 0 : 1 + (c0 >> 3)));
    }
    SB_T(t0);
    const uint32_t peers = __match_any_sync(0xffffffffu, key);
    const uint32_t rank = __popc(peers & lt);
    // No barrier before this: the previous chunk's readers of hist (warp 0's scan) finished before its second
    // barrier; binstart / the slots are rewritten only after the next barrier.
    S.hist[warp][lane] = 0u;
    S.hist[warp][lane + 32] = 0u;
    if (lane < SB_NBIN - 64) S.hist[warp][lane + 64] = 0u;
    __syncwarp();
    if (rank == 0 && key < SB_NBIN) S.hist[warp][key] = __popc(peers);
    // next chunk's star id now (its record is requested just before the accumulation)
    const uint32_t nb = base + SB_CHUNK;
    const uint32_t nid = tid < SB_CHUNK && nb + tid < j1 ? __ldg(&ids[nb + tid]) : 0u;
    __syncthreads();
    SB_T(t1);
    if (warp == 0) {
      // per bin: its 8 histogram words first (independent loads), then the prefix over the warps
      uint32_t tot[3], sum = 0;
#pragma unroll
      for (int h = 0; h < 3; ++h) {
        const int bin = 3 * lane + h;
        uint32_t c[TILE_WARPS];
#pragma unroll
        for (int w = 0; w < TILE_WARPS; ++w) c[w] = bin < SB_NBIN ? S.hist[w][bin] : 0u;
        uint32_t run = 0;
#pragma unroll
        for (int w = 0; w < TILE_WARPS; ++w) {
          if (bin < SB_NBIN) S.binoff[w][bin] = run;
          run += c[w];
        }
        tot[h] = run;
        sum += run;
      }
      uint32_t incl = sum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
      }
      uint32_t ex = incl - sum;
#pragma unroll
      for (int h = 0; h < 3; ++h) {
        const int bin = 3 * lane + h;
        if (bin <= SB_NBIN) S.binstart[bin] = ex;  // bin SB_NBIN (lane 28, h 1) receives the total
        ex += tot[h];
      }
    }
    __syncthreads();
    SB_T(t2);
    // ======================= prep: the star's profiles at its sorted place j
    if (key < SB_NBIN) {
      const uint32_t j = S.binstart[key] + S.binoff[warp][key] + rank;
      const float yr = r.y - (float)IY0, xr = r.x - (float)X0;  // exact
      const float2 sk2 = make_float2(sk, sk), s2 = make_float2(r.s, r.s);
      if (CIRC) S.lo2[j] = lo2;
      // first band / strip of the slots: the corner bin's (-1 for an ROI that comes in over the top / left edge)
      const int b0 = (int)(key / SB_NSK) - 1, q0 = (int)(key % SB_NSK) - 1;
      // band slots (lane hq reads rows 4 hq .. 4 hq + 3 of a band): the two bands b0, b0+1 are 8 row quads w = 0..7
      // (band w >> 2, rows 4 (w & 3) ..) of which the ROI's <= 17 rows touch at most 5 consecutive ones, from
      // qfirst: iterations c = 0..4 compute quads qfirst + c, c = 5..7 store the other three as zeros (mod 8)
      const int ra0 = r0 - 16 * b0, rb0 = r1 - 16 * b0;      // ROI rows relative to band b0 (band b0+1: -16)
      const uint32_t m0 = (0xFFFFFFFFu >> (31 - min(rb0, 31))) & (0xFFFFFFFFu << ra0);  // ROI rows over both bands
      const float bf0 = (float)(16 * b0) - yr;              // exact
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        // lane-rotated order: u = (c + lane) & 7 picks the slot half u & 1 and the row group u >> 1, so the 8 lanes
        // of each quarter warp store to 8 distinct bank quads
        const int u = (c + lane) & 7;
        const int hh = u >> 1, k = (u ^ (int)j) & 1;
        const int w = 4 * k + hh;
        float4* dst = reinterpret_cast<float4*>(&S.gy[j * 32 + (u & 1) * 16 + hh * 4]);
        const uint32_t m = m0 >> (4 * w);                  // bit i: row 4 w + i of the window in the ROI
        const float bf = bf0 + (float)(4 * w);              // exact
        float v[4];
        if (!INTEG) {
          const float2 bb = make_float2(bf, bf);
#pragma unroll
          for (int i = 0; i < 4; i += 2) {
            float2 d = __fadd2_rn(bb, make_float2((float)i, (float)(i + 1)));
            d = __fmul2_rn(d, sk2);
            d = __fmul2_rn(d, make_float2(-d.x, -d.y));
            const float2 e = __fmul2_rn(make_float2(ex2_approx(d.x), ex2_approx(d.y)), s2);
            v[i] = (m >> i) & 1u ? e.x : 0.f;
            v[i + 1] = (m >> (i + 1)) & 1u ? e.y : 0.f;
          }
        } else {
          // pixel-integrated rows: the 4 consecutive rows share their 5 edges
          float t = (bf - 0.5f) * fp.kint, e = edge_erfc(t);
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float tn = (bf + (float)i + 0.5f) * fp.kint, en = edge_erfc(tn);
            v[i] = (m >> i) & 1u ? r.s * pix_mass(t, e, tn, en) : 0.f;
            t = tn;
            e = en;
          }
        }
        *dst = make_float4(v[0], v[1], v[2], v[3]);
      }
#pragma unroll
      for (int k = 0; k < 3; ++k) {
        const int Qs = q0 + k;
        const int rel = 8 * Qs;                              // first column of the strip (tile-relative)
        const int lo = max(c0 - rel, 0), hi = min(c1 - rel, 7);
        const uint32_t m = hi >= lo ? ((0xFFu >> (7 - hi)) & (0xFFu << lo)) : 0u;
        const float bf = (float)rel - xr;                    // exact
        float v[8];
        if (!INTEG) {
#pragma unroll
          for (int p = 0; p < 8; p += 2) {
            float2 d = __fmul2_rn(__fadd2_rn(make_float2(bf, bf), make_float2((float)p, (float)(p + 1))), sk2);
            d = __fmul2_rn(d, make_float2(-d.x, -d.y));
            v[p] = (m >> p) & 1u ? ex2_approx(d.x) : 0.f;
            v[p + 1] = (m >> (p + 1)) & 1u ? ex2_approx(d.y) : 0.f;
          }
        } else {
          float t = (bf - 0.5f) * fp.kint, e = edge_erfc(t);
#pragma unroll
          for (int p = 0; p < 8; ++p) {
            const float tn = (bf + (float)p + 0.5f) * fp.kint, en = edge_erfc(tn);
            v[p] = (m >> p) & 1u ? pix_mass(t, e, tn, en) : 0.f;
            t = tn;
            e = en;
          }
        }
        float* gs = &S.gx[j * 32 + (Qs & 3) * 8];
        const int sw = ((Qs >> 2) & 1) * 4;
        *reinterpret_cast<float4*>(gs + sw) = make_float4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<float4*>(gs + (sw ^ 4)) = make_float4(v[4], v[5], v[6], v[7]);
      }
    }
    // this lane group's two ranges of the sorted order: corner bins (B-1, qlo..Q) then (B, qlo..Q)
    // strip keys max(Q-2, -1) + 1 .. Q + 1; band key B (corner band B-1, incl. the top-edge key 0), then B + 1
    const int sklo = max(Q - 1, 0);
    const uint32_t s1r = S.binstart[B * SB_NSK + sklo], e1r = S.binstart[B * SB_NSK + Q + 2];
    const uint32_t s2r = S.binstart[(B + 1) * SB_NSK + sklo], e2r = S.binstart[(B + 1) * SB_NSK + Q + 2];
    const uint32_t len1 = e1r - s1r, L = len1 + (e2r - s2r);
    const uint32_t steps = __reduce_max_sync(0xffffffffu, L);
    // step t of the walk reads sorted star j = t + c (c = s1r in range 1, s2r - len1 in range 2); its band slot
    // k (1 in range 1, 0 in range 2) sits in half (j ^ k) & 1 = (t & 1) ^ ((c + k) & 1).  So per range and per
    // parity of t the gy address is base + 128 t: the loop below runs step pairs (even, odd).
    const uint32_t c1v = s1r, c2v = s2r - len1;
    const uint32_t e1 = (c1v + 1u) & 1u, e2 = c2v & 1u;
    const uint32_t g1e = gy_base + c1v * 128u + e1 * 64u, g1o = gy_base + c1v * 128u + (e1 ^ 1u) * 64u;
    const uint32_t g2e = gy_base + c2v * 128u + e2 * 64u, g2o = gy_base + c2v * 128u + (e2 ^ 1u) * 64u;
    const uint32_t x1 = gx_base + c1v * 128u, x2 = gx_base + c2v * 128u;
    const uint32_t gz = gy_base + SB_ZJ * 128u, xz = gx_base + SB_ZJ * 128u;
    const bool first = base == wi.jb, last = nb >= j1;
    if (first && tid == 0) s_next = nxt;
    SB_T(t3);
    __syncthreads();
    SB_T(t4);

    if (first) {
      fetched = true;
      item_n = s_next;
      if (item_n < nitems) wn = items[item_n];
    }
    if (!last) {
      if (tid < SB_CHUNK && nb + tid < j1) rnext = rec[nid];
    } else if (item_n < nitems && tid < SB_CHUNK && wn.jb + tid < wn.je) {
      nid0 = __ldg(&ids[wn.jb + tid]);
    }
    // ======================= accumulate: lane group q walks its two ranges (padded with the zero slot)
    auto step = [&](uint32_t t, bool odd) {
      const bool in1 = t < len1, in = t < L;
      uint32_t ga = (in1 ? (odd ? g1o : g1e) : (odd ? g2o : g2e)) + t * 128u;
      uint32_t xa = (in1 ? x1 : x2) + t * 128u;
      ga = in ? ga : gz;
      xa = in ? xa : xz;
      float4 g, a, c;
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g.x), "=f"(g.y), "=f"(g.z), "=f"(g.w) : "r"(ga));
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w) : "r"(xa));
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(c.x), "=f"(c.y), "=f"(c.z), "=f"(c.w) : "r"(xa + 16u));
      const float gi[4] = {g.x, g.y, g.z, g.w};
      if (!CIRC) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 gg = make_float2(gi[i], gi[i]);
          acc[i][0] = __ffma2_rn(gg, make_float2(a.x, a.y), acc[i][0]);
          acc[i][1] = __ffma2_rn(gg, make_float2(a.z, a.w), acc[i][1]);
          acc[i][2] = __ffma2_rn(gg, make_float2(c.x, c.y), acc[i][2]);
          acc[i][3] = __ffma2_rn(gg, make_float2(c.z, c.w), acc[i][3]);
        }
      } else {
        // the star's ROI origin (its slot's), then per row the largest squared column offset inside the circle
        const uint32_t jj = in ? t + (in1 ? c1v : c2v) : SB_ZJ;
        const uint32_t lo = S.lo2[jj];
        const int lx = (int)(int16_t)(lo & 0xFFFFu), ly = (int)(int16_t)(lo >> 16);
        const float gx[8] = {a.x, a.y, a.z, a.w, c.x, c.y, c.z, c.w};  // columns 8 Q + ((p + 4 swz) & 7)
        const int RR = fp.R * fp.R, R1 = fp.R - 1;
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int v = 2 * (16 * B + 4 * hq + i - ly) - R1;
          const int thr = RR - v * v;
          float gm[8];
#pragma unroll
          for (int p = 0; p < 8; ++p) {
            const int u = 2 * (8 * Q + ((p + 4 * swz) & 7) - lx) - R1;
            gm[p] = u * u <= thr ? gx[p] : 0.f;
          }
          const float2 gg = make_float2(gi[i], gi[i]);
          acc[i][0] = __ffma2_rn(gg, make_float2(gm[0], gm[1]), acc[i][0]);
          acc[i][1] = __ffma2_rn(gg, make_float2(gm[2], gm[3]), acc[i][1]);
          acc[i][2] = __ffma2_rn(gg, make_float2(gm[4], gm[5]), acc[i][2]);
          acc[i][3] = __ffma2_rn(gg, make_float2(gm[6], gm[7]), acc[i][3]);
        }
      }
    };
    uint32_t st = 0;
#pragma unroll 2
    for (; st + 1 < steps; st += 2) {
      step(st, false);
      step(st + 1, true);
    }
    if (st < steps) step(st, false);
#ifdef STARSIM_SB_TIMING
    {
      SB_T(t5);
      SB_ACC(0, t1 - t0);
      SB_ACC(1, t2 - t1);
      SB_ACC(2, t3 - t2);
      SB_ACC(3, t4 - t3);
      SB_ACC(4, t5 - t4);
      SB_ACC(5, 1);
    }
#endif
    if ((base + SB_CHUNK - wi.jb) % SPLIT_LEN == 0 && base + SB_CHUNK < j1) {
      seg_flush(acc, seg_scratch, segs_done == 0);
      ++segs_done;
    }
  }

  // ======================= output
  if (segs_done) seg_finish(acc, seg_scratch);
  if (swz) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 t0 = acc[i][0], t1 = acc[i][1];
      acc[i][0] = acc[i][2];
      acc[i][1] = acc[i][3];
      acc[i][2] = t0;
      acc[i][3] = t1;
    }
  }
  if (tile_reduce_parts<true>(acc, wi, split_tab, part_buf, done, B, wx, q, hq, &s_last))
    tile_store<true>(acc, fp, out_, Y0, X0 + 64 * wx + 8 * q, B, hq);
  if (!fetched) {  // an item with an empty list ran no chunk
    if (tid == 0) s_next = nxt;
    __syncthreads();
    item_n = s_next;
    if (item_n < nitems) {
      wn = items[item_n];
      if (tid < SB_CHUNK && wn.jb + tid < wn.je) nid0 = __ldg(&ids[wn.jb + tid]);
    }
  }
  if (item_n >= nitems) break;
  rnext = StarRec{};
  if (tid < SB_CHUNK && wn.jb + tid < wn.je) rnext = rec[nid0];
  wi = wn;
  item = item_n;
  }  // work loop
}


// One chunk of <= CAP stars of a tile's list, given in list order (thread t < n holds star t's record r): the stars
// ranked by corner bin (stable: then list order) exactly as a k_tile_sb chunk is sorted, and walked by every warp whose
// 64 x 16 region the ROI meets, each lane evaluating its own 4 row and 8 column factors with the very operations of
// k_tile_sb's slot preparation and adding them in that order (same per-pixel sums, bit for bit).  Two barriers; the
// arrays are the caller's shared memory.
template <bool INTEG, bool CIRC, int CAP>
__device__ __forceinline__ void lite_chunk(float2 (&acc)[4][4], uint32_t* lkey, float4* lrec, uint32_t* llo,
                                           const StarRec& r, int n, const FrameParams& fp, int X0, int IY0,
                                           int TWe, int THe) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const float sk = fp.sk;
  uint32_t key = SB_NBIN, lo2 = 0u;
  if (tid < n) {
    const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
    lo2 = (uint32_t)(lx & 0xFFFF) | (uint32_t)ly << 16;
    const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TWe - 1);
    const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, THe - 1);
    if (c0 <= c1 && r0 <= r1) key = (uint32_t)((ly < 0 ? 0 : 1 + (r0 >> 4)) * SB_NSK + (lx < 0 ? 0 : 1 + (c0 >> 3)));
    lkey[tid] = key;
  }
  __syncthreads();
  if (tid < n) {
    uint32_t rank = 0;
    for (int u = 0; u < n; ++u) {
      const uint32_t ku = lkey[u];
      rank += (ku < key || (ku == key && u < tid)) ? 1u : 0u;
    }
    lrec[rank] = make_float4(r.x - (float)X0, r.y - (float)IY0, r.s, __uint_as_float(key));  // exact
    llo[rank] = lo2;
  }
  __syncthreads();
  const float2 sk2 = make_float2(sk, sk);
  for (int k = 0; k < n; ++k) {
    const float4 st = lrec[k];
    const uint32_t sk_key = __float_as_uint(st.w);
    if (sk_key >= (uint32_t)SB_NBIN) continue;
    const uint32_t lo = llo[k];
    const int lx = (int)(int16_t)(lo & 0xFFFFu), ly = (int)(int16_t)(lo >> 16);
    const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TWe - 1);
    const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, THe - 1);
    // the warp's 64 x 16 region (uniform branch)
    if (r1 < 16 * B || r0 > 16 * B + 15 || c1 < 64 * wx || c0 > 64 * wx + 63) continue;
    const int b0 = (int)(sk_key / SB_NSK) - 1, q0 = (int)(sk_key % SB_NSK) - 1;
    const float xr = st.x, yr = st.y;
    // row factors of rows 16 B + 4 hq + i: quad w = 4 (B - b0) + hq of the star's two bands (slot preparation)
    float gyv[4];
    {
      const int ra0 = r0 - 16 * b0, rb0 = r1 - 16 * b0;
      const uint32_t m0 = (0xFFFFFFFFu >> (31 - min(rb0, 31))) & (0xFFFFFFFFu << ra0);
      const int w = 4 * (B - b0) + hq;
      const uint32_t m = (w >= 0 && w < 8) ? m0 >> (4 * w) : 0u;
      const float bf0 = (float)(16 * b0) - yr;
      const float bf = bf0 + (float)(4 * w);
      if (!INTEG) {
        const float2 s2 = make_float2(st.z, st.z);
        const float2 bb = make_float2(bf, bf);
#pragma unroll
        for (int i = 0; i < 4; i += 2) {
          float2 d = __fadd2_rn(bb, make_float2((float)i, (float)(i + 1)));
          d = __fmul2_rn(d, sk2);
          d = __fmul2_rn(d, make_float2(-d.x, -d.y));
          const float2 e = __fmul2_rn(make_float2(ex2_approx(d.x), ex2_approx(d.y)), s2);
          gyv[i] = (m >> i) & 1u ? e.x : 0.f;
          gyv[i + 1] = (m >> (i + 1)) & 1u ? e.y : 0.f;
        }
      } else {
        float t = (bf - 0.5f) * fp.kint, e = edge_erfc(t);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float tn = (bf + (float)i + 0.5f) * fp.kint, en = edge_erfc(tn);
          gyv[i] = (m >> i) & 1u ? st.z * pix_mass(t, e, tn, en) : 0.f;
          t = tn;
          e = en;
        }
      }
    }
    // column factors of strip Q (one of the star's strips q0 .. q0 + 2, else zero) in the lane's load order:
    // slot p holds column 8 Q + pp, pp = (p + 4 swz) & 7 (the same operations on the same operands as k_tile_sb)
    float gxv[8];
    {
      const int rel = 8 * Q;
      const int lo_ = max(c0 - rel, 0), hi = min(c1 - rel, 7);
      const uint32_t m = (Q >= q0 && Q <= q0 + 2 && hi >= lo_) ? ((0xFFu >> (7 - hi)) & (0xFFu << lo_)) : 0u;
      const float bf = (float)rel - xr;
      if (!INTEG) {
#pragma unroll
        for (int p = 0; p < 8; p += 2) {
          const int pp = (p + 4 * swz) & 7;
          float2 d = __fmul2_rn(__fadd2_rn(make_float2(bf, bf), make_float2((float)pp, (float)(pp + 1))), sk2);
          d = __fmul2_rn(d, make_float2(-d.x, -d.y));
          gxv[p] = (m >> pp) & 1u ? ex2_approx(d.x) : 0.f;
          gxv[p + 1] = (m >> (pp + 1)) & 1u ? ex2_approx(d.y) : 0.f;
        }
      } else {
        float v[8];
        float t = (bf - 0.5f) * fp.kint, e = edge_erfc(t);
#pragma unroll
        for (int p = 0; p < 8; ++p) {
          const float tn = (bf + (float)p + 0.5f) * fp.kint, en = edge_erfc(tn);
          v[p] = (m >> p) & 1u ? pix_mass(t, e, tn, en) : 0.f;
          t = tn;
          e = en;
        }
#pragma unroll
        for (int p = 0; p < 8; ++p) gxv[p] = swz ? v[(p + 4) & 7] : v[p];
      }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 gg = make_float2(gyv[i], gyv[i]);
      if (CIRC) {
        const int RR = fp.R * fp.R, R1 = fp.R - 1;
        const int v = 2 * (16 * B + 4 * hq + i - ly) - R1;
        const int thr = RR - v * v;
        float gm[8];
#pragma unroll
        for (int p = 0; p < 8; ++p) {
          const int u = 2 * (8 * Q + ((p + 4 * swz) & 7) - lx) - R1;
          gm[p] = u * u <= thr ? gxv[p] : 0.f;
        }
        acc[i][0] = __ffma2_rn(gg, make_float2(gm[0], gm[1]), acc[i][0]);
        acc[i][1] = __ffma2_rn(gg, make_float2(gm[2], gm[3]), acc[i][1]);
        acc[i][2] = __ffma2_rn(gg, make_float2(gm[4], gm[5]), acc[i][2]);
        acc[i][3] = __ffma2_rn(gg, make_float2(gm[6], gm[7]), acc[i][3]);
      } else {
        acc[i][0] = __ffma2_rn(gg, make_float2(gxv[0], gxv[1]), acc[i][0]);
        acc[i][1] = __ffma2_rn(gg, make_float2(gxv[2], gxv[3]), acc[i][1]);
        acc[i][2] = __ffma2_rn(gg, make_float2(gxv[4], gxv[5]), acc[i][2]);
        acc[i][3] = __ffma2_rn(gg, make_float2(gxv[6], gxv[7]), acc[i][3]);
      }
    }
  }
  }

// ---------------------------------------------------------------------------------------------------------------
// k_tile_lite: the light items (whole tiles of at most LITE_MAX stars, empty ones included: the planner puts them
// last, from Header::lite0 on), one CTA per item, many CTAs per SM -- with k_tile_sb, whose persistent CTAs take the
// items before lite0.  No slots and no per-block ranges: the tile's stars, sorted by corner bin exactly as a chunk of
// k_tile_sb is (stable: corner bin, then list order), are walked by every warp whose 64 x 16 region the ROI meets,
// and each lane evaluates its own 4 row and 8 column factors with the very operations of k_tile_sb's slot
// preparation (same roundings, same zero masks, same circle mask) and adds them in that order: the same per-pixel
// sums, bit for bit, as k_tile_sb (and k_tile_ws) give the tile -- only cheaper to start (the sparse-frame floor,
// DESIGN.md §9).  Same lane layout and epilogue (tile_store<true>).
// ---------------------------------------------------------------------------------------------------------------
#ifndef LITE_MINB
#define LITE_MINB 4
#endif
template <bool INTEG, bool CIRC, int OB>  // OB: output bits (0: fp32 image, 8 / 16: the fused output stage)
__global__ void __launch_bounds__(TILE_THREADS, CIRC ? 3 : LITE_MINB) k_tile_lite(const uint32_t* __restrict__ ids,
                                                                      const StarRec* __restrict__ rec, FrameParams fp,
                                                                      void* __restrict__ out_,
                                                                      const uint32_t* __restrict__ tile_off) {
  __shared__ uint32_t lkey[LITE_MAX > 0 ? LITE_MAX : 1];
  __shared__ float4 lrec[LITE_MAX > 0 ? LITE_MAX : 1];
  __shared__ uint32_t llo[LITE_MAX > 0 ? LITE_MAX : 1];
  // CTA b takes tile b if its list is light (heavy tiles are k_tile_sb's items): one load less than the item list
  const uint32_t tile = blockIdx.x;
  const uint32_t jb = __ldg(&tile_off[tile]), je = __ldg(&tile_off[tile + 1]);
  if (je - jb > (uint32_t)LITE_MAX) return;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const float sk = fp.sk;
  const int tx = (int)(tile % (uint32_t)fp.ntx), ty = (int)(tile / (uint32_t)fp.ntx);
  const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
  const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
  const int n = (int)(je - jb);  // <= LITE_MAX
  float2 acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  if (n > 0) {
    StarRec r = {};
    if (tid < n) r = rec[__ldg(&ids[jb + tid])];
    lite_chunk<INTEG, CIRC, LITE_MAX>(acc, lkey, lrec, llo, r, n, fp, X0, IY0, TWe, THe);
  }
  // the lanes with swz = 1 hold columns 4-7 of their strip in acc[i][0..1] (k_tile_sb's load order)
  if (swz) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 t0 = acc[i][0], t1 = acc[i][1];
      acc[i][0] = acc[i][2];
      acc[i][1] = acc[i][3];
      acc[i][2] = t0;
      acc[i][3] = t1;
    }
  }
  if (OB == 0) {
    tile_store<true, 0>(acc, fp, out_, Y0, X0 + 64 * wx + 8 * q, B, hq);
  } else {
    // the gray image: staged in shared memory and quantised from there (the register-resident form spills here)
    __shared__ __align__(16) float gbuf[OB ? TILE_W * TILE_H : 4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float4* d = reinterpret_cast<float4*>(gbuf + lane_row<true>(B, hq, i) * TILE_W + 64 * wx + 8 * q);
      d[0] = make_float4(acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y);
      d[1] = make_float4(acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y);
    }
    __syncthreads();
    tile_store_gray_staged(gbuf, fp, out_, Y0, X0, TWe, THe);
  }
}


// ---------------------------------------------------------------------------------------------------------------
// The sparse path (STARSIM_TILE_AUTO, catalogues of <= SPARSE_MAX stars with stars x tiles <= SPARSE_TESTS,
// R <= SB_MAXR): no binning.  k_srec writes the star records (step a1) and each star's packed tile box (the tiles its
// clipped ROI meets: at most 2 x 2); k_tile_sparse runs one CTA per tile that streams the box array in star order,
// keeps the stars whose box holds its tile -- exactly the tile's CSR list, in the same order -- and renders every
// 256 list entries as one chunk with lite_chunk (the remainder at the end), summing lists longer than SPLIT_LEN in
// segments through its own slot of the segment scratch (reading R19): the same per-pixel sums as k_tile_sb /
// k_tile_ws, bit for bit, in two launches instead of four.  starsim_get_bins after a sparse render bins the same
// arrays on demand (api.cu).
// ---------------------------------------------------------------------------------------------------------------
constexpr uint32_t SP_NONE = 0xFFFFFFFFu;
__device__ __forceinline__ uint32_t sp_box(int tx0, int ty0, int dx, int dy) {  // 8 + 9 + 1 + 1 bits
  return (uint32_t)tx0 | (uint32_t)ty0 << 8 | (uint32_t)dx << 17 | (uint32_t)dy << 18;
}

__global__ void __launch_bounds__(256) k_srec(const float* __restrict__ X, const float* __restrict__ Y,
                                              const float* __restrict__ M, int64_t n, FrameParams fp,
                                              StarRec* __restrict__ rec, uint32_t* __restrict__ box) {
  const int64_t i = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (i >= frame_n(n, fp)) return;
  int cx0, cx1, cy0, cy1;
  const StarRec r = prep_star(__ldg(&X[i]), __ldg(&Y[i]), __ldg(&M[i]), fp, cx0, cx1, cy0, cy1);
  rec[i] = r;
  uint32_t b = SP_NONE;
  if (r.lo != LO_CULLED) {
    const int tx0 = cx0 / TILE_W, ty0 = (cy0 - fp.row0) / TILE_H;
    b = sp_box(tx0, ty0, cx1 / TILE_W - tx0, (cy1 - fp.row0) / TILE_H - ty0);
  }
  box[i] = b;
}

#ifndef SP_PER_OPT
#define SP_PER_OPT 8
#endif
constexpr int SP_PER = SP_PER_OPT;                        // stars per thread and round (loads issued together)
constexpr int SP_BUF = SB_CHUNK + TILE_THREADS * SP_PER;  // pending list entries: < one chunk + one round's hits
template <bool INTEG, bool CIRC, int OB>
__global__ void __launch_bounds__(TILE_THREADS, (CIRC && INTEG) ? 2 : (CIRC || INTEG) ? 3 : LITE_MINB) k_tile_sparse(
    const StarRec* __restrict__ rec, const uint32_t* __restrict__ box, int64_t n, FrameParams fp,
    void* __restrict__ out_, float* __restrict__ seg_scratch) {
  // the pending list and the chunk arrays, and (gray output) the staged tile afterwards, share one buffer
  struct Lists {
    uint32_t lidx[SP_BUF];
    uint32_t lkey[SB_CHUNK];
    float4 lrec[SB_CHUNK];
    uint32_t llo[SB_CHUNK];
  };
  __shared__ __align__(16) unsigned char sraw[OB && sizeof(float) * TILE_W * TILE_H > sizeof(Lists)
                                                  ? sizeof(float) * TILE_W * TILE_H
                                                  : sizeof(Lists)];
  Lists& L = *reinterpret_cast<Lists*>(sraw);
  __shared__ uint32_t wcnt[TILE_WARPS];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t tile = blockIdx.x;
  const int tx = (int)(tile % (uint32_t)fp.ntx), ty = (int)(tile / (uint32_t)fp.ntx);
  const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
  const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
  n = frame_n(n, fp);
  float2 acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t pending = 0, done_chunks = 0, segs_done = 0;
  // a round: warp w takes the 32 SP_PER consecutive stars from base + 32 SP_PER w, so the hits come out in star order
  // as (warp, sub-round, lane); one block prefix over the warps places them after the pending entries
  auto render_chunk = [&](int nn) {
    StarRec r = {};
    if (tid < nn) r = rec[L.lidx[tid]];
    lite_chunk<INTEG, CIRC, SB_CHUNK>(acc, L.lkey, L.lrec, L.llo, r, nn, fp, X0, IY0, TWe, THe);
    ++done_chunks;
  };
  for (int64_t base = 0; base < n; base += (int64_t)TILE_THREADS * SP_PER) {
    uint32_t hm[SP_PER];
    uint32_t bx[SP_PER];
    uint32_t cw = 0;
    const int64_t wb = base + (int64_t)(32 * SP_PER) * warp + lane;
#pragma unroll
    for (int j = 0; j < SP_PER; ++j) bx[j] = wb + 32 * j < n ? __ldg(&box[wb + 32 * j]) : SP_NONE;
#pragma unroll
    for (int j = 0; j < SP_PER; ++j) {
      bool hit = false;
      const uint32_t b = bx[j];
      if (b != SP_NONE) {
        const int btx = (int)(b & 0xFFu), bty = (int)((b >> 8) & 0x1FFu);
        hit = tx >= btx && tx <= btx + (int)((b >> 17) & 1u) && ty >= bty && ty <= bty + (int)((b >> 18) & 1u);
      }
      hm[j] = __ballot_sync(0xffffffffu, hit);
      cw += __popc(hm[j]);
    }
    if (lane == 0) wcnt[warp] = cw;
    __syncthreads();
    uint32_t pre = 0, tot = 0;
#pragma unroll
    for (int w = 0; w < TILE_WARPS; ++w) {
      const uint32_t c = wcnt[w];
      pre += w < warp ? c : 0u;
      tot += c;
    }
    uint32_t pos = pending + pre;
#pragma unroll
    for (int j = 0; j < SP_PER; ++j) {
      if ((hm[j] >> lane) & 1u) L.lidx[pos + __popc(hm[j] & lt)] = (uint32_t)(wb + 32 * j);
      pos += __popc(hm[j]);
    }
    pending += tot;
    __syncthreads();
    // whole chunks: render them in list order, then move the remainder to the front
    uint32_t off = 0;
    while (pending - off >= (uint32_t)SB_CHUNK) {
      if (off) {  // bring the next chunk's entries to the front of the list buffer
        uint32_t v = tid < SB_CHUNK ? L.lidx[off + tid] : 0u;
        __syncthreads();
        if (tid < SB_CHUNK) L.lidx[tid] = v;
        __syncthreads();
        // (the entries after it stay where they are; off counts from the moved chunk)
        for (uint32_t k = SB_CHUNK + tid; k < pending - off; k += TILE_THREADS) L.lidx[k] = L.lidx[off + k];
        __syncthreads();
        pending -= off;
        off = 0;
      }
      render_chunk(SB_CHUNK);
      if (((done_chunks * SB_CHUNK) % SPLIT_LEN) == 0) {
        seg_flush(acc, seg_scratch, segs_done == 0);  // a full segment: more list entries may follow
        ++segs_done;
      }
      off = SB_CHUNK;
      __syncthreads();
    }
    if (off) {  // keep the remainder (< one chunk) at the front
      const uint32_t rem = pending - off;
      uint32_t v = tid < (int)rem ? L.lidx[off + tid] : 0u;
      __syncthreads();
      if ((uint32_t)tid < rem) L.lidx[tid] = v;
      pending = rem;
      __syncthreads();
    }
  }
  if (pending) render_chunk((int)pending);
  // a segment flushed right at the list's end holds the whole last segment: fold it back (the order of R19 is kept:
  // the flushed partial sums come first, the empty rest adds zeros)
  if (segs_done) seg_finish(acc, seg_scratch);
  if (swz) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 t0 = acc[i][0], t1 = acc[i][1];
      acc[i][0] = acc[i][2];
      acc[i][1] = acc[i][3];
      acc[i][2] = t0;
      acc[i][3] = t1;
    }
  }
  if (OB == 0) {
    tile_store<true, 0>(acc, fp, out_, Y0, X0 + 64 * wx + 8 * q, B, hq);
  } else {
    float* gbuf = reinterpret_cast<float*>(sraw);
    __syncthreads();  // the last chunk's walk is done with the list arrays
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float4* d = reinterpret_cast<float4*>(gbuf + lane_row<true>(B, hq, i) * TILE_W + 64 * wx + 8 * q);
      d[0] = make_float4(acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y);
      d[1] = make_float4(acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y);
    }
    __syncthreads();
    tile_store_gray_staged(gbuf, fp, out_, Y0, X0, TWe, THe);
  }
}

// every tile CTA streams every star's 4-B tile box: worth it while stars x tiles stays small (measured)
bool sparse_ok(int64_t n, int64_t ntiles) { return n <= SPARSE_MAX && n * ntiles <= SPARSE_TESTS; }

void launch_srec(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                 uint32_t* box, cudaStream_t st) {
  if (n > 0) k_srec<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(x, y, m, n, fp, rec, box);
}

void launch_tile_sparse(const StarRec* rec, const uint32_t* box, int64_t n, const FrameParams& fp, void* out,
                        float* seg_scratch, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  using KS = void (*)(const StarRec*, const uint32_t*, int64_t, FrameParams, void*, float*);
  static const KS ks[2][2][3] = {
      {{k_tile_sparse<false, false, 0>, k_tile_sparse<false, false, 8>, k_tile_sparse<false, false, 16>},
       {k_tile_sparse<false, true, 0>, k_tile_sparse<false, true, 8>, k_tile_sparse<false, true, 16>}},
      {{k_tile_sparse<true, false, 0>, k_tile_sparse<true, false, 8>, k_tile_sparse<true, false, 16>},
       {k_tile_sparse<true, true, 0>, k_tile_sparse<true, true, 8>, k_tile_sparse<true, true, 16>}}};
  const KS k = ks[fp.psf ? 1 : 0][fp.roi ? 1 : 0][fp.obits == 8 ? 1 : fp.obits == 16 ? 2 : 0];
  k<<<(unsigned)ntiles, TILE_THREADS, 0, st>>>(rec, box, n, fp, out, seg_scratch);
}

#ifdef STARSIM_SB_TIMING
extern "C" int starsim_debug_sb_timing(double* out6, int reset) {
  unsigned long long h[6];
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(h, g_sb_prof, sizeof(h));
  for (int i = 0; i < 6; ++i) out6[i] = (double)h[i];
  if (reset) {
    unsigned long long z[6] = {0, 0, 0, 0, 0, 0};
    cudaMemcpyToSymbol(g_sb_prof, z, sizeof(z));
  }
  return 0;
}
#endif

void init_tile_sb_kernel() {
  cudaFuncSetAttribute(k_tile_sb<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(SbSmem));
  cudaFuncSetAttribute(k_tile_sb<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(SbSmem));
  cudaFuncSetAttribute(k_tile_sb<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(SbSmem));
  cudaFuncSetAttribute(k_tile_sb<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(SbSmem));
}

void launch_tile_sb(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                    const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                    cudaStream_t st, float* seg_scratch, const uint32_t* tile_off) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  const int64_t grid =
      std::min<int64_t>(ntiles + part_cap, (int64_t)(fp.roi ? SB_MINB_CIRC : SB_MINB) * num_sms);  // persistent CTAs
  auto* k = fp.psf ? (fp.roi ? k_tile_sb<true, true> : k_tile_sb<true, false>)
                   : (fp.roi ? k_tile_sb<false, true> : k_tile_sb<false, false>);
  k<<<(unsigned)grid, TILE_THREADS, sizeof(SbSmem), st>>>(ids, rec, fp, out, items, split_tab, part_buf, done, hdr,
                                                          seg_scratch);
  if (fp.lite) {  // the light items: one CTA each (at most one per tile; the surplus CTAs return at once)
    using KL = void (*)(const uint32_t*, const StarRec*, FrameParams, void*, const uint32_t*);
    static const KL kls[2][2][3] = {
        {{k_tile_lite<false, false, 0>, k_tile_lite<false, false, 8>, k_tile_lite<false, false, 16>},
         {k_tile_lite<false, true, 0>, k_tile_lite<false, true, 8>, k_tile_lite<false, true, 16>}},
        {{k_tile_lite<true, false, 0>, k_tile_lite<true, false, 8>, k_tile_lite<true, false, 16>},
         {k_tile_lite<true, true, 0>, k_tile_lite<true, true, 8>, k_tile_lite<true, true, 16>}}};
    const KL kl = kls[fp.psf ? 1 : 0][fp.roi ? 1 : 0][fp.obits == 8 ? 1 : fp.obits == 16 ? 2 : 0];
    kl<<<(unsigned)ntiles, TILE_THREADS, 0, st>>>(ids, rec, fp, out, tile_off);
  }
}

}  // namespace starsim
