// k_tile_wide: tile accumulation with sorted corner bins for wide ROIs, WIDE_MINR <= R <= WIDE_MAXR (27 <= R <= 65,
// wide_ok(): the wide end of the C4 ROI sweep, BASELINE configs[3]; Table III's ROI-side axis) --
// SURVEY.md §8a step a5, Eqs. 2-3.  Measured and discussed in DESIGN.md §9b.
//
// The design of k_tile_sb (tile_sb.cu) generalised from "an ROI spans <= 2 bands x 3 strips" to <= KB bands x
// KS = 2 KB - 1 strips (KB = 3, 4, 5 for R <= 33, 49, 65).  Same tile geometry, lane layout (warp (wx, B) owns the
// 64 x 16 block at columns 64 wx, rows 16 B; lane group q = lane / 4 the 8-column strip Q = 8 wx + q; lane hq = lane % 4
// the rows 16 B + 4 hq .. + 3), accumulators, epilogue, heavy-tile parts and R19 segments.  Per chunk of <= 128 stars
// of the tile's list:
//
//   sort   (thread = star): the star's UNCLIPPED ROI origin (ly, lx), tile-relative, lies in band b0 = ly >> 4 and
//          strip q0 = lx >> 3 (b0 >= -(KB-1), q0 >= -(KS-1): an ROI coming in over the top or left edge keeps its
//          true extent, so it is a candidate only for the blocks it can reach) -- its corner bin (NBK x NSK bins,
//          band-major).  A stable counting sort by corner bin gives sorted index j.  The stars that can touch the
//          block (B, Q) are exactly the corner bins of bands B - k (k = 0 .. KB-1) and strips Q - KS + 1 .. Q: KB
//          contiguous ranges of the sorted order, range k reading band slot k.  No per-block lists (k_tile builds one
//          per (band, strip) block: its preparation costs more than its walk at wide R).
//   prep   (two threads per star: threads 0-127 the row profile, 128-255 the column profile): s' gy on the KB bands
//          b0 .. b0 + KB - 1 (16-float band slots) and gx on the strips q0 .. q0 + KS - 1 (8-float strip slots in a
//          ring of RS = 8 or 16 indexed by Q mod RS), zero outside the ROI, one MUFU.EX2 per value inside it (a quad
//          or strip the ROI misses is stored as zeros without evaluating it); bands and strips outside the tile are
//          never read and not stored.
//   accumulate (warp): lane group q walks its KB ranges one after the other (a divergent loop: the warp runs its
//          longest range, the other groups idle): a step is three LDS.128 (4 row factors, 8 column factors) and 16
//          FFMA2.
//
// Bank conflicts: strip Q's slot sits at ring position Q mod RS (slot stride RS x 32 B, a multiple of 128 B) with its
// two 16-B halves swapped when bit 2 of Q is set, so the 8 lane groups of a warp always hit 8 distinct bank quads;
// the row slot of a star is an odd number of 64-B band slots, so the band slots of consecutive stars alternate 64-B
// halves of the 128-B bank line.
//
// Heavy tiles: parts and segments of FrameParams::split = WIDE_SPLIT (256) stars (reading R19), so a heavy tile's
// R^2-FMA stars spread over several CTAs.
//
// Summation order of a pixel: per chunk (in list order; lists longer than fp.split in R19 segments), range k = 0 ..
// KB-1, each in sorted order (corner bin, then list order): deterministic and a function of the tile's own list only,
// so tile-aligned band renders are bitwise the frame's pixels (reading R12).  No atomics on the image.
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "tile_common.cuh"
#include "tile_wide.cuh"

namespace starsim {

namespace {

constexpr int WD_CHUNK = 128;                     // stars per chunk (two prep threads per star)
#ifndef WD_MINB_SMALL_OPT
#define WD_MINB_SMALL_OPT 2
#endif
// CTAs per SM: 2 for KB = 5 (128 registers, <= 112 KB shared memory); KB = 3, 4 (R <= 49) fit WD_MINB_SMALL_OPT
template <int KB>
struct WdMinB {
  static constexpr int value = KB >= 5 ? 2 : WD_MINB_SMALL_OPT;
};
constexpr int WD_SW = 4;                          // warps that own a star in the sort (threads 0..127)
static_assert(SPLIT_LEN % WD_CHUNK == 0 && WIDE_SPLIT % WD_CHUNK == 0, "segments are whole chunks");
static_assert(WD_CHUNK * 2 == TILE_THREADS, "two prep threads per star");

template <int KB>
struct WideSmem {
  float gy[WD_CHUNK * WideGeom<KB>::SYF];  // sorted star j: band slot k at j * SYF + 16 k
  float gx[WD_CHUNK * WideGeom<KB>::SXF];  // sorted star j: strip Q at j * SXF + 8 * (Q mod RS)
  uint32_t hist[WD_SW][WideGeom<KB>::NBIN];      // per sorting warp: stars of each corner bin, then (scanned in
                                                 // place) the stars of the bin in the warps before
  uint32_t binstart[WideGeom<KB>::PER * 32 + 1]; // exclusive scan of the bin totals (+ the total)
  uint32_t lo2[WD_CHUNK];                    // CIRC: sorted star j's ROI origin (int16 x | int16 y << 16)
};


}  // namespace

template <int KB, bool INTEG, bool CIRC>
__global__ void __launch_bounds__(TILE_THREADS, WdMinB<KB>::value) k_tile_wide(const uint32_t* __restrict__ ids,
                                                                     const StarRec* __restrict__ rec, FrameParams fp,
                                                                     void* __restrict__ out_,
                                                                     const WorkItem* __restrict__ items,
                                                                     const uint2* __restrict__ split_tab,
                                                                     float* __restrict__ part_buf,
                                                                     uint32_t* __restrict__ done, Header* hdr,
                                                                     float* __restrict__ seg_scratch) {
  using G = WideGeom<KB>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  WideSmem<KB>& S = *reinterpret_cast<WideSmem<KB>*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int sid = tid & (WD_CHUNK - 1);   // the chunk star this thread sorts and prepares
  const bool colhalf = tid >= WD_CHUNK;   // prep: false = row profile, true = column profile
  const uint32_t lt = (1u << lane) - 1u;

  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base = (uint32_t)__cvta_generic_to_shared(S.gy) + 16u * hq;
  const uint32_t gx_base = (uint32_t)__cvta_generic_to_shared(S.gx) + 32u * (uint32_t)(Q & (G::RS - 1));
  __shared__ int s_last;
  __shared__ uint32_t s_next;

  // persistent CTAs (WdMinB per SM): item blockIdx.x first, then items from the counter the planner zeroed (the
  // parts of heavy tiles come first); the next item's records are fetched while this one is walked (as k_tile_sb)
  const uint32_t nitems = __ldcg(&hdr->nitems);
  uint32_t item = blockIdx.x;
  if (item >= nitems) return;
  WorkItem wi = items[item];
  StarRec rnext = {};
  if (wi.jb + sid < wi.je) rnext = rec[ids[wi.jb + sid]];
  for (;;) {
    uint32_t nxt = 0;
    if (tid == 0) nxt = atomicAdd(&hdr->next_item, 1u) + gridDim.x;
    uint32_t item_n = 0xFFFFFFFFu, nid0 = 0;
    WorkItem wn = {0u, 0u, 0u, 0u};
    bool fetched = false;
    const int tx = (int)(wi.tile % (uint32_t)fp.ntx), ty = (int)(wi.tile / (uint32_t)fp.ntx);
    const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
    const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
    float2 acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);

    const uint32_t j1 = wi.je;
    uint32_t segs_done = 0;
    for (uint32_t base = wi.jb; base < j1; base += WD_CHUNK) {
      // ======================= sort: star sid of the chunk (both halves hold it; warps 0-3 count it)
      const int nvalid = (int)min((uint32_t)WD_CHUNK, j1 - base);
      const StarRec r = rnext;
      int c0 = 0, c1 = -1, r0 = 0, r1 = -1;
      uint32_t key = G::NBIN, lo2 = 0u;
      if (sid < nvalid) {
        const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
        lo2 = (uint32_t)(lx & 0xFFFF) | (uint32_t)ly << 16;
        c0 = max(lx, 0);
        c1 = min(lx + fp.R - 1, TWe - 1);
        r0 = max(ly, 0);
        r1 = min(ly + fp.R - 1, THe - 1);
        key = wide_key<KB>(lx, ly, c0, c1, r0, r1);
      }
      // warps w and w + 4 hold the same stars in the same lanes: the same peers and ranks
      const uint32_t peers = key_peers(key);
      const uint32_t rank = __popc(peers & lt);
      if (warp < WD_SW) {
        // (the previous chunk's readers of hist -- warp 0's scan -- finished before its second barrier)
#pragma unroll
        for (int h = 0; h < G::PER; ++h)
          if (lane + 32 * h < G::NBIN) S.hist[warp][lane + 32 * h] = 0u;
        __syncwarp();
        if (rank == 0 && key < G::NBIN) S.hist[warp][key] = __popc(peers);
      }
      const uint32_t nb = base + WD_CHUNK;
      const uint32_t nid = nb + sid < j1 ? __ldg(&ids[nb + sid]) : 0u;
      __syncthreads();
      if (warp == 0) wide_scan<KB, WD_SW>(S.hist, S.binstart, lane);
      __syncthreads();
      // ======================= prep: the star's profiles at its sorted place j
      if (key < G::NBIN) {
        const uint32_t j = S.binstart[key] + S.hist[warp & (WD_SW - 1)][key] + rank;
        SS_CHECK(j < S.binstart[G::NBIN] && S.binstart[G::NBIN] <= (uint32_t)nvalid);
        // the unclipped ROI origin's band and strip (bands b0 .. b0 + KB - 1, strips q0 .. q0 + KS - 1 hold it)
        const int b0 = (int)(key / G::NSK) - (KB - 1), q0 = (int)(key % G::NSK) - (G::KS - 1);
        if (!colhalf) {
          if (CIRC) S.lo2[j] = lo2;
          wide_rows<KB, INTEG>(&S.gy[j * G::SYF], b0, r0, r1, r.y - (float)IY0, r.s, fp, lane);
        } else {
          wide_cols<KB, INTEG>(&S.gx[j * G::SXF], q0, c0, c1, r.x - (float)X0, fp);
        }
      }
      const bool first = base == wi.jb, last = nb >= j1;
      if (first && tid == 0) s_next = nxt;
      __syncthreads();

      if (first) {
        fetched = true;
        item_n = s_next;
        if (item_n < nitems) wn = items[item_n];
      }
      if (!last) {
        if (nb + sid < j1) rnext = rec[nid];
      } else if (item_n < nitems && wn.jb + sid < wn.je) {
        nid0 = __ldg(&ids[wn.jb + sid]);
      }
      // ======================= accumulate: lane group q walks its KB ranges
      wide_walk<KB, CIRC>(acc, S.binstart, gy_base, gx_base, S.lo2, B, Q, hq, swz, fp);
      if ((base + WD_CHUNK - wi.jb) % (uint32_t)fp.split == 0 && base + WD_CHUNK < j1) {
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
        if (wn.jb + sid < wn.je) nid0 = __ldg(&ids[wn.jb + sid]);
      }
    }
    if (item_n >= nitems) break;
    rnext = StarRec{};
    if (wn.jb + sid < wn.je) rnext = rec[nid0];
    wi = wn;
    item = item_n;
  }  // work loop
}

// ---------------------------------------------------------------------------------------------------------------
// k_tile_wws: the same chunks, slots, ranges and per-pixel order as k_tile_wide (the two give bitwise-identical
// images), warp-specialised as k_tile_ws is for R <= 17: 4 producer warps (one star per thread) sort each chunk and
// write its profiles into stage s of an NS-deep ring, then arrive on full[s]; 8 consumer warps (the accumulators,
// threads 0..255) wait on full[s], walk, arrive on empty[s] and write the tile after an item's last chunk.  At wide R
// the walk dominates: the producers' sort, scan and profiles overlap it instead of sitting between CTA barriers, and
// a consumer warp waits only for the producers or, NS - 1 chunks ahead, for the slowest consumer.  One CTA per SM,
// work items in static round-robin order (parts of heavy tiles first).
// ---------------------------------------------------------------------------------------------------------------
namespace {
#ifndef WW_PROD_OPT
#define WW_PROD_OPT 4
#endif
#ifndef WW_MINB_OPT
#define WW_MINB_OPT 1
#endif
constexpr int WW_PROD = WW_PROD_OPT, WW_CONS = 8;  // producer warps (one star per thread), consumer warps
constexpr int WW_CHUNK = 32 * WW_PROD;
constexpr int WW_MINB = WW_MINB_OPT;               // CTAs per SM
constexpr int WW_THREADS = 32 * (WW_PROD + WW_CONS);
constexpr uint32_t WW_LAST = 1u, WW_STOP = 2u, WW_SEGEND = 4u;
static_assert(WW_CHUNK == 32 * WW_PROD && SPLIT_LEN % WW_CHUNK == 0, "one producer thread per star, whole segments");

template <int KB>
struct WwStage {
  float gy[WW_CHUNK * WideGeom<KB>::SYF];
  float gx[WW_CHUNK * WideGeom<KB>::SXF];
  uint32_t binstart[(WideGeom<KB>::PER * 32 + 4) & ~3];
  uint32_t lo2[WW_CHUNK];
  uint32_t tile, aux, flags, pad;
};
template <int KB>
__host__ __device__ constexpr int ww_ns() {
  return WW_MINB * (3 * sizeof(WwStage<KB>) + sizeof(uint32_t) * WW_PROD * WideGeom<KB>::NBIN + 1200) <= 228 * 1024
             ? 3 : 2;
}
template <int KB>
struct WwSmem {
  unsigned long long full[4], empty[4];
  WwStage<KB> st[ww_ns<KB>()];
  uint32_t hist[WW_PROD][WideGeom<KB>::NBIN];
  int s_last;
};
static_assert(WW_MINB * (sizeof(WwSmem<5>) + 1024) <= 228 * 1024, "WW_MINB CTAs per SM fit");

__device__ __forceinline__ uint32_t ww_smem(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void ww_mbar_init(unsigned long long* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(ww_smem(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void ww_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(ww_smem(b)) : "memory");
}
__device__ __forceinline__ void ww_wait(unsigned long long* b, uint32_t parity) {
  const uint32_t a = ww_smem(b);
  uint32_t ok;
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!ok);
}
__device__ __forceinline__ void ww_prod_barrier() { asm volatile("bar.sync 1, %0;" ::"n"(32 * WW_PROD) : "memory"); }
}  // namespace

template <int KB, bool INTEG, bool CIRC>
__device__ __forceinline__ void wws_producer(WwSmem<KB>& S, const uint32_t* __restrict__ ids,
                                             const StarRec* __restrict__ rec, const FrameParams& fp,
                                             const WorkItem* __restrict__ items, uint32_t nitems) {
  using G = WideGeom<KB>;
  constexpr int NS = ww_ns<KB>();
  const int pt = threadIdx.x - 32 * WW_CONS, lane = pt & 31, pw = pt >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const uint32_t GS = gridDim.x;
  const WorkItem none = {0u, 0u, 0u, 0u};
  uint32_t it = blockIdx.x, c = 0;
  WorkItem wi = it < nitems ? items[it] : none;
  StarRec rcur = {};
  if (wi.jb + (uint32_t)pt < wi.je) rcur = rec[__ldg(&ids[wi.jb + pt])];
  while (it < nitems) {
    const uint32_t nch = wi.je > wi.jb ? (wi.je - wi.jb + WW_CHUNK - 1) / WW_CHUNK : 1u;  // an empty item: 1 chunk
    const bool more = it + GS < nitems;
    const WorkItem wn = more ? items[it + GS] : none;
    const int tx = (int)(wi.tile % (uint32_t)fp.ntx), ty = (int)(wi.tile / (uint32_t)fp.ntx);
    const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
    const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
    for (uint32_t k = 0; k < nch; ++k, ++c) {
      const uint32_t s = c % NS, ph = (c / NS) & 1u;
      WwStage<KB>& T = S.st[s];
      const uint32_t base = wi.jb + k * WW_CHUNK;
      const StarRec r = rcur;
      const bool valid = base + (uint32_t)pt < wi.je;
      {  // the next chunk's record (this item's or the next item's first), one chunk ahead
        const uint32_t nb = k + 1 < nch ? base + WW_CHUNK : wn.jb, ne = k + 1 < nch ? wi.je : wn.je;
        rcur = StarRec{};
        if (nb + (uint32_t)pt < ne) rcur = rec[__ldg(&ids[nb + pt])];
      }
      int c0 = 0, c1 = -1, r0 = 0, r1 = -1;
      uint32_t key = G::NBIN, lo2 = 0u;
      if (valid) {
        const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
        lo2 = (uint32_t)(lx & 0xFFFF) | (uint32_t)ly << 16;
        c0 = max(lx, 0);
        c1 = min(lx + fp.R - 1, TWe - 1);
        r0 = max(ly, 0);
        r1 = min(ly + fp.R - 1, THe - 1);
        key = wide_key<KB>(lx, ly, c0, c1, r0, r1);
      }
      const uint32_t peers = key_peers(key);
      const uint32_t rank = __popc(peers & lt);
      // (hist[pw] was last read by this warp's prep and by producer warp 0's scan, before the last producer barrier)
#pragma unroll
      for (int h = 0; h < G::PER; ++h)
        if (lane + 32 * h < G::NBIN) S.hist[pw][lane + 32 * h] = 0u;
      __syncwarp();
      if (rank == 0 && key < G::NBIN) S.hist[pw][key] = __popc(peers);
      ww_prod_barrier();
      // stage s is free once every consumer thread has walked the chunk it held NS chunks ago
      ww_wait(&S.empty[s], ph ^ 1u);
      if (pw == 0) wide_scan<KB, WW_PROD>(S.hist, T.binstart, lane);
      ww_prod_barrier();
      if (key < G::NBIN) {
        const uint32_t j = T.binstart[key] + S.hist[pw][key] + rank;
        SS_CHECK(j < (uint32_t)WW_CHUNK && j < T.binstart[G::NBIN]);
        const int b0 = (int)(key / G::NSK) - (KB - 1), q0 = (int)(key % G::NSK) - (G::KS - 1);
        if (CIRC) T.lo2[j] = lo2;
        wide_rows<KB, INTEG>(&T.gy[j * G::SYF], b0, r0, r1, r.y - (float)IY0, r.s, fp, lane);
        wide_cols<KB, INTEG>(&T.gx[j * G::SXF], q0, c0, c1, r.x - (float)X0, fp);
      }
      if (pt == 0) {
        T.tile = wi.tile;
        T.aux = wi.aux;
        T.flags = k + 1 == nch ? WW_LAST : (((k + 1) % ((uint32_t)fp.split / WW_CHUNK)) == 0 ? WW_SEGEND : 0u);
      }
      ww_arrive(&S.full[s]);
    }
    it += GS;
    wi = wn;
  }
  const uint32_t s = c % NS;  // the stop chunk releases the consumers
  ww_wait(&S.empty[s], ((c / NS) & 1u) ^ 1u);
  if (pt == 0) S.st[s].flags = WW_STOP;
  ww_arrive(&S.full[s]);
}

template <int KB, bool CIRC>
__device__ __forceinline__ void wws_consumer(WwSmem<KB>& S, const FrameParams& fp, void* __restrict__ out_,
                                             const uint2* __restrict__ split_tab, float* __restrict__ part_buf,
                                             uint32_t* __restrict__ done, float* __restrict__ seg_scratch) {
  using G = WideGeom<KB>;
  constexpr int NS = ww_ns<KB>();
  constexpr uint32_t STB = sizeof(WwStage<KB>);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base0 = ww_smem(S.st[0].gy) + 16u * hq;
  const uint32_t gx_base0 = ww_smem(S.st[0].gx) + 32u * (uint32_t)(Q & (G::RS - 1));
  uint32_t segs_done = 0;
  float2 acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  for (uint32_t c = 0;; ++c) {
    const uint32_t s = c % NS, ph = (c / NS) & 1u;
    const WwStage<KB>& T = S.st[s];
    ww_wait(&S.full[s], ph);
    const uint32_t flags = T.flags;
    if (flags & WW_STOP) break;
    const uint32_t tile = T.tile, aux = T.aux;
    wide_walk<KB, CIRC>(acc, T.binstart, gy_base0 + s * STB, gx_base0 + s * STB, T.lo2, B, Q, hq, swz, fp);
    ww_arrive(&S.empty[s]);
    if (flags & WW_SEGEND) {
      seg_flush(acc, seg_scratch, segs_done == 0);
      ++segs_done;
      continue;
    }
    if (!(flags & WW_LAST)) continue;
    if (segs_done) {
      seg_finish(acc, seg_scratch);
      segs_done = 0;
    }
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
    const WorkItem wi = {tile, 0u, 0u, aux};
    const int tx = (int)(tile % (uint32_t)fp.ntx), ty = (int)(tile / (uint32_t)fp.ntx);
    if (tile_reduce_parts<true, 32 * WW_CONS>(acc, wi, split_tab, part_buf, done, B, wx, q, hq, &S.s_last))
      tile_store<true>(acc, fp, out_, ty * TILE_H, tx * TILE_W + 64 * wx + 8 * q, B, hq);
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  }
}

template <int KB, bool INTEG, bool CIRC>
__global__ void __launch_bounds__(WW_THREADS, WW_MINB) k_tile_wws(const uint32_t* __restrict__ ids,
                                                            const StarRec* __restrict__ rec, FrameParams fp,
                                                            void* __restrict__ out_, const WorkItem* __restrict__ items,
                                                            const uint2* __restrict__ split_tab,
                                                            float* __restrict__ part_buf, uint32_t* __restrict__ done,
                                                            Header* hdr, float* __restrict__ seg_scratch) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  WwSmem<KB>& S = *reinterpret_cast<WwSmem<KB>*>(smem_raw);
  const int tid = threadIdx.x;
  if (tid < ww_ns<KB>()) {
    ww_mbar_init(&S.full[tid], 32 * WW_PROD);  // every producer thread arrives once per chunk
    ww_mbar_init(&S.empty[tid], 32 * WW_CONS);  // every consumer thread arrives once per chunk
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  const uint32_t nitems = __ldcg(&hdr->nitems);
  if (tid >= 32 * WW_CONS)
    wws_producer<KB, INTEG, CIRC>(S, ids, rec, fp, items, nitems);
  else
    wws_consumer<KB, CIRC>(S, fp, out_, split_tab, part_buf, done, seg_scratch);
}

namespace {
using KW = void (*)(const uint32_t*, const StarRec*, FrameParams, void*, const WorkItem*, const uint2*, float*,
                    uint32_t*, Header*, float*);
template <int KB>
struct WideTab {
  static constexpr KW k[2][2] = {{k_tile_wide<KB, false, false>, k_tile_wide<KB, false, true>},
                                 {k_tile_wide<KB, true, false>, k_tile_wide<KB, true, true>}};
  static constexpr KW w[2][2] = {{k_tile_wws<KB, false, false>, k_tile_wws<KB, false, true>},
                                 {k_tile_wws<KB, true, false>, k_tile_wws<KB, true, true>}};
};
static_assert(WideGeom<5>::MAXR == WIDE_MAXR, "KB = 5 covers the widest ROI");
static_assert(2 * (sizeof(WideSmem<5>) + 1024 + 64) <= 228 * 1024, "two CTAs per SM fit");
int wide_kb(int R) { return R <= WideGeom<3>::MAXR ? 3 : R <= WideGeom<4>::MAXR ? 4 : 5; }
}  // namespace

// from WIDE_MINR on (measured on the clustered C4 sweep: at R = 21 k_tile's lists are faster, from R = 31 on this
// kernel, 1.3-1.5x at R = 47-63)
#ifndef WIDE_MINR_OPT
#define WIDE_MINR_OPT 27
#endif
bool wide_ok(int R) { return R >= WIDE_MINR_OPT && R > SB_MAXR && R <= WIDE_MAXR; }

void init_tile_wide_kernel() {
  for (int a = 0; a < 2; ++a)
    for (int b = 0; b < 2; ++b) {
      cudaFuncSetAttribute(WideTab<3>::w[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WwSmem<3>));
      cudaFuncSetAttribute(WideTab<4>::w[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WwSmem<4>));
      cudaFuncSetAttribute(WideTab<5>::w[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WwSmem<5>));
      cudaFuncSetAttribute(WideTab<3>::k[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WideSmem<3>));
      cudaFuncSetAttribute(WideTab<4>::k[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WideSmem<4>));
      cudaFuncSetAttribute(WideTab<5>::k[a][b], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WideSmem<5>));
    }
}

void launch_tile_wide(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                      const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                      cudaStream_t st, float* seg_scratch) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  const int kb = wide_kb(fp.R), a = fp.psf ? 1 : 0, b = fp.roi ? 1 : 0;
  if (fp.tile_impl != 2) {  // every mode but STARSIM_TILE_SB: the warp-specialised kernel, one CTA per SM
    const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)WW_MINB * num_sms);
    const KW k = kb == 3 ? WideTab<3>::w[a][b] : kb == 4 ? WideTab<4>::w[a][b] : WideTab<5>::w[a][b];
    const size_t smem = kb == 3 ? sizeof(WwSmem<3>) : kb == 4 ? sizeof(WwSmem<4>) : sizeof(WwSmem<5>);
    k<<<(unsigned)grid, WW_THREADS, smem, st>>>(ids, rec, fp, out, items, split_tab, part_buf, done, hdr, seg_scratch);
    return;
  }
  const int minb = kb >= 5 ? WdMinB<5>::value : WdMinB<3>::value;
  const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)minb * num_sms);  // persistent CTAs
  const KW k = kb == 3 ? WideTab<3>::k[a][b] : kb == 4 ? WideTab<4>::k[a][b] : WideTab<5>::k[a][b];
  const size_t smem = kb == 3 ? sizeof(WideSmem<3>) : kb == 4 ? sizeof(WideSmem<4>) : sizeof(WideSmem<5>);
  k<<<(unsigned)grid, TILE_THREADS, smem, st>>>(ids, rec, fp, out, items, split_tab, part_buf, done, hdr, seg_scratch);
}

}  // namespace starsim
