// Warp-specialised tile accumulation -- the default kernel for R <= SB_MAXR.
//
// Same work, order of summation, lane layout and epilogue as k_tile_sb (tile_sb.cu): every chunk of <= WS_CHUNK
// stars of a tile's list is sorted by ROI corner bin, each star's row / column profiles are evaluated once into
// fixed shared-memory slots, and every lane group walks the two contiguous ranges of the sorted order that can reach
// its 8 x 16 block, accumulating [s' gy(r)] * gx(c) (Eqs. 2-3) in fp32 registers.  What differs is who does what:
//
//   producer warps (WS_PROD = WS_CHUNK / 32, one star per thread): fetch work items, gather the star records, sort
//           the chunk by corner bin, write its profiles and bin starts into stage s of a WS_NSTAGE-deep ring, and
//           arrive on full[s].  They synchronise among themselves with named barrier 1 only.
//   consumer warps (8, warp (wx, B) owns the tile's 64 x 16 block at columns 64 wx, rows 16 B): wait on full[s],
//           walk stage s, arrive on empty[s], and at the last chunk of an item write the tile (named barrier 2 for
//           the heavy-tile part reduction).
//
// k_tile_sb runs the two roles one after the other in the same warps, with three CTA barriers per chunk: every warp
// waits for the slowest walk and for warp 0's bin scan, and the MUFU-heavy profile phase never overlaps the
// FMA/shared-memory-heavy walk.  Here the roles overlap and a consumer warp waits only when the producers are behind
// (or, WS_NSTAGE - 1 chunks ahead, for the slowest consumer).  The per-pixel summation order is the same as
// k_tile_sb's (range 1 then range 2 of every chunk, chunks in list order): the two kernels give bitwise-identical
// images (tested).
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "tile_common.cuh"

namespace starsim {

constexpr int WS_NSK = NSTRIPS + 1;                  // strip keys 0..16 (0: ROI enters over the left edge)
constexpr int WS_NBIN = (NBANDS + 1) * WS_NSK;       // 85 corner bins, band-major (band key 0: over the top edge)
static_assert(WS_NBIN < 128, "bin keys (and the no-bin key WS_NBIN) fit 7 bits");
#ifndef WS_CHUNK_OPT
#define WS_CHUNK_OPT 256
#endif
#ifndef WS_CTAS_OPT
#define WS_CTAS_OPT 1
#endif
constexpr int WS_CHUNK = WS_CHUNK_OPT;               // stars per chunk
constexpr int WS_CTAS = WS_CTAS_OPT;                 // CTAs per SM
constexpr int WS_PROD = WS_CHUNK / 32;               // producer warps
constexpr int WS_CONS = 8;                           // consumer warps
#ifndef WS_PGROUPS
#define WS_PGROUPS 1                                 // producer groups: group g produces the chunks c = g mod WS_PGROUPS
#endif
constexpr int WS_THREADS = 32 * (WS_PGROUPS * WS_PROD + WS_CONS);
#ifndef WS_NSTAGE_OPT
#define WS_NSTAGE_OPT 2
#endif
#ifndef WS_RSTAGE_OPT
#define WS_RSTAGE_OPT SPLIT_LEN
#endif
#ifndef WS_WALK_UNROLL
#define WS_WALK_UNROLL 2
#endif
constexpr int WS_UNROLL = WS_WALK_UNROLL;              // walk steps per loop iteration (pairs of even/odd)
constexpr int WS_NSTAGE = WS_NSTAGE_OPT;              // depth of the chunk ring (chunk c in stage c mod WS_NSTAGE)
constexpr uint32_t WS_ZJ = WS_CHUNK;                 // the all-zero slot of every stage
constexpr uint32_t WS_LAST = 1u, WS_STOP = 2u, WS_SEGEND = 4u;  // chunk flags (SEGEND: a SPLIT_LEN segment ends)
static_assert(SPLIT_LEN % WS_CHUNK == 0, "segments are whole chunks");
constexpr int WS_RSTAGE = WS_RSTAGE_OPT;             // star records of a work item staged in shared memory
constexpr int WS_RPT = WS_RSTAGE / WS_CHUNK;         // ... per producer thread

struct WsStage {
  float gy[(WS_CHUNK + 1) * 32];  // sorted star j: two 16-float band slots, slot k at j*32 + ((j ^ k) & 1) * 16
  float gx[(WS_CHUNK + 1) * 32];  // sorted star j: ring of four 8-float strip slots, strip Q at j*32 + (Q & 3) * 8
  uint32_t binstart[WS_NBIN + 3]; // exclusive scan of the bin totals (padded: stages stay 16-B aligned)
  uint32_t tile, aux, flags, pad;
};
static_assert(sizeof(WsStage) % 16 == 0, "stages hold float4 slots");

struct WsSmem {
  unsigned long long full[WS_NSTAGE], empty[WS_NSTAGE];
  WsStage st[WS_NSTAGE];
  StarRec rst[WS_PGROUPS][2][WS_RSTAGE];  // per group: records of the current and the next work item (thread-private)
  uint32_t hist[WS_PGROUPS][WS_PROD][WS_NBIN];
  uint32_t binoff[WS_PGROUPS][WS_PROD][WS_NBIN];
  int s_last;
};

#ifdef STARSIM_WS_TIMING
// per-phase SM cycles summed over warps (debug builds only): producer record+sort / barrier 1 / empty wait / scan +
// barrier 2 / profiles, producer warp-chunks, consumer full wait / walk / epilogue, consumer warp-chunks
__device__ unsigned long long g_ws_prof[10];
#define WS_T(v) const long long v = clock64()
#define WS_ACC(k, d) if ((threadIdx.x & 31) == 0) atomicAdd(&g_ws_prof[k], (unsigned long long)(d))
#else
#define WS_T(v)
#define WS_ACC(k, d)
#endif

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t parity) {
  const uint32_t a = smem_u32(b);
  uint32_t ok;
  do {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!ok);
}
// named barriers: 1 and 3 for the two producer groups, 2 for the consumers (acc_barrier)
__device__ __forceinline__ void prod_barrier(int g) {
  asm volatile("bar.sync %0, %1;" ::"r"(1 + 2 * g), "n"(WS_CHUNK) : "memory");
}

__device__ __forceinline__ uint32_t item_chunks(const WorkItem& w) {
  return w.je > w.jb ? (w.je - w.jb + WS_CHUNK - 1) / WS_CHUNK : 1u;  // an empty item still sends one (empty) chunk
}
// The ids of the stars of work item w that producer thread pt of group g reads: star e = pt + WS_CHUNK k sits in
// chunk k, which group g produces iff (cb + k) % WS_PGROUPS == g (cb: the CTA's index of the item's first chunk).
template <bool PRE>
__device__ __forceinline__ void load_ids(uint32_t (&id)[WS_RPT], const uint32_t* __restrict__ ids, const WorkItem& w,
                                         uint32_t cb, int g, int pt) {
  if (PRE) return;  // presorted records are read in list order: no ids
  const uint32_t len = w.je - w.jb;
#pragma unroll
  for (int k = 0; k < WS_RPT; ++k) {
    const uint32_t e = (uint32_t)pt + (uint32_t)(k * WS_CHUNK);
    id[k] = e < len && (cb + (uint32_t)k) % WS_PGROUPS == (uint32_t)g ? __ldg(&ids[w.jb + e]) : 0u;
  }
}
// ... and their records, copied into the group's record stage at the same places: thread pt is the only reader of
// its slots, so cp.async + wait_all needs no barrier.
template <bool PRE>
__device__ __forceinline__ void stage_records(StarRec* dst, const StarRec* __restrict__ rec, const uint32_t (&id)[WS_RPT],
                                              const WorkItem& w, uint32_t cb, int g, int pt) {
  const uint32_t len = w.je - w.jb;
#pragma unroll
  for (int k = 0; k < WS_RPT; ++k) {
    const uint32_t e = (uint32_t)pt + (uint32_t)(k * WS_CHUNK);
    // PRE: rec is the presorted record array (list order within each chunk sorted by corner bin, k_chsort)
    const StarRec* src = PRE ? rec + w.jb + e : rec + id[k];
    if (e < len && (cb + (uint32_t)k) % WS_PGROUPS == (uint32_t)g)
      asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst + e)), "l"(src) : "memory");
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
}

// PRE: the chunks come presorted by k_chsort (records in sorted order, bin starts per chunk): the producers skip the
// sort, its two barriers and the record gather through the ids, and only evaluate the profiles (sorted star j = pt).
template <bool INTEG, bool PRE>
__device__ __forceinline__ void ws_producer(WsSmem& S, const uint32_t* __restrict__ ids,
                                            const StarRec* __restrict__ rec, const FrameParams& fp,
                                            const WorkItem* __restrict__ items, uint32_t nitems,
                                            const uint16_t* __restrict__ cbin) {
  const int pq = threadIdx.x - 32 * WS_CONS;
  const int g = pq / WS_CHUNK, pt = pq % WS_CHUNK, lane = pt & 31, pw = pt >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const float sk = fp.sk;
  uint32_t (&hist)[WS_PROD][WS_NBIN] = S.hist[g];
  uint32_t (&binoff)[WS_PROD][WS_NBIN] = S.binoff[g];
  // Static round-robin over the work items (parts of heavy tiles first): the CTA's item and chunk sequence is known
  // ahead, so item i + 1's records are gathered while item i is processed, item i + 2's ids loaded and item i + 3's
  // WorkItem.  Every group walks the whole sequence; group g produces the chunks c = g mod WS_PGROUPS.
  const uint32_t G = gridDim.x;
  const WorkItem none = {0u, 0u, 0u, 0u};
  uint32_t it = blockIdx.x, cb = 0, p = 0;
  WorkItem wi = it < nitems ? items[it] : none;
  WorkItem wn = it + G < nitems ? items[it + G] : none;
  WorkItem wnn = it + 2 * G < nitems ? items[it + 2 * G] : none;
  uint32_t idn[WS_RPT];
  load_ids<PRE>(idn, ids, wi, 0u, g, pt);
  stage_records<PRE>(S.rst[g][0], rec, idn, wi, 0u, g, pt);
  load_ids<PRE>(idn, ids, wn, item_chunks(wi), g, pt);
  while (it < nitems) {
    const uint32_t nch = item_chunks(wi), cbn = cb + nch;
    asm volatile("cp.async.wait_all;" ::: "memory");
    stage_records<PRE>(S.rst[g][p ^ 1u], rec, idn, wn, cbn, g, pt);
    load_ids<PRE>(idn, ids, wnn, cbn + item_chunks(wn), g, pt);
    const WorkItem w3 = it + 3 * G < nitems ? items[it + 3 * G] : none;
    const StarRec* rs = S.rst[g][p];
    const int tx = (int)(wi.tile % (uint32_t)fp.ntx), ty = (int)(wi.tile / (uint32_t)fp.ntx);
    const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
    const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
    for (uint32_t k = ((uint32_t)g + WS_PGROUPS - cb % WS_PGROUPS) % WS_PGROUPS; k < nch; k += WS_PGROUPS) {
      const uint32_t c = cb + k, s = c % WS_NSTAGE, ph = (c / WS_NSTAGE) & 1u;
      WsStage& T = S.st[s];
      const uint32_t base = wi.jb + k * WS_CHUNK;
      const bool last = k + 1 == nch;
      const int nvalid = base < wi.je ? (int)min((uint32_t)WS_CHUNK, wi.je - base) : 0;
      // ---- corner bin of star base + pt (its ROI clipped to the tile starts in band r0/16, strip c0/8)
      WS_T(p0);
      StarRec r = {};
      if (pt < nvalid) {
        const uint32_t off = base - wi.jb + (uint32_t)pt;
        r = off < (uint32_t)WS_RSTAGE ? rs[off] : (PRE ? rec[base + pt] : rec[__ldg(&ids[base + pt])]);
      }
      int c0 = 0, c1 = -1, r0 = 0, r1 = -1;
      uint32_t key = WS_NBIN;
      if (pt < nvalid) {
        const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
        c0 = max(lx, 0);
        c1 = min(lx + fp.R - 1, TWe - 1);
        r0 = max(ly, 0);
        r1 = min(ly + fp.R - 1, THe - 1);
        if (c0 <= c1 && r0 <= r1)
          key = (uint32_t)((ly < 0 ? 0 : 1 + (r0 >> 4)) * WS_NSK + (lx < 0 ? 0 : 1 + (c0 >> 3)));
      }
      // PRE: this chunk's bin starts (k_chsort), loaded ahead of the stage wait
      uint32_t cbv = 0u;
      if (PRE && pt <= WS_NBIN && nvalid > 0)
        cbv = __ldg(&cbin[(size_t)((base >> 8) + wi.tile) * (WS_NBIN + 1) + pt]);
      // stars of the warp with the same key (what __match_any_sync gives, from 7 ballots: MATCH.ANY costs a loop over
      // the distinct keys of the warp)
      uint32_t peers = 0xffffffffu, rank = 0u;
      if (!PRE) {
#pragma unroll
      for (int b = 0; b < 7; ++b) {
        const uint32_t kb = (key >> b) & 1u;
        const uint32_t m = __ballot_sync(0xffffffffu, kb);
        peers &= kb ? m : ~m;
      }
      rank = __popc(peers & lt);
      // hist was last read by producer warp 0's scan of the previous chunk, before its second producer barrier
      hist[pw][lane] = 0u;
      hist[pw][lane + 32] = 0u;
      if (lane < WS_NBIN - 64) hist[pw][lane + 64] = 0u;
      __syncwarp();
      if (rank == 0 && key < WS_NBIN) hist[pw][key] = __popc(peers);
      }
      WS_T(p1);
      if (!PRE) prod_barrier(g);
      WS_T(p2);
      // stage s is free once every consumer warp has walked the chunk it held WS_NSTAGE chunks ago
      mbar_wait(&S.empty[s], ph ^ 1u);
      WS_T(p3);
      if (PRE) {
        if (pt <= WS_NBIN) T.binstart[pt] = cbv;
      } else if (pw == 0) {
        uint32_t tot[3], sum = 0;
#pragma unroll
        for (int h = 0; h < 3; ++h) {
          const int bin = 3 * lane + h;
          uint32_t cw[WS_PROD];
#pragma unroll
          for (int w = 0; w < WS_PROD; ++w) cw[w] = bin < WS_NBIN ? hist[w][bin] : 0u;
          uint32_t run = 0;
#pragma unroll
          for (int w = 0; w < WS_PROD; ++w) {
            if (bin < WS_NBIN) binoff[w][bin] = run;
            run += cw[w];
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
          if (bin <= WS_NBIN) T.binstart[bin] = ex;
          ex += tot[h];
        }
      }
      if (!PRE) prod_barrier(g);
      WS_T(p4);
      // ---- the star's profiles at its sorted place j (exactly k_tile_sb's values and slots)
#ifdef WS_NOPROF
      if (false) {
#else
      if (key < WS_NBIN) {
#endif
        const uint32_t j = PRE ? (uint32_t)pt : T.binstart[key] + binoff[pw][key] + rank;
        const float yr = r.y - (float)IY0, xr = r.x - (float)X0;  // exact
        const float2 sk2 = make_float2(sk, sk), s2 = make_float2(r.s, r.s);
        const int b0 = (int)(key / WS_NSK) - 1, q0 = (int)(key % WS_NSK) - 1;
        const int ra0 = r0 - 16 * b0, rb0 = r1 - 16 * b0;
        const uint32_t m0 = (0xFFFFFFFFu >> (31 - min(rb0, 31))) & (0xFFFFFFFFu << ra0);
        const float bf0 = (float)(16 * b0) - yr;  // exact
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const int u = (c + lane) & 7;
          const int hh = u >> 1, k = (u ^ (int)j) & 1;
          const int w = 4 * k + hh;
          float4* dst = reinterpret_cast<float4*>(&T.gy[j * 32 + (u & 1) * 16 + hh * 4]);
          const uint32_t m = m0 >> (4 * w);
          const float bf = bf0 + (float)(4 * w);  // exact
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
          const int rel = 8 * Qs;
          const int lo = max(c0 - rel, 0), hi = min(c1 - rel, 7);
          const uint32_t m = hi >= lo ? ((0xFFu >> (7 - hi)) & (0xFFu << lo)) : 0u;
          const float bf = (float)rel - xr;  // exact
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
          float* gs = &T.gx[j * 32 + (Qs & 3) * 8];
          const int sw = ((Qs >> 2) & 1) * 4;
          *reinterpret_cast<float4*>(gs + sw) = make_float4(v[0], v[1], v[2], v[3]);
          *reinterpret_cast<float4*>(gs + (sw ^ 4)) = make_float4(v[4], v[5], v[6], v[7]);
        }
      }
      if (pt == 0) {
        T.tile = wi.tile;
        T.aux = wi.aux;
        T.flags = last ? WS_LAST : (((k + 1) % (SPLIT_LEN / WS_CHUNK)) == 0 ? WS_SEGEND : 0u);
      }
      mbar_arrive(&S.full[s]);
#ifdef STARSIM_WS_TIMING
      {
        WS_T(p5);
        WS_ACC(0, p1 - p0);
        WS_ACC(1, p2 - p1);
        WS_ACC(2, p3 - p2);
        WS_ACC(3, p4 - p3);
        WS_ACC(4, p5 - p4);
        WS_ACC(5, 1);
      }
#endif
    }
    it += G;
    cb = cbn;
    wi = wn;
    wn = wnn;
    wnn = w3;
    p ^= 1u;
  }
  // no more items: the group that owns chunk cb sends the stop chunk that releases the consumers
  if (cb % WS_PGROUPS == (uint32_t)g) {
    const uint32_t s = cb % WS_NSTAGE;
    mbar_wait(&S.empty[s], ((cb / WS_NSTAGE) & 1u) ^ 1u);
    if (pt == 0) S.st[s].flags = WS_STOP;
    mbar_arrive(&S.full[s]);
  }
}

__device__ __forceinline__ void ws_consumer(WsSmem& S, const FrameParams& fp, void* __restrict__ out_,
                                            const uint2* __restrict__ split_tab, float* __restrict__ part_buf,
                                            uint32_t* __restrict__ done, float* __restrict__ seg_scratch) {
  uint32_t segs_done = 0;  // SPLIT_LEN segments of the current item already in the scratch (tile_common.cuh)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base0 = smem_u32(S.st[0].gy) + 16u * hq;
  const uint32_t gx_base0 = smem_u32(S.st[0].gx) + 32u * (Q & 3);
  constexpr uint32_t STB = sizeof(WsStage);
  const int sklo = max(Q - 1, 0);
  float2 acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  for (uint32_t chunk = 0;; ++chunk) {
    const uint32_t s = chunk % WS_NSTAGE, ph = (chunk / WS_NSTAGE) & 1u;
    const WsStage& T = S.st[s];
    WS_T(q0);
    mbar_wait(&S.full[s], ph);
    WS_T(q1);
    const uint32_t flags = T.flags;
    if (flags & WS_STOP) break;
    const uint32_t tile = T.tile, aux = T.aux;
    const uint32_t gy_base = gy_base0 + s * STB, gx_base = gx_base0 + s * STB;
    const uint32_t s1r = T.binstart[B * WS_NSK + sklo], e1r = T.binstart[B * WS_NSK + Q + 2];
    const uint32_t s2r = T.binstart[(B + 1) * WS_NSK + sklo], e2r = T.binstart[(B + 1) * WS_NSK + Q + 2];
    const uint32_t len1 = e1r - s1r, L = len1 + (e2r - s2r);
    const uint32_t steps = __reduce_max_sync(0xffffffffu, L);
    const uint32_t c1v = s1r, c2v = s2r - len1;
    const uint32_t e1 = (c1v + 1u) & 1u, e2 = c2v & 1u;
    const uint32_t g1e = gy_base + c1v * 128u + e1 * 64u, g1o = gy_base + c1v * 128u + (e1 ^ 1u) * 64u;
    const uint32_t g2e = gy_base + c2v * 128u + e2 * 64u, g2o = gy_base + c2v * 128u + (e2 ^ 1u) * 64u;
    const uint32_t x1 = gx_base + c1v * 128u, x2 = gx_base + c2v * 128u;
    const uint32_t gz = gy_base + WS_ZJ * 128u, xz = gx_base + WS_ZJ * 128u;
    auto step = [&](uint32_t t, bool odd) {
      const bool in1 = t < len1, in = t < L;
      uint32_t ga = (in1 ? (odd ? g1o : g1e) : (odd ? g2o : g2e)) + t * 128u;
      uint32_t xa = (in1 ? x1 : x2) + t * 128u;
      ga = in ? ga : gz;
      xa = in ? xa : xz;
      float4 g, a, c;
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g.x), "=f"(g.y), "=f"(g.z), "=f"(g.w) : "r"(ga));
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w) : "r"(xa));
      asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];"
                   : "=f"(c.x), "=f"(c.y), "=f"(c.z), "=f"(c.w)
                   : "r"(xa + 16u));
      const float gi[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 gg = make_float2(gi[i], gi[i]);
        acc[i][0] = __ffma2_rn(gg, make_float2(a.x, a.y), acc[i][0]);
        acc[i][1] = __ffma2_rn(gg, make_float2(a.z, a.w), acc[i][1]);
        acc[i][2] = __ffma2_rn(gg, make_float2(c.x, c.y), acc[i][2]);
        acc[i][3] = __ffma2_rn(gg, make_float2(c.z, c.w), acc[i][3]);
      }
    };
    uint32_t st = 0;
#ifdef WS_NOWALK
    st = steps;
#endif
#pragma unroll WS_UNROLL
    for (; st + 1 < steps; st += 2) {
      step(st, false);
      step(st + 1, true);
    }
    if (st < steps) step(st, false);
    mbar_arrive(&S.empty[s]);
    WS_T(q2);
    WS_ACC(6, q1 - q0);
    WS_ACC(7, q2 - q1);
    WS_ACC(9, 1);
    if (flags & WS_SEGEND) {
      seg_flush(acc, seg_scratch, segs_done == 0);
      ++segs_done;
      continue;
    }
    if (!(flags & WS_LAST)) continue;
    // ---- the item's last chunk: write the tile (or this part of a split heavy tile)
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
    if (tile_reduce_parts<true, 32 * WS_CONS>(acc, wi, split_tab, part_buf, done, B, wx, q, hq, &S.s_last))
      tile_store<true>(acc, fp, out_, ty * TILE_H, tx * TILE_W + 64 * wx + 8 * q, B, hq);
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
    WS_T(q3);
    WS_ACC(8, q3 - q2);
  }
}

template <bool INTEG, bool PRE>
__global__ void __launch_bounds__(WS_THREADS, WS_CTAS) k_tile_ws(const uint32_t* __restrict__ ids,
                                                           const StarRec* __restrict__ rec, FrameParams fp,
                                                           void* __restrict__ out_, const WorkItem* __restrict__ items,
                                                           const uint2* __restrict__ split_tab,
                                                           float* __restrict__ part_buf, uint32_t* __restrict__ done,
                                                           Header* hdr, float* __restrict__ seg_scratch,
                                                           const uint16_t* __restrict__ cbin) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  WsSmem& S = *reinterpret_cast<WsSmem*>(smem_raw);
  const int tid = threadIdx.x;
  if (tid < WS_NSTAGE) {
    mbar_init(&S.full[tid], WS_CHUNK);       // every producer thread arrives once per chunk
    mbar_init(&S.empty[tid], 32 * WS_CONS);  // every consumer thread arrives once per chunk
  }
  for (int i = tid; i < WS_NSTAGE * 32; i += WS_THREADS) {
    S.st[i / 32].gy[WS_ZJ * 32 + (i & 31)] = 0.f;
    S.st[i / 32].gx[WS_ZJ * 32 + (i & 31)] = 0.f;
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  const uint32_t nitems = __ldcg(&hdr->nitems);
  if (tid >= 32 * WS_CONS)
    ws_producer<INTEG, PRE>(S, ids, rec, fp, items, nitems, cbin);
  else
    ws_consumer(S, fp, out_, split_tab, part_buf, done, seg_scratch);
}


// ---------------------------------------------------------------------------------------------------------------
// k_chsort: the producers' per-chunk sort, done ahead for the whole frame.  One warp per (work item, chunk k mod 4):
// the chunk's <= 256 stars (list positions base + 32 r + lane, r = 0..7) get their corner bin exactly as a producer
// computes it, the chunk's bin starts go to cbin[(base >> 8) + tile] (86 u16: bins 0..84 and the total), and every
// record is written to srec[base + its stable rank by (bin, list position)] -- the order k_tile_sb / k_tile_ws walk
// (reading R12): k_tile_ws<PRE> then reads each chunk's records contiguously and only evaluates profiles.  The slot
// index (base >> 8) + tile is unique: chunks of one tile start 256 apart, and a later tile's first chunk starts at a
// later list position.
// ---------------------------------------------------------------------------------------------------------------
constexpr int CHS_WARPS = 8;
__global__ void __launch_bounds__(32 * CHS_WARPS) k_chsort(const uint32_t* __restrict__ ids,
                                                           const StarRec* __restrict__ rec, FrameParams fp,
                                                           const WorkItem* __restrict__ items,
                                                           const Header* __restrict__ hdr, StarRec* __restrict__ srec,
                                                           uint16_t* __restrict__ cbin) {
  static_assert(WS_CHUNK == 256, "k_chsort sorts 256-star chunks (8 rounds of 32)");
  __shared__ uint32_t cnt[CHS_WARPS][WS_NBIN + 1];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const uint32_t gw = blockIdx.x * CHS_WARPS + (uint32_t)w;
  const uint32_t item = gw >> 2;
  if (item >= __ldcg(&hdr->nitems)) return;
  const WorkItem wi = items[item];
  const int tx = (int)(wi.tile % (uint32_t)fp.ntx), ty = (int)(wi.tile / (uint32_t)fp.ntx);
  const int X0 = tx * TILE_W, Y0 = ty * TILE_H, IY0 = fp.row0 + Y0;
  const int TWe = min(TILE_W, fp.W - X0), THe = min(TILE_H, fp.rows - Y0);
  uint32_t* c = cnt[w];
  for (uint32_t base = wi.jb + (gw & 3u) * WS_CHUNK; base < wi.je; base += 4u * WS_CHUNK) {
    const uint32_t n = min((uint32_t)WS_CHUNK, wi.je - base);
    StarRec r[8];
    uint32_t key[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const uint32_t e = (uint32_t)(32 * k + lane);
      r[k] = e < n ? rec[__ldg(&ids[base + e])] : StarRec{0.f, 0.f, 0.f, LO_CULLED};
    }
    for (int b = lane; b <= WS_NBIN; b += 32) c[b] = 0u;
    __syncwarp();
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      key[k] = WS_NBIN;
      if ((uint32_t)(32 * k + lane) < n) {
        const int lx = lo_x_of(r[k].lo) - X0, ly = lo_y_of(r[k].lo) - IY0;
        const int c0 = max(lx, 0), c1 = min(lx + fp.R - 1, TWe - 1);
        const int r0 = max(ly, 0), r1 = min(ly + fp.R - 1, THe - 1);
        if (c0 <= c1 && r0 <= r1)
          key[k] = (uint32_t)((ly < 0 ? 0 : 1 + (r0 >> 4)) * WS_NSK + (lx < 0 ? 0 : 1 + (c0 >> 3)));
        atomicAdd(&c[key[k]], 1u);  // bin WS_NBIN collects the stars that miss the tile (placed last)
      }
    }
    __syncwarp();
    // exclusive scan of the 86 bin counts (3 per lane) -> bin starts; the chunk's row of cbin
    uint32_t v[3], sum = 0;
#pragma unroll
    for (int h = 0; h < 3; ++h) {
      const int bin = 3 * lane + h;
      v[h] = bin <= WS_NBIN ? c[bin] : 0u;
      sum += v[h];
    }
    uint32_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += u;
    }
    uint32_t ex = incl - sum;
    uint16_t* row = cbin + (size_t)((base >> 8) + wi.tile) * (WS_NBIN + 1);
    __syncwarp();
#pragma unroll
    for (int h = 0; h < 3; ++h) {
      const int bin = 3 * lane + h;
      if (bin <= WS_NBIN) {
        c[bin] = ex;                // running position of the bin
        row[bin] = (uint16_t)ex;    // bin starts; row[WS_NBIN] = the stars that meet the tile
      }
      ex += v[h];
    }
    __syncwarp();
    // stable placement, round by round (list order): rank among the round's equal keys, then the bin's cursor
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const bool in = (uint32_t)(32 * k + lane) < n;
      const uint32_t mi = __ballot_sync(0xffffffffu, in);
      uint32_t peers = mi;  // the round's lanes with the same key
#pragma unroll
      for (int b = 0; b < 7; ++b) {
        const uint32_t kb = (key[k] >> b) & 1u;
        const uint32_t m = __ballot_sync(0xffffffffu, kb && in);
        peers &= kb ? m : ~m;
      }
      const uint32_t rank = __popc(peers & lt);
      const uint32_t pos = in ? c[key[k]] + rank : 0u;
      __syncwarp();
      if (in && rank == 0) c[key[k]] += __popc(peers);
      __syncwarp();
      if (in) srec[base + pos] = r[k];
    }
    __syncwarp();
  }
}

size_t chsort_slots(int64_t ntiles, int64_t pmax) { return (size_t)(pmax / WS_CHUNK + ntiles + 2); }
size_t chsort_words16() { return WS_NBIN + 1; }

void launch_chsort(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, const WorkItem* items, int part_cap,
                   const Header* hdr, StarRec* srec, uint16_t* cbin, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  const int64_t warps = 4 * (ntiles + part_cap);
  k_chsort<<<(unsigned)((warps + CHS_WARPS - 1) / CHS_WARPS), 32 * CHS_WARPS, 0, st>>>(ids, rec, fp, items, hdr, srec,
                                                                                      cbin);
}

#ifdef STARSIM_WS_TIMING
extern "C" int starsim_debug_ws_timing(double* out10, int reset) {
  unsigned long long h[10];
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(h, g_ws_prof, sizeof(h));
  for (int i = 0; i < 10; ++i) out10[i] = (double)h[i];
  if (reset) {
    unsigned long long z[10] = {};
    cudaMemcpyToSymbol(g_ws_prof, z, sizeof(z));
  }
  return 0;
}
#endif

void init_tile_ws_kernel() {
  cudaFuncSetAttribute(k_tile_ws<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WsSmem));
  cudaFuncSetAttribute(k_tile_ws<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WsSmem));
  cudaFuncSetAttribute(k_tile_ws<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WsSmem));
  cudaFuncSetAttribute(k_tile_ws<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(WsSmem));
}

void launch_tile_ws(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                    const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                    cudaStream_t st, float* seg_scratch, const StarRec* srec, const uint16_t* cbin) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)WS_CTAS * num_sms);  // persistent CTAs
  // srec != nullptr: the chunks were presorted by k_chsort (srec, cbin)
  auto* k = srec ? (fp.psf ? k_tile_ws<true, true> : k_tile_ws<false, true>)
                 : (fp.psf ? k_tile_ws<true, false> : k_tile_ws<false, false>);
  k<<<(unsigned)grid, WS_THREADS, sizeof(WsSmem), st>>>(ids, srec ? srec : rec, fp, out, items, split_tab, part_buf,
                                                         done, hdr, seg_scratch, cbin);
}

}  // namespace starsim
