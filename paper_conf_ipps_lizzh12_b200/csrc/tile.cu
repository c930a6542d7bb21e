// Tile accumulation (DESIGN.md §Path step a5, §The tile kernel).
//
// One CTA renders one 128 x 64 tile from its star list (CSR from the binning, star-index order), in chunks of up to
// 256 stars.  Eq. 2 is separable: a star's contribution at pixel (r, c) is [s' gy(r)] * gx(c) with
// gy(r) = exp(-(r-y)^2 / 2 sigma^2), gx(c) = exp(-(c-x)^2 / 2 sigma^2) and s' = A 2.512^-m / (2 pi sigma^2)
// (Eq. 1 and the normaliser of Eq. 2, evaluated in fp64 by k_prep).
//
// Layout.  Warp (wx, B) owns the 64 x 16 block at tile columns 64 wx, rows 16 B ("band" B); inside it, lane group
// q = lane/4 owns the 8-column strip Q = 8 wx + q and lane hq = lane%4 the rows 16 B + hq + 4 i (i = 0..3): 4 rows x
// 8 columns = 32 fp32 accumulators per lane, updated with FFMA2 (gy broadcast x a column pair).
//
// Per chunk:
//   prep (thread = star): clip the star's ROI to the tile; evaluate its row profile s' gy on the ROI rows and its
//     column profile gx on the ROI columns (one MUFU.EX2 each, the ROI's R + R values, not R^2) into shared-memory
//     slots: a 16-float "band slot" per (star, band) in the [hq][i] order the lanes read, an 8-float "strip slot"
//     per (star, strip) placed at index rank * 16 + Q with its two halves XOR-swizzled by bit 2 of Q -- so the 8 lane
//     groups of a warp always hit 8 distinct bank groups; and one entry (band slot, strip slot) in the list of every
//     (band, strip) block the ROI overlaps.  Ranks and list positions come from warp ballots + a cross-warp prefix,
//     so every list is in star order.  A chunk is cut short (deterministically) when a capacity would overflow.
//   accumulate (warp): lane group q walks the list of its block (B, Q); step t loads entry t (one LDS), the row
//     profile (one LDS.128: rows hq + 4i), the column profile (two LDS.128: 8 columns) and issues 16 FFMA2.  Groups
//     whose list is shorter pad with an all-zero strip slot.
// The per-pixel order of the fp32 additions is star order within the tile's list -- deterministic, and the same for a
// tile whatever the band decomposition.  The tile is written once, coalesced (each lane stores 2 x 16 B per row).
// No atomics on the image.
#include <algorithm>
#include <cstddef>

#include "common.cuh"
#include "launch.h"
#include "tile_common.cuh"

namespace starsim {

struct TileSmem {
  float gy[GY_CAP * 16];                 // band slots [slot][hq][i]
  float gx[(RCAP * NSTRIPS + 1) * 8];    // strip slots [rank*16 + Q][half ^ swz(Q)][4]; last slot = zeros
  uint32_t ent[LCAP * NBANDS * NSTRIPS]; // entries [t][B][Q] = band slot | strip slot << 16
  uint32_t bb[TILE_WARPS][NBANDS];       // per-warp ballots: stars overlapping band B
  uint32_t sb[TILE_WARPS][NSTRIPS];      // per-warp ballots: stars overlapping strip Q
  uint32_t lpre[NBANDS * NSTRIPS][TILE_WARPS];  // per (B,Q): entries of the warps before
  uint32_t rpre[NSTRIPS][TILE_WARPS];           // per Q: strip slots of the warps before
  uint32_t wsum[TILE_WARPS];
  float4 py[CHUNK];                      // per star: (y - IY0, s', r0 | r1 << 8, ROI origin lx | ly << 16 (CIRC))
  float2 px[CHUNK];                      // per star: (x - X0, c0 | c1 << 8)
  uint16_t gyown[GY_CAP];                // band slot -> star | band << 8
  uint32_t gxown[GX_PAIRS];              // (star, strip) pair j -> strip slot | star << 16
  StarRec rn[CHUNK];                     // per thread: its star record of the next chunk (cp.async, one chunk ahead)
  int ns, ngy, ngx;
};

// thread tid's record of the chunk starting at list position jb -> S.rn[tid], asynchronously (no registers held
// across the accumulation; the thread alone reads its slot, after cp.async.wait_all)
__device__ __forceinline__ void prefetch_rec(StarRec* slot, const StarRec* __restrict__ rec, uint32_t id) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((uint32_t)__cvta_generic_to_shared(slot)),
               "l"(rec + id)
               : "memory");
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}

static_assert(sizeof(float) * (GY_CAP * 16 + (RCAP * NSTRIPS + 1) * 8) >= sizeof(float) * TILE_W * TILE_H &&
                  offsetof(TileSmem, gx) == sizeof(float) * GY_CAP * 16,
              "the gray epilogue stages the tile in gy + gx");

constexpr uint32_t ZERO_GX = RCAP * NSTRIPS;
constexpr uint32_t ZERO_ENT = ZERO_GX * 32u << 16;  // gy byte offset 0, all-zero strip slot

// ---------------------------------------------------------------------------------------------------------------
// k_tile: one CTA per work item (item = blockIdx.x; parts first, so the heavy work starts first).  A whole tile is written to `out`
// directly; a part writes its 128 x 64 partial to part_buf, and the last part to finish (per-tile counter) sums the
// parts in part order -- a fixed order, so the image stays deterministic.
// ---------------------------------------------------------------------------------------------------------------
// INTEG: the pixel-integrated PSF (NEXT-2) instead of the paper's point-sampled Eq. 2; GRAY: the fused output stage
// (u8 / u16 image) instead of the fp32 image; CIRC: the pixel-circle ROI (NEXT-3, reading R21) -- the walk masks each
// of the lane's 4 x 8 pixels by the integer disc test against the star's ROI origin (looked up through its band slot),
// 2 CTAs per SM for the extra registers.  k_tile serves the circle for R > SB_MAXR (k_tile_sb below).
// CTAs per SM: 2 (128 registers) -- measured 1.2-1.35x faster than 3 at 80 registers on the clustered C4 frames at
// R = 21 / 31 / 63 (profiles/r2_ktile_ab.txt), and spill-free
#ifndef TILE_MINB_OPT
#define TILE_MINB_OPT 2
#endif
template <bool INTEG, bool GRAY, bool CIRC>
__global__ void __launch_bounds__(TILE_THREADS, CIRC ? 2 : TILE_MINB_OPT) k_tile(const uint32_t* __restrict__ ids,
                                                          const StarRec* __restrict__ rec, FrameParams fp,
                                                          void* __restrict__ out_, const WorkItem* __restrict__ items,
                                                          const uint2* __restrict__ split_tab,
                                                          float* __restrict__ part_buf, uint32_t* __restrict__ done,
                                                          Header* hdr, float* __restrict__ seg_scratch) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  TileSmem& S = *reinterpret_cast<TileSmem*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  // exp(-d^2 / 2 sigma^2) = 2^(-(d * sk)^2), sk = sqrt(log2(e) / (2 sigma^2)).  d = pixel - centre is formed exactly
  // (tile-relative integer minus the tile-relative centre, both exact in fp32) before the one scaling rounding.
  const float sk = fp.sk;

  // accumulate-phase identity of this lane
  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base = (uint32_t)__cvta_generic_to_shared(S.gy) + 16u * hq;
  const uint32_t gxa_base = (uint32_t)__cvta_generic_to_shared(S.gx) + 16u * swz;
  const uint32_t gxb_base = (uint32_t)__cvta_generic_to_shared(S.gx) + 16u * (swz ^ 1);
  __shared__ int s_last;
  if (tid < 8) S.gx[ZERO_GX * 8 + tid] = 0.f;

  // persistent CTAs: item blockIdx.x first, then items from the counter the planner zeroed
  // (the item count and an item's fields are re-read where needed rather than held across the accumulation:
  // registers are the limit at 3 CTAs per SM)
  for (uint32_t item = blockIdx.x; item < ld_volatile_u32(&hdr->nitems);) {
  const WorkItem wi = items[item];
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
  uint32_t segs_done = 0;  // SPLIT_LEN segments of this item already in the scratch (tile_common.cuh)
  // this thread's star record of the current chunk, loaded one chunk ahead (its latency hides behind the
  // accumulation of the previous chunk)
#ifdef KT_REG_PREFETCH
  StarRec rnext = {};
  if (wi.jb + tid < j1) rnext = rec[ids[wi.jb + tid]];
#else
  if (wi.jb + tid < j1) prefetch_rec(&S.rn[tid], rec, ids[wi.jb + tid]);
#endif
  for (uint32_t base = wi.jb; base < j1;) {
    // ======================= prep: thread = star (base + tid)
    // chunks never cross a SPLIT_LEN segment boundary of the list (segments are summed like the parts of a split tile)
    const uint32_t seg_end = min(j1, wi.jb + ((base - wi.jb) / (uint32_t)fp.split + 1u) * (uint32_t)fp.split);
    const int nvalid = (int)min((uint32_t)CHUNK, seg_end - base);
    const bool valid = tid < nvalid;
    StarRec r = {};
#ifdef KT_REG_PREFETCH
    r = rnext;
#else
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    if (valid) r = S.rn[tid];
#endif
    int c0 = 0, c1 = -1, r0 = 0, r1 = -1;
    if (valid) {
      const int lx = lo_x_of(r.lo) - X0, ly = lo_y_of(r.lo) - IY0;
      c0 = max(lx, 0);
      c1 = min(lx + fp.R - 1, TWe - 1);
      r0 = max(ly, 0);
      r1 = min(ly + fp.R - 1, THe - 1);
    }
    const int b0 = r0 >> 4, b1 = r1 >> 4, q0 = c0 >> 3, q1 = c1 >> 3;  // empty ranges when !valid
    const int ngy = valid ? b1 - b0 + 1 : 0, ngx = valid ? q1 - q0 + 1 : 0;
    // No barrier here: this phase writes only S.bb, S.sb, S.wsum and S.ns, which the previous chunk stopped reading
    // before its last barrier; the slot and list buffers are rewritten only after the next barrier, which every
    // warp reaches after finishing its accumulation of the previous chunk.
    if (tid == 0) S.ns = CHUNK;
    {
      uint32_t bbv = 0, sbv = 0;
#pragma unroll
      for (int k = 0; k < NBANDS; ++k) {
        const uint32_t m = __ballot_sync(0xffffffffu, b0 <= k && k <= b1);
        if (lane == k) bbv = m;
      }
#pragma unroll
      for (int k = 0; k < NSTRIPS; ++k) {
        const uint32_t m = __ballot_sync(0xffffffffu, q0 <= k && k <= q1);
        if (lane == k) sbv = m;
      }
      if (lane < NBANDS) S.bb[warp][lane] = bbv;
      if (lane < NSTRIPS) S.sb[warp][lane] = sbv;
    }
    // band-slot and (star, strip)-pair scans in star order (packed: ngy | ngx << 16)
    const uint32_t pk = (uint32_t)ngy | ((uint32_t)ngx << 16);
    uint32_t incl = pk;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    if (lane == 31) S.wsum[warp] = incl;
    __syncthreads();
    if (tid < NBANDS * NSTRIPS) {
      const int pb = tid >> 4, pq = tid & 15;
      uint32_t run = 0;
#pragma unroll
      for (int w = 0; w < TILE_WARPS; ++w) {
        S.lpre[tid][w] = run;
        run += __popc(S.bb[w][pb] & S.sb[w][pq]);
      }
    } else if (tid < NBANDS * NSTRIPS + NSTRIPS) {
      const int pq = tid - NBANDS * NSTRIPS;
      uint32_t run = 0;
#pragma unroll
      for (int w = 0; w < TILE_WARPS; ++w) {
        S.rpre[pq][w] = run;
        run += __popc(S.sb[w][pq]);
      }
    }
    uint32_t excl = incl - pk, ptot = 0;
#pragma unroll
    for (int w = 0; w < TILE_WARPS; ++w) {
      const uint32_t u = S.wsum[w];
      if (w < warp) excl += u;
      ptot += u;
    }
    const uint32_t gyb = excl & 0xFFFFu, gxb = excl >> 16;
    __syncthreads();
    // slots, list entries and the capacity check in one pass: a star whose slot or list position would overflow
    // ends the chunk (its own writes land beyond the lengths used below and are ignored / overwritten)
    if (valid) {
      bool fits = gyb + (uint32_t)ngy <= (uint32_t)GY_CAP && gxb + (uint32_t)ngx <= (uint32_t)GX_PAIRS;
      uint32_t j = gxb;
      for (int k = q0; k <= q1 && fits; ++k, ++j) {
        const uint32_t sbk = S.sb[warp][k];
        const uint32_t rk = S.rpre[k][warp] + __popc(sbk & lt);
        fits = rk < (uint32_t)RCAP;
        const uint32_t slot = rk * NSTRIPS + k;
        if (fits) S.gxown[j] = slot | ((uint32_t)tid << 16);
        for (int b = b0; b <= b1 && fits; ++b) {
          const uint32_t pos = S.lpre[b * NSTRIPS + k][warp] + __popc(S.bb[warp][b] & sbk & lt);
          fits = pos < (uint32_t)LCAP;
          if (fits) S.ent[(pos * NBANDS + b) * NSTRIPS + k] = (gyb + (uint32_t)(b - b0)) * 64u | (slot * 32u << 16);
        }
      }
      if (fits) {
        for (int b = b0; b <= b1; ++b) S.gyown[gyb + b - b0] = (uint16_t)(tid | (b << 8));
      } else {
        atomicMin(&S.ns, tid);
      }
      S.py[tid] = make_float4(r.y - (float)IY0, r.s, __int_as_float(r0 | (r1 << 8)),
                              __uint_as_float((uint32_t)((lo_x_of(r.lo) - X0) & 0xFFFF) |
                                              (uint32_t)(lo_y_of(r.lo) - IY0) << 16));
      S.px[tid] = make_float2(r.x - (float)X0, __int_as_float(c0 | (c1 << 8)));
    }
    __syncthreads();
    const int ns = min(S.ns, nvalid);
    // next chunk's star id now (its record is requested just before the accumulation)
    const uint32_t nb = base + (uint32_t)ns;
    const uint32_t nid = nb + tid < j1 ? __ldg(&ids[nb + tid]) : 0u;
    // slot totals of the chunk: the block totals, unless the chunk was cut short (rare: one more barrier)
    int ngy_tot = (int)(ptot & 0xFFFFu), ngx_tot = (int)(ptot >> 16);
    if (ns < nvalid) {
      if (tid == ns - 1) {
        S.ngy = (int)(gyb + ngy);
        S.ngx = (int)(gxb + ngx);
      }
      __syncthreads();
      ngy_tot = S.ngy;
      ngx_tot = S.ngx;
    }
    // profiles: thread = 8 values.  Band slot (row profile s' gy, [hq][i] = row 16 b + hq + 4 i): one thread per half
    // slot (hq = 2h, 2h+1); strip slot (column profile gx, columns 8 k .. 8 k + 7, halves swizzled): one thread per
    // slot.  d = (pixel - centre) is exact before the scaling; values outside the ROI are 0 (unsigned range test).
    // FADD2/FMUL2 pairs, one MUFU.EX2 per value.
    {
      const float2 sk2 = make_float2(sk, sk);
      const int ngh = ngy_tot * 2;
      for (int g = tid; g < ngh; g += TILE_THREADS) {
        const int k = g >> 1, hh = g & 1;
        const uint32_t own = S.gyown[k];
        const float4 pp = S.py[own & 0xFFu];
        const int rel = 16 * (int)(own >> 8) + 2 * hh;            // first row of this half slot (tile-relative)
        const int prr = __float_as_int(pp.z);
        const uint32_t u0 = (uint32_t)(rel - (prr & 0xFF)), span = (uint32_t)((prr >> 8) - (prr & 0xFF));
        const float bf = (float)rel - pp.x;                         // exact
        const float2 b2 = make_float2(bf, bf), s2 = make_float2(pp.y, pp.y);
        float2 d[4] = {__fadd2_rn(b2, make_float2(0.f, 4.f)), __fadd2_rn(b2, make_float2(8.f, 12.f)),
                       __fadd2_rn(b2, make_float2(1.f, 5.f)), __fadd2_rn(b2, make_float2(9.f, 13.f))};
        float v[8];
        if (!INTEG) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            d[j] = __fmul2_rn(d[j], sk2);
            d[j] = __fmul2_rn(d[j], make_float2(-d[j].x, -d[j].y));
            const float2 e = __fmul2_rn(make_float2(ex2_approx(d[j].x), ex2_approx(d[j].y)), s2);
            const int o0 = (j & 1) * 8 + (j >> 1), o1 = o0 + 4;     // row offsets of the pair
            v[2 * j] = u0 + (uint32_t)o0 <= span ? e.x : 0.f;
            v[2 * j + 1] = u0 + (uint32_t)o1 <= span ? e.y : 0.f;
          }
        } else {
          // pixel-integrated rows: the pairs (r, r+1) of the two quads share their middle edge
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const float dr = bf + (float)(4 * i);                     // exact
            const float t0 = (dr - 0.5f) * fp.kint, t1 = (dr + 0.5f) * fp.kint, t2 = (dr + 1.5f) * fp.kint;
            const float e0 = edge_erfc(t0), e1 = edge_erfc(t1), e2 = edge_erfc(t2);
            v[i] = u0 + (uint32_t)(4 * i) <= span ? pp.y * pix_mass(t0, e0, t1, e1) : 0.f;
            v[4 + i] = u0 + (uint32_t)(4 * i + 1) <= span ? pp.y * pix_mass(t1, e1, t2, e2) : 0.f;
          }
        }
        // v = rows +0,+4,+8,+12 (quad hq=2hh) and +1,+5,+9,+13 (quad 2hh+1), [hq][i] order
        float4* dst = reinterpret_cast<float4*>(&S.gy[k * 16 + hh * 8]);
        dst[0] = make_float4(v[0], v[1], v[2], v[3]);
        dst[1] = make_float4(v[4], v[5], v[6], v[7]);
      }
      const int nx = ngx_tot;
      for (int g = tid; g < nx; g += TILE_THREADS) {
        const uint32_t own = S.gxown[g];
        const uint32_t slot = own & 0xFFFFu;
        const int k = (int)(slot & 15u);
        const float2 pp = S.px[own >> 16];
        const int rel = 8 * k;
        const int pcc = __float_as_int(pp.y);
        const uint32_t u0 = (uint32_t)(rel - (pcc & 0xFF)), span = (uint32_t)((pcc >> 8) - (pcc & 0xFF));
        const float bf = (float)rel - pp.x;
        const float2 b2 = make_float2(bf, bf);
        float v[8];
        if (!INTEG) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            float2 dd = __fmul2_rn(__fadd2_rn(b2, make_float2((float)(2 * j), (float)(2 * j + 1))), sk2);
            dd = __fmul2_rn(dd, make_float2(-dd.x, -dd.y));
            v[2 * j] = u0 + (uint32_t)(2 * j) <= span ? ex2_approx(dd.x) : 0.f;
            v[2 * j + 1] = u0 + (uint32_t)(2 * j + 1) <= span ? ex2_approx(dd.y) : 0.f;
          }
        } else {
          // pixel-integrated columns: 9 edges shared by the 8 consecutive columns
          float t = (bf - 0.5f) * fp.kint, e = edge_erfc(t);
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const float tn = (bf + (float)j + 0.5f) * fp.kint, en = edge_erfc(tn);
            v[j] = u0 + (uint32_t)j <= span ? pix_mass(t, e, tn, en) : 0.f;
            t = tn;
            e = en;
          }
        }
        float* gs = &S.gx[slot * 8];
        const int sw = ((k >> 2) & 1) * 4;
        *reinterpret_cast<float4*>(gs + sw) = make_float4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<float4*>(gs + (sw ^ 4)) = make_float4(v[4], v[5], v[6], v[7]);
      }
    }
    // the length of this lane group's list (stars < ns), and the warp's longest; pad the own list with all-zero
    // entries up to it (each list belongs to one lane group, so no other warp touches these entries)
    uint32_t len = 0;
#pragma unroll
    for (int w = 0; w < TILE_WARPS; ++w) {
      const int lo = ns - 32 * w;
      const uint32_t below = lo >= 32 ? 0xffffffffu : (lo <= 0 ? 0u : ((1u << lo) - 1u));
      len += __popc(S.bb[w][B] & S.sb[w][Q] & below);
    }
    const uint32_t steps = __reduce_max_sync(0xffffffffu, len);
    uint32_t* ent = &S.ent[B * NSTRIPS + Q];
    if (hq == 0)
      for (uint32_t st = len; st < steps; ++st) ent[st * (NBANDS * NSTRIPS)] = ZERO_ENT;
    __syncthreads();

#ifdef KT_REG_PREFETCH
    if (nb + tid < j1) rnext = rec[nid];
#else
    if (nb + tid < j1) prefetch_rec(&S.rn[tid], rec, nid);
#endif
    // ======================= accumulate: lane group q walks the (padded) list of block (B, Q)
    {
#pragma unroll 4
      for (uint32_t st = 0; st < steps; ++st) {
        const uint32_t e = ent[st * (NBANDS * NSTRIPS)];
        const uint32_t go = e & 0xFFFFu, xo = e >> 16;
        float4 g, a, c;
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g.x), "=f"(g.y), "=f"(g.z), "=f"(g.w) : "r"(gy_base + go));
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(a.x), "=f"(a.y), "=f"(a.z), "=f"(a.w) : "r"(gxa_base + xo));
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(c.x), "=f"(c.y), "=f"(c.z), "=f"(c.w) : "r"(gxb_base + xo));
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
          // the star of the entry's band slot and its ROI origin; pixel (row, col) of the lane's block is inside the
          // circle iff (2 (col - lx) - (R-1))^2 + (2 (row - ly) - (R-1))^2 <= R^2 (reading R21)
          const uint32_t lo = __float_as_uint(S.py[S.gyown[go >> 6] & 0xFFu].w);
          const int lx = (int)(int16_t)(lo & 0xFFFFu), ly = (int)(int16_t)(lo >> 16);
          const int RR = fp.R * fp.R, R1 = fp.R - 1;
          const float gx[8] = {a.x, a.y, a.z, a.w, c.x, c.y, c.z, c.w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int v = 2 * (16 * B + hq + 4 * i - ly) - R1;
            const int thr = RR - v * v;
            float gm[8];
#pragma unroll
            for (int p = 0; p < 8; ++p) {
              const int u = 2 * (8 * Q + p - lx) - R1;
              gm[p] = u * u <= thr ? gx[p] : 0.f;
            }
            const float2 gg = make_float2(gi[i], gi[i]);
            acc[i][0] = __ffma2_rn(gg, make_float2(gm[0], gm[1]), acc[i][0]);
            acc[i][1] = __ffma2_rn(gg, make_float2(gm[2], gm[3]), acc[i][1]);
            acc[i][2] = __ffma2_rn(gg, make_float2(gm[4], gm[5]), acc[i][2]);
            acc[i][3] = __ffma2_rn(gg, make_float2(gm[6], gm[7]), acc[i][3]);
          }
        }
      }
    }
    base += (uint32_t)ns;
    if (base < j1 && (base - wi.jb) % (uint32_t)fp.split == 0) {
      seg_flush(acc, seg_scratch, segs_done == 0);
      ++segs_done;
    }
  }
  if (segs_done) seg_finish(acc, seg_scratch);

  // ======================= output: rows 16 B + hq + 4 i, columns 64 wx + 8 q .. +7 of the tile
  if (tile_reduce_parts<false>(acc, ld_volatile_item(items + item), split_tab, part_buf, done, B, wx, q, hq, &s_last)) {
    if (!GRAY) {
      tile_store<false, 0>(acc, fp, out_, Y0, X0 + 64 * wx + 8 * q, B, hq);
    } else {
      // fused output stage: the fp32 tile is staged in shared memory (the profile slots are free now) and quantised
      // from there by all threads, 4 pixels each -- the register-resident form would spill at 3 CTAs per SM
      float* buf = S.gy;  // gy + gx: >= TILE_W * TILE_H floats
      __syncthreads();
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        float4* d = reinterpret_cast<float4*>(buf + lane_row<false>(B, hq, i) * TILE_W + 64 * wx + 8 * q);
        d[0] = make_float4(acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y);
        d[1] = make_float4(acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y);
      }
      __syncthreads();
      // the tile geometry again from the item (not held in registers across the accumulation)
      const uint32_t t2 = ld_volatile_item(items + item).tile;
      const int X2 = (int)(t2 % (uint32_t)fp.ntx) * TILE_W, Y2 = (int)(t2 / (uint32_t)fp.ntx) * TILE_H;
      tile_store_gray_staged(buf, fp, out_, Y2, X2, min(TILE_W, fp.W - X2), min(TILE_H, fp.rows - Y2));
    }
  }
  __shared__ uint32_t s_next;
  __syncthreads();  // every thread is past this item's shared-memory reads
  if (tid == 0) s_next = atomicAdd(&hdr->next_item, 1u) + gridDim.x;
  __syncthreads();
  item = s_next;
  }  // work loop
}

void init_tile_kernel() {
#define STARSIM_KT_ATTR(I, G, C) \
  cudaFuncSetAttribute(k_tile<I, G, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(TileSmem))
  STARSIM_KT_ATTR(false, false, false);
  STARSIM_KT_ATTR(true, false, false);
  STARSIM_KT_ATTR(false, true, false);
  STARSIM_KT_ATTR(true, true, false);
  STARSIM_KT_ATTR(false, false, true);
  STARSIM_KT_ATTR(true, false, true);
  STARSIM_KT_ATTR(false, true, true);
  STARSIM_KT_ATTR(true, true, true);
#undef STARSIM_KT_ATTR
}

void launch_tile(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                 const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                 cudaStream_t st, float* seg_scratch, const uint32_t* tile_off, const StarRec* ws_srec,
                 const uint16_t* ws_cbin) {
  if (fp.R <= SB_MAXR && fp.tile_impl == 3) {
    launch_tile_ws(ids, rec, fp, out, items, split_tab, part_buf, part_cap, done, hdr, num_sms, st, seg_scratch,
                   ws_srec, ws_cbin);
    return;
  }
  if (fp.R <= SB_MAXR && fp.tile_impl == 2) {
    launch_tile_sb(ids, rec, fp, out, items, split_tab, part_buf, part_cap, done, hdr, num_sms, st, seg_scratch,
                   tile_off);
    return;
  }
  if (wide_ok(fp.R) && fp.tile_impl != 1) {  // every mode but STARSIM_TILE_LISTS: the sorted-bin kernel for wide ROIs
    launch_tile_wide(ids, rec, fp, out, items, split_tab, part_buf, part_cap, done, hdr, num_sms, st, seg_scratch);
    return;
  }
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  // persistent, 3 CTAs per SM (2 for the circle ROI)
  const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)(fp.roi ? 2 : TILE_MINB_OPT) * num_sms);
  using KT = void (*)(const uint32_t*, const StarRec*, FrameParams, void*, const WorkItem*, const uint2*, float*,
                      uint32_t*, Header*, float*);
  static const KT kts[2][2][2] = {
      {{k_tile<false, false, false>, k_tile<false, false, true>}, {k_tile<false, true, false>, k_tile<false, true, true>}},
      {{k_tile<true, false, false>, k_tile<true, false, true>}, {k_tile<true, true, false>, k_tile<true, true, true>}}};
  const KT k = kts[fp.psf ? 1 : 0][fp.obits ? 1 : 0][fp.roi ? 1 : 0];
  k<<<(unsigned)grid, TILE_THREADS, sizeof(TileSmem), st>>>(ids, rec, fp, out, items, split_tab, part_buf, done, hdr,
                                                            seg_scratch);
}

}  // namespace starsim
