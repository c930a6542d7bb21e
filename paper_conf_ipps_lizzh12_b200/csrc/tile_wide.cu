// k_tile_wide: tile accumulation with sorted corner bins for wide ROIs, SB_MAXR < R <= WIDE_MAXR (17 < R <= 65:
// the wide end of the C4 ROI sweep, BASELINE configs[3]; Table III's ROI-side axis) -- SURVEY.md
// §8a step a5, Eqs. 2-3.
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
// Summation order of a pixel: per chunk (in list order; lists longer than SPLIT_LEN in R19 segments), range k = 0 ..
// KB-1, each in sorted order (corner bin, then list order): deterministic and a function of the tile's own list only,
// so tile-aligned band renders are bitwise the frame's pixels (reading R12).  No atomics on the image.
#include <algorithm>

#include "common.cuh"
#include "launch.h"
#include "tile_common.cuh"

namespace starsim {

namespace {

constexpr int WD_CHUNK = 128;                     // stars per chunk (two prep threads per star)
constexpr int WD_MINB = 2;                        // CTAs per SM (128 registers, <= 112 KB shared memory)
constexpr int WD_SW = 4;                          // warps that own a star in the sort (threads 0..127)
static_assert(SPLIT_LEN % WD_CHUNK == 0, "segments are whole chunks");
static_assert(WD_CHUNK * 2 == TILE_THREADS, "two prep threads per star");

template <int KB>
struct WideGeom {
  static constexpr int KS = 2 * KB - 1;           // strips an ROI of side <= MAXR spans
  static constexpr int RS = KS <= 8 ? 8 : 16;     // strip ring
  static constexpr int SYF = (KB | 1) * 16;       // floats per star: row profile (an odd number of 64-B slots)
  static constexpr int SXF = RS * 8;              // floats per star: column profile ring
  static constexpr int MAXR = 16 * (KB - 1) + 1;  // widest ROI side
  // corner bins of the UNCLIPPED ROI origin (ly, lx), tile-relative: band key (ly >> 4) + KB - 1 (ly >= -(R - 1)),
  // strip key (lx >> 3) + KS - 1, band-major
  static constexpr int NBK = NBANDS + KB - 1;
  static constexpr int NSK = NSTRIPS + KS - 1;
  static constexpr int NBIN = NBK * NSK;          // 120 / 154 / 192
  static constexpr int PER = NBIN / 32 + 1;       // bins per lane of the scanning warp (32 PER > NBIN: one lane
                                                  // writes the total at bin NBIN)
};

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
__global__ void __launch_bounds__(TILE_THREADS, WD_MINB) k_tile_wide(const uint32_t* __restrict__ ids,
                                                                     const StarRec* __restrict__ rec, FrameParams fp,
                                                                     void* __restrict__ out_,
                                                                     const WorkItem* __restrict__ items,
                                                                     const uint2* __restrict__ split_tab,
                                                                     float* __restrict__ part_buf,
                                                                     uint32_t* __restrict__ done, Header* hdr,
                                                                     float* __restrict__ seg_scratch) {
  using G = WideGeom<KB>;
  constexpr uint32_t SYB = G::SYF * 4u, SXB = G::SXF * 4u;  // slot strides in bytes
  extern __shared__ __align__(16) unsigned char smem_raw[];
  WideSmem<KB>& S = *reinterpret_cast<WideSmem<KB>*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int sid = tid & (WD_CHUNK - 1);   // the chunk star this thread sorts and prepares
  const bool colhalf = tid >= WD_CHUNK;   // prep: false = row profile, true = column profile
  const uint32_t lt = (1u << lane) - 1u;
  const float sk = fp.sk;

  const int q = lane >> 2, hq = lane & 3, wx = warp & 1, B = warp >> 1;
  const int Q = 8 * wx + q;
  const int swz = (Q >> 2) & 1;
  const uint32_t gy_base = (uint32_t)__cvta_generic_to_shared(S.gy) + 16u * hq;
  const uint32_t gx_base = (uint32_t)__cvta_generic_to_shared(S.gx) + 32u * (uint32_t)(Q & (G::RS - 1));
  __shared__ int s_last;
  __shared__ uint32_t s_next;

  // persistent CTAs (WD_MINB per SM): item blockIdx.x first, then items from the counter the planner zeroed (the
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
        if (c0 <= c1 && r0 <= r1) key = (uint32_t)(((ly >> 4) + KB - 1) * G::NSK + (lx >> 3) + G::KS - 1);
      }
      // warps w and w + 4 hold the same stars in the same lanes: the same peers and ranks
      // (the stars of the warp with the same key from 8 ballots: MATCH.ANY loops over the warp's distinct keys)
      static_assert(G::NBIN < 256, "bin keys (and the no-bin key) fit 8 bits");
      uint32_t peers = 0xffffffffu;
#pragma unroll
      for (int b = 0; b < 8; ++b) {
        const uint32_t kb = (key >> b) & 1u;
        const uint32_t m = __ballot_sync(0xffffffffu, kb);
        peers &= kb ? m : ~m;
      }
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
      if (warp == 0) {
        uint32_t tot[G::PER], sum = 0;
#pragma unroll
        for (int h = 0; h < G::PER; ++h) {
          const int bin = G::PER * lane + h;
          uint32_t c[WD_SW];
#pragma unroll
          for (int w = 0; w < WD_SW; ++w) c[w] = bin < G::NBIN ? S.hist[w][bin] : 0u;
          uint32_t run = 0;
#pragma unroll
          for (int w = 0; w < WD_SW; ++w) {
            if (bin < G::NBIN) S.hist[w][bin] = run;
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
        for (int h = 0; h < G::PER; ++h) {
          const int bin = G::PER * lane + h;
          if (bin <= G::NBIN) S.binstart[bin] = ex;  // bin NBIN receives the total
          ex += tot[h];
        }
      }
      __syncthreads();
      // ======================= prep: the star's profiles at its sorted place j
      if (key < G::NBIN) {
        const uint32_t j = S.binstart[key] + S.hist[warp & (WD_SW - 1)][key] + rank;
        const float2 sk2 = make_float2(sk, sk);
        // the unclipped ROI origin's band and strip (bands b0 .. b0 + KB - 1, strips q0 .. q0 + KS - 1 hold it)
        const int b0 = (int)(key / G::NSK) - (KB - 1), q0 = (int)(key % G::NSK) - (G::KS - 1);
        if (!colhalf) {
          if (CIRC) S.lo2[j] = lo2;
          const float yr = r.y - (float)IY0;  // exact
          const float2 s2 = make_float2(r.s, r.s);
#pragma unroll
          for (int k = 0; k < KB; ++k) {
            const int bb = b0 + k;
            if (bb < 0 || bb >= NBANDS) continue;  // never read
            const int ra = r0 - 16 * bb, rb = r1 - 16 * bb;
            const uint32_t m16 = (ra > 15 || rb < 0) ? 0u
                                                     : (0xFFFFu >> (15 - min(rb, 15))) & (0xFFFFu << max(ra, 0)) & 0xFFFFu;
            float4* dst = reinterpret_cast<float4*>(&S.gy[j * G::SYF + 16 * k]);
#pragma unroll
            for (int c = 0; c < 4; ++c) {
              const int w = (c + lane) & 3;  // lane-rotated quad order (spreads the stores over the banks)
              const uint32_t m = (m16 >> (4 * w)) & 0xFu;
              float v[4] = {0.f, 0.f, 0.f, 0.f};
              if (m) {
                const float bf = (float)(16 * bb + 4 * w) - yr;  // exact
                if (!INTEG) {
                  const float2 bbv = make_float2(bf, bf);
#pragma unroll
                  for (int i = 0; i < 4; i += 2) {
                    float2 d = __fadd2_rn(bbv, make_float2((float)i, (float)(i + 1)));
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
              }
              dst[w] = make_float4(v[0], v[1], v[2], v[3]);
            }
          }
        } else {
          const float xr = r.x - (float)X0;  // exact
#pragma unroll
          for (int k = 0; k < G::KS; ++k) {
            const int Qs = q0 + k;
            if (Qs < 0 || Qs >= NSTRIPS) continue;  // never read
            const int rel = 8 * Qs;
            const int lo = max(c0 - rel, 0), hi = min(c1 - rel, 7);
            const uint32_t m = hi >= lo ? ((0xFFu >> (7 - hi)) & (0xFFu << lo)) : 0u;
            float v[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
            if (m) {
              const float bf = (float)rel - xr;  // exact
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
            }
            float* gs = &S.gx[j * G::SXF + (Qs & (G::RS - 1)) * 8];
            const int sw = ((Qs >> 2) & 1) * 4;
            *reinterpret_cast<float4*>(gs + sw) = make_float4(v[0], v[1], v[2], v[3]);
            *reinterpret_cast<float4*>(gs + (sw ^ 4)) = make_float4(v[4], v[5], v[6], v[7]);
          }
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
      // ======================= accumulate: lane group q walks its KB ranges (each padded with the zero slot)
#pragma unroll 1
      for (int k = 0; k < KB; ++k) {
        // corner band B - k (band key B - k + KB - 1), corner strips Q - KS + 1 .. Q (strip keys Q .. Q + KS - 1)
        const int bk = B - k + KB - 1;
        const uint32_t s = S.binstart[bk * G::NSK + Q], e = S.binstart[bk * G::NSK + Q + G::KS];
        const uint32_t len = e - s;
        // sorted star j = s + t, band slot k; each lane group runs its own trip count (the warp's longest: the
        // other groups' lanes idle), no padding reads
        uint32_t ga = gy_base + s * SYB + 64u * (uint32_t)k, xa = gx_base + s * SXB;
        uint32_t jj = s;
        const uint32_t gend = ga + len * SYB;
        // one step of look-ahead: the next star's operands are loaded before this one's FMAs (past the range end the
        // loads read other shared-memory words, never used)
        float4 gn, an, cn;
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(gn.x), "=f"(gn.y), "=f"(gn.z), "=f"(gn.w) : "r"(ga));
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(an.x), "=f"(an.y), "=f"(an.z), "=f"(an.w) : "r"(xa));
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(cn.x), "=f"(cn.y), "=f"(cn.z), "=f"(cn.w) : "r"(xa + 16u));
#pragma unroll 2
        for (; ga < gend; ga += SYB, xa += SXB) {
          const float4 g = gn, a = an, c = cn;
          asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(gn.x), "=f"(gn.y), "=f"(gn.z), "=f"(gn.w) : "r"(ga + SYB));
          asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(an.x), "=f"(an.y), "=f"(an.z), "=f"(an.w) : "r"(xa + SXB));
          asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(cn.x), "=f"(cn.y), "=f"(cn.z), "=f"(cn.w) : "r"(xa + SXB + 16u));
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
            // reading R21: the star's ROI origin from its slot, the per-pixel integer disc test (as k_tile_sb)
            const uint32_t lo = S.lo2[jj++];
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
        }
      }
      if ((base + WD_CHUNK - wi.jb) % SPLIT_LEN == 0 && base + WD_CHUNK < j1) {
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

namespace {
using KW = void (*)(const uint32_t*, const StarRec*, FrameParams, void*, const WorkItem*, const uint2*, float*,
                    uint32_t*, Header*, float*);
template <int KB>
struct WideTab {
  static constexpr KW k[2][2] = {{k_tile_wide<KB, false, false>, k_tile_wide<KB, false, true>},
                                 {k_tile_wide<KB, true, false>, k_tile_wide<KB, true, true>}};
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
  const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)WD_MINB * num_sms);  // persistent CTAs
  const int kb = wide_kb(fp.R), a = fp.psf ? 1 : 0, b = fp.roi ? 1 : 0;
  const KW k = kb == 3 ? WideTab<3>::k[a][b] : kb == 4 ? WideTab<4>::k[a][b] : WideTab<5>::k[a][b];
  const size_t smem = kb == 3 ? sizeof(WideSmem<3>) : kb == 4 ? sizeof(WideSmem<4>) : sizeof(WideSmem<5>);
  k<<<(unsigned)grid, TILE_THREADS, smem, st>>>(ids, rec, fp, out, items, split_tab, part_buf, done, hdr, seg_scratch);
}

}  // namespace starsim
