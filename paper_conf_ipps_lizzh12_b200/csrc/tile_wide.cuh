// Pieces of the wide-ROI sorted-corner-bin tile kernels (tile_wide.cu: k_tile_wide, both roles in every warp, and
// k_tile_wws, warp-specialised): geometry, corner-bin key, the bin scan, the profile preparation of one
// star and the walk of one chunk.  The design is described at the top of tile_wide.cu.
#pragma once
#include "common.cuh"

namespace starsim {

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
  static_assert(NBIN < 256, "bin keys (and the no-bin key NBIN) fit 8 bits");
};

// corner bin of a star whose ROI origin is (lx, ly) relative to the tile, NBIN if its clipped ROI misses the tile
template <int KB>
__device__ __forceinline__ uint32_t wide_key(int lx, int ly, int c0, int c1, int r0, int r1) {
  using G = WideGeom<KB>;
  return (c0 <= c1 && r0 <= r1) ? (uint32_t)(((ly >> 4) + KB - 1) * G::NSK + (lx >> 3) + G::KS - 1)
                                : (uint32_t)G::NBIN;
}

// The stars of the warp with the same key (8 ballots: MATCH.ANY loops over the warp's distinct keys).
__device__ __forceinline__ uint32_t key_peers(uint32_t key) {
  uint32_t peers = 0xffffffffu;
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    const uint32_t kb = (key >> b) & 1u;
    const uint32_t m = __ballot_sync(0xffffffffu, kb);
    peers &= kb ? m : ~m;
  }
  return peers;
}

// One warp: hist[w][bin] (stars of warp w in the bin) becomes, in place, the stars of the bin in the warps before w;
// binstart[bin] the exclusive scan of the bin totals, binstart[NBIN] the total.
template <int KB, int NW>
__device__ __forceinline__ void wide_scan(uint32_t (*hist)[WideGeom<KB>::NBIN], uint32_t* binstart, int lane) {
  using G = WideGeom<KB>;
  uint32_t tot[G::PER], sum = 0;
#pragma unroll
  for (int h = 0; h < G::PER; ++h) {
    const int bin = G::PER * lane + h;
    uint32_t c[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) c[w] = bin < G::NBIN ? hist[w][bin] : 0u;
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
      if (bin < G::NBIN) hist[w][bin] = run;
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
    if (bin <= G::NBIN) binstart[bin] = ex;
    ex += tot[h];
  }
}

// Row profile s' gy of one star on the bands b0 .. b0 + KB - 1 (those inside the tile) into its slot gyj (band slot k
// = 16 floats at 16 k), zero outside the clipped ROI rows r0..r1; a quad the ROI misses is stored as zeros without
// evaluating it.  yr: the star's y relative to the tile (exact).
template <int KB, bool INTEG>
__device__ __forceinline__ void wide_rows(float* gyj, int b0, int r0, int r1, float yr, float s, const FrameParams& fp,
                                          int rot) {
  const float2 sk2 = make_float2(fp.sk, fp.sk), s2 = make_float2(s, s);
#pragma unroll
  for (int k = 0; k < KB; ++k) {
    const int bb = b0 + k;
    if (bb < 0 || bb >= NBANDS) continue;  // never read
    const int ra = r0 - 16 * bb, rb = r1 - 16 * bb;
    const uint32_t m16 = (ra > 15 || rb < 0) ? 0u : (0xFFFFu >> (15 - min(rb, 15))) & (0xFFFFu << max(ra, 0)) & 0xFFFFu;
    float4* dst = reinterpret_cast<float4*>(gyj + 16 * k);
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const int w = (c + rot) & 3;  // rotated quad order (spreads the stores of a warp over the banks)
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
            v[i] = (m >> i) & 1u ? s * pix_mass(t, e, tn, en) : 0.f;
            t = tn;
            e = en;
          }
        }
      }
      dst[w] = make_float4(v[0], v[1], v[2], v[3]);
    }
  }
}

// Column profile gx of one star on the strips q0 .. q0 + KS - 1 (those inside the tile) into its ring gxj (strip Q at
// 8 (Q mod RS), its 16-B halves swapped when bit 2 of Q is set), zero outside the clipped ROI columns c0..c1.
template <int KB, bool INTEG>
__device__ __forceinline__ void wide_cols(float* gxj, int q0, int c0, int c1, float xr, const FrameParams& fp) {
  using G = WideGeom<KB>;
  const float2 sk2 = make_float2(fp.sk, fp.sk);
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
    SS_CHECK(k < G::RS);  // the KS strips of a star have distinct ring positions
    float* gs = gxj + (Qs & (G::RS - 1)) * 8;
    const int sw = ((Qs >> 2) & 1) * 4;
    *reinterpret_cast<float4*>(gs + sw) = make_float4(v[0], v[1], v[2], v[3]);
    *reinterpret_cast<float4*>(gs + (sw ^ 4)) = make_float4(v[4], v[5], v[6], v[7]);
  }
}

// The walk of one chunk by lane (group Q of warp band B, rows 4 hq.. of the band): range k = 0 .. KB-1 holds the
// corner bins of band B - k and strips Q - KS + 1 .. Q, read with band slot k; each lane group runs its own trip count
// (a divergent loop: the warp runs its longest range), one step of look-ahead on the operand loads.  gy_base /
// gx_base: the shared addresses of star 0's band slot 0 (+ 16 hq) and of strip Q's place in star 0's ring.
template <int KB, bool CIRC>
__device__ __forceinline__ void wide_walk(float2 (&acc)[4][4], const uint32_t* binstart, uint32_t gy_base,
                                          uint32_t gx_base, const uint32_t* lo2, int B, int Q, int hq, int swz,
                                          const FrameParams& fp) {
  using G = WideGeom<KB>;
  constexpr uint32_t SYB = G::SYF * 4u, SXB = G::SXF * 4u;
#pragma unroll 1
  for (int k = 0; k < KB; ++k) {
    // corner band B - k (band key B - k + KB - 1), corner strips Q - KS + 1 .. Q (strip keys Q .. Q + KS - 1)
    const int bk = B - k + KB - 1;
    const uint32_t s = binstart[bk * G::NSK + Q], e = binstart[bk * G::NSK + Q + G::KS];
    SS_CHECK(s <= e && e <= binstart[G::NBIN] && bk >= 0 && bk < G::NBK);
    uint32_t ga = gy_base + s * SYB + 64u * (uint32_t)k, xa = gx_base + s * SXB;
    uint32_t jj = s;
    const uint32_t gend = ga + (e - s) * SYB;
    // past the range end the look-ahead loads read other shared-memory words of the CTA, never used
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
        const uint32_t lo = lo2[jj++];
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
}

}  // namespace starsim
