// k_tile8: the round-2 tile-accumulation kernel for R <= 17 (Eqs. 2-3,
// PAPER.md:35, 48), and k_t8sort, the per-tile corner-bin sort that feeds it.
//
// What bounds a register-tiled gather of Eq. 3 on B200 is shared-memory operand delivery and instruction issue
// (bench_micro/walk8.cu, profiles/r2_microbench_walk8.jsonl).  This kernel is built around the layout that measured
// best:
//
//   * lane block 8 x 8 pixels (64 fp32 accumulators as 32 float2, FFMA2 of a row factor times a column pair): 16
//     profile floats (4 x LDS.128) per 32 FFMA2;
//   * a star's profiles live in a 256-B slot as two rings of 32 floats indexed by the ABSOLUTE tile row / column
//     mod 32 (rows 8B..8B+7 of band B at ring slot B mod 4), so a lane reads its band's 8 row factors and its strip's
//     8 column factors at lane-constant offsets whatever star it visits;
//   * the lanes of each quarter-warp phase of an LDS.128 sit on two diagonals of a 4 x 4 block group, with the 16-B
//     halves swapped by bit 1 of the other coordinate: every phase hits 8 distinct bank quads (conflict-free for any
//     stars the lanes visit; 20 SM-cycles per 32-FFMA2 step measured, vs 48 for a row-major lane order);
//   * k_t8sort (one CTA per work item, fully parallel) sorts every segment (<= SPLIT_LEN stars) of a tile list by
//     ROI corner bin (strip-major 8 x 8 bins, stable: star order inside a bin) and writes the star records in that
//     order at the list's own positions -- the tile kernel does no sorting and no gathers;
//   * k_tile8's producer warps cut each sorted segment into stratified chunks (chunk c = sorted positions
//     j = c mod nch): every chunk is a thin sample of every bin, so each lane's share of a chunk is ~1/nch of its
//     tile-level candidate list and the per-warp padding stays at the tile level (~78 %) rather than the chunk level;
//     they evaluate each star's two profiles into a ring of shared-memory stages;
//   * consumer warps (one 32 x 64 pixel quadrant each) walk, per chunk, the three sorted ranges (corner strips
//     Q-2..Q, bands B-2..B each) that can reach their 8 x 8 block, accumulating in registers, and write every pixel
//     once.
//
// Summation order (reading R12/R19): per pixel, segments of SPLIT_LEN stars of the tile list in list order; inside a
// segment, chunk by chunk, and inside a chunk the corner-strip ranges Q-2, Q-1, Q, each in (band, star) order.  It
// is a function of the tile's own list only, so tile-aligned bands give bitwise the frame's pixels; a heavy tile
// split into parts (one segment each) and the same tile processed whole (segment by segment, partial sums kept in a
// per-CTA scratch tile) give the same bits.
#include <algorithm>

#include "common.cuh"
#include "launch.h"

namespace starsim {

namespace {

constexpr int T8_NB = TILE_H / 8;              // 8 bands of 8 rows
constexpr int T8_NQ = TILE_W / 8;              // 16 strips of 8 columns
constexpr int T8_KB = T8_NB + 2;               // corner-band keys: b0 = -2 .. 7 (ROI origin up to 16 rows above)
constexpr int T8_KQ = T8_NQ + 2;               // corner-strip keys: q0 = -2 .. 15
constexpr int T8_NBIN = T8_KB * T8_KQ;         // 180 corner bins, strip-major: key = (q0 + 2) * T8_KB + b0 + 2
#ifndef T8_CHUNK_OPT
#define T8_CHUNK_OPT 128
#endif
#ifndef T8_NS_OPT
#define T8_NS_OPT 3
#endif
constexpr int T8_CHUNK = T8_CHUNK_OPT;         // stars per stage
constexpr int T8_SEG = SPLIT_LEN;              // stars per sorted segment
constexpr int T8_NS = T8_NS_OPT;               // stages
constexpr int T8_CONS = 4;                     // consumer warps (one 32 x 64 quadrant each)
#ifndef T8_PROD_OPT
#define T8_PROD_OPT 4
#endif
constexpr int T8_PROD = T8_PROD_OPT;           // producer warps: 4 (row + column profile per thread) or 8 (one each)
constexpr int T8_PT = 32 * T8_PROD;            // producer threads
constexpr int T8_CT = 32 * T8_CONS;            // consumer threads
constexpr int T8_THREADS = T8_PT + T8_CT;
constexpr int T8_HDR = T8_NBIN + 1 + 3;        // bin starts (+ padding)
static_assert(T8_NBIN < 256, "bin keys fit a byte");
static_assert(T8_CHUNK <= T8_PT, "at most one row and one column profile per producer thread per chunk");

constexpr uint32_t T8_SEG_LAST = 1u, T8_ITEM_LAST = 2u, T8_STOP = 4u;

struct T8Stage {
  float4 prof[T8_CHUNK][16];        // star k: [0..8) gy ring quads (rows mod 32), [8..16) gx ring quads
  float4 zero[16];                  // an all-zero star slot: what a lane whose ranges are exhausted reads
  uint32_t binstart[T8_HDR];        // the segment's sorted bin starts (tile-level)
  uint32_t tile, aux, flags, c;     // work item, chunk c of nch
  uint32_t nch, magic, seg, asg;    // magic = ceil(2^32 / nch), 0 for nch = 1; asg: 4 x 2 block groups (4 bits)
};
static_assert(sizeof(T8Stage) % 16 == 0, "stages hold float4");

struct T8Smem {
  unsigned long long full[T8_NS], empty[T8_NS];
  T8Stage st[T8_NS];
  uint32_t binstart[T8_NBIN + 1 + 3];
  uint32_t gsum[8];                 // candidate count of each 4 x 4 block group of the item (for the balancing)
  uint32_t next_item, asg;
};

constexpr size_t T8_SMEM_BYTES = (sizeof(T8Smem) + 15) & ~size_t(15);
#ifdef T8_TIMING
constexpr size_t T8_SMEM_LAUNCH = T8_SMEM_BYTES + 16 * 8 * (T8_THREADS / 32);
// per-phase SM cycles summed over warps (debug builds only, tools/t8_timing.py)
__device__ unsigned long long g_t8_prof[16];
__device__ __forceinline__ unsigned long long* t8_acc_slot() {  // per-warp accumulators in shared memory
  extern __shared__ __align__(16) unsigned char smem_raw[];
  return reinterpret_cast<unsigned long long*>(smem_raw + T8_SMEM_BYTES) + 16 * (threadIdx.x >> 5);
}
#define T8_T(v) const long long v = clock64()
#define T8_ACC(k, d) if ((threadIdx.x & 31) == 0) t8_acc_slot()[k] += (unsigned long long)(d)
#else
constexpr size_t T8_SMEM_LAUNCH = T8_SMEM_BYTES;
#define T8_T(v)
#define T8_ACC(k, d)
#endif

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// T8_WARP_ARRIVE: one arrival per warp -- the lanes' shared-memory writes are ordered before lane 0's (release)
// arrive by the __syncwarp, and release is cumulative; 1 instead of 32 arrivals per warp, but compute-sanitizer's
// racecheck does not model it (it reports the hand-offs as hazards).  Default: every thread arrives (the counts below
// are threads), the form racecheck verifies.
#ifdef T8_WARP_ARRIVE
constexpr uint32_t T8_ARRIVALS_PER_WARP = 1;
__device__ __forceinline__ void mbar_arrive_warp(unsigned long long* b) {
  __syncwarp();
  if ((threadIdx.x & 31) == 0) mbar_arrive(b);
}
#else
constexpr uint32_t T8_ARRIVALS_PER_WARP = 32;
__device__ __forceinline__ void mbar_arrive_warp(unsigned long long* b) { mbar_arrive(b); }
#endif
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t parity) {
  const uint32_t a = smem_u32(b);
  uint32_t ok;
  do {
#ifdef T8_TESTWAIT
    asm volatile(
        "{ .reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(a), "r"(parity)
        : "memory");
#else
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(ok)
        : "r"(a), "r"(parity)
        : "memory");
#endif
  } while (!ok);
}
__device__ __forceinline__ void prod_sync() { asm volatile("bar.sync 1, %0;" ::"n"(T8_PT) : "memory"); }
__device__ __forceinline__ void cons_sync() { asm volatile("bar.sync 2, %0;" ::"n"(T8_CT) : "memory"); }

__device__ __forceinline__ uint32_t seg_count(const WorkItem& w) {
  const uint32_t len = w.je - w.jb;
  return len ? (len + T8_SEG - 1) / T8_SEG : 1u;
}
__device__ __forceinline__ uint32_t seg_len(const WorkItem& w, uint32_t s) {
  const uint32_t len = w.je - w.jb;
  return min((uint32_t)T8_SEG, len - min(len, s * (uint32_t)T8_SEG));
}
// strip-major corner-bin key of a star record in the tile with origin (X0, IY0)
__device__ __forceinline__ uint32_t t8_key(uint32_t lo, int X0, int IY0) {
  const int lx = lo_x_of(lo) - X0, ly = lo_y_of(lo) - IY0;
  return (uint32_t)(((lx >> 3) + 2) * T8_KB + (ly >> 3) + 2);
}

// ------------------------------------------------------------------------------------------------ k_t8sort
// One CTA per work item: every segment of its tile list (list positions [jb + s SPLIT_LEN, ...)) is stably sorted
// by strip-major corner bin and its star records are written in that order at the same positions of `srec`.
constexpr int TS_THREADS = 256;
constexpr int TS_WARPS = TS_THREADS / 32;
constexpr int TS_EPT = T8_SEG / TS_THREADS;    // elements per thread (4)

// The segment's bin starts go to row sid of `sbin` (T8_HDR words): sid = item for its first segment, else
// items_cap + sext[item] + s - 1 (extra rows taken from a counter, only for unsplit lists longer than SPLIT_LEN).
__global__ void __launch_bounds__(TS_THREADS) k_t8sort(const uint32_t* __restrict__ ids,
                                                       const StarRec* __restrict__ rec, FrameParams fp,
                                                       const WorkItem* __restrict__ items, Header* hdr,
                                                       StarRec* __restrict__ srec, uint32_t* __restrict__ sbin,
                                                       uint32_t* __restrict__ sext, uint32_t items_cap) {
  __shared__ uint32_t wc[TS_WARPS][T8_NBIN];
  __shared__ uint32_t s_ext;
  const uint32_t nitems = __ldcg(&hdr->nitems);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  for (uint32_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const WorkItem w = items[item];
    const int tx = (int)(w.tile % (uint32_t)fp.ntx), ty = (int)(w.tile / (uint32_t)fp.ntx);
    const int X0 = tx * TILE_W, IY0 = fp.row0 + ty * TILE_H;
    const uint32_t nseg = seg_count(w);
    if (threadIdx.x == 0) {
      s_ext = nseg > 1 ? atomicAdd(&hdr->next_seg, nseg - 1) : 0u;
      sext[item] = s_ext;
    }
    for (uint32_t s = 0; s < nseg; ++s) {
      const uint32_t L = seg_len(w, s), base = w.jb + s * (uint32_t)T8_SEG;
      // warp `warp` takes elements [warp G, (warp + 1) G) in list order, 32 at a time
      const uint32_t G = ((L + TS_WARPS - 1) / TS_WARPS + 31) & ~31u;
      for (int b = threadIdx.x; b < TS_WARPS * T8_NBIN; b += TS_THREADS) (&wc[0][0])[b] = 0u;
      __syncthreads();  // s_ext
      const uint32_t sid = s == 0 ? item : items_cap + s_ext + s - 1u;
      uint32_t id[TS_EPT];
#pragma unroll
      for (int k = 0; k < TS_EPT; ++k) {
        const uint32_t i = (uint32_t)warp * G + (uint32_t)(32 * k + lane);
        id[k] = ((uint32_t)(32 * k) < G && i < L && i < (uint32_t)(warp + 1) * G) ? __ldg(&ids[base + i]) : 0xFFFFFFFFu;
      }
      StarRec r[TS_EPT];
#pragma unroll
      for (int k = 0; k < TS_EPT; ++k) r[k] = id[k] != 0xFFFFFFFFu ? rec[id[k]] : StarRec{0.f, 0.f, 0.f, 0u};
      __syncthreads();
      uint32_t key[TS_EPT], lrank[TS_EPT];
#pragma unroll
      for (int k = 0; k < TS_EPT; ++k) {
        key[k] = 0xFFu;
        lrank[k] = 0u;
        if ((uint32_t)(32 * k) >= G) continue;  // warp-uniform
        if (id[k] != 0xFFFFFFFFu) key[k] = t8_key(r[k].lo, X0, IY0);
        uint32_t peers = 0xFFFFFFFFu;  // the lanes with the same key (from 8 ballots)
#pragma unroll
        for (int b = 0; b < 8; ++b) {
          const uint32_t kb = (key[k] >> b) & 1u;
          const uint32_t mm = __ballot_sync(0xFFFFFFFFu, kb);
          peers &= kb ? mm : ~mm;
        }
        uint32_t cnt = 0;
        if (key[k] < T8_NBIN) cnt = wc[warp][key[k]];
        __syncwarp();
        if (key[k] < T8_NBIN && (peers & lt) == 0u) wc[warp][key[k]] = cnt + __popc(peers);
        __syncwarp();
        lrank[k] = cnt + __popc(peers & lt);
      }
      __syncthreads();
      if (warp == 0) {  // bin starts: lane l scans bins [6 l, 6 l + 6); per-warp first positions in place
        uint32_t tot[6], sum = 0;
#pragma unroll
        for (int h = 0; h < 6; ++h) {
          const int b = 6 * lane + h;
          uint32_t t = 0;
          if (b < T8_NBIN)
#pragma unroll
            for (int q = 0; q < TS_WARPS; ++q) t += wc[q][b];
          tot[h] = t;
          sum += t;
        }
        uint32_t incl = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t v = __shfl_up_sync(0xFFFFFFFFu, incl, o);
          if (lane >= o) incl += v;
        }
        uint32_t run = incl - sum;
#pragma unroll
        for (int h = 0; h < 6; ++h) {
          const int b = 6 * lane + h;
          if (b < T8_NBIN) {
            uint32_t r2 = run;
#pragma unroll
            for (int q = 0; q < TS_WARPS; ++q) {
              const uint32_t cw = wc[q][b];
              wc[q][b] = r2;
              r2 += cw;
            }
          }
          if (b <= T8_NBIN) sbin[(size_t)sid * T8_HDR + b] = run;
          run += tot[h];
        }
      }
      __syncthreads();
#pragma unroll
      for (int k = 0; k < TS_EPT; ++k)
        if (key[k] < T8_NBIN) srec[base + wc[warp][key[k]] + lrank[k]] = r[k];
      __syncthreads();
    }
  }
}

// ------------------------------------------------------------------------------------------------ producer side

// One axis of a star's profile into its 32-float ring: positions p = 8 b0 + w, w in [0, 24) (tile-relative pixel
// coordinate of the window, 8-aligned), value at ring index p mod 32.  Window positions outside the ROI [lo, lo+R)
// get exact zeros; the ring's fourth slot is never read (a lane only visits stars whose window covers its band).
//   point PSF (Eq. 2): v = scale * 2^(-(d sk)^2), d = p - c exactly as the oracle's pixel - centre;
//   integrated (NEXT-2): v = scale * (Phi(d + 1/2) - Phi(d - 1/2)).
template <bool INTEG, bool SCALE>
__device__ __forceinline__ void t8_axis(float4* slot, int lo, float cr, float scale, int R, float sk, float kint,
                                        uint32_t swp) {
  const int b0 = lo >> 3;                       // floor(lo / 8), lo >= -16
  const int o = lo & 7;                         // lo - 8 b0
  const uint32_t M = (0xFFFFFFFFu >> (32 - R)) << o;  // window positions inside the ROI
  const float d0 = (float)(lo - o) - cr;        // 8 b0 - c
  // step c stores window chunk cc = c ^ swp (the two halves of a band in either order): the producer lanes of a
  // quarter-warp pass swp = bit 2 of their lane, so lanes whose bands agree mod 4 store to different bank quads
#pragma unroll
  for (int c = 0; c < 6; ++c) {
    const uint32_t cc = (uint32_t)c ^ swp;
    const uint32_t m = M >> (4 * cc);
    float v[4];
    if (!INTEG) {
      const float2 sk2 = make_float2(sk, sk);
      const float bf = d0 + (float)(4 * cc);
#pragma unroll
      for (int i = 0; i < 4; i += 2) {
        float2 t = __fmul2_rn(__fadd2_rn(make_float2(bf, bf), make_float2((float)i, (float)(i + 1))), sk2);
        t = __fmul2_rn(t, make_float2(-t.x, -t.y));
        float2 e = make_float2(ex2_approx(t.x), ex2_approx(t.y));
        if (SCALE) e = __fmul2_rn(e, make_float2(scale, scale));
        v[i] = (m >> i) & 1u ? e.x : 0.f;
        v[i + 1] = (m >> (i + 1)) & 1u ? e.y : 0.f;
      }
    } else {
      const float bf = d0 + (float)(4 * cc);
      float t = (bf - 0.5f) * kint, e = edge_erfc(t);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float tn = (bf + (float)i + 0.5f) * kint, en = edge_erfc(tn);
        v[i] = (m >> i) & 1u ? scale * pix_mass(t, e, tn, en) : 0.f;
        t = tn;
        e = en;
      }
    }
    slot[(2 * b0 + (int)cc) & 7] = make_float4(v[0], v[1], v[2], v[3]);
  }
}

// Both profiles a producer thread evaluates per chunk -- the row profile of star A and the column profile of star B
// -- interleaved chunk by chunk, so the two independent exp chains overlap (the producer is latency-bound).
template <bool INTEG>
__device__ __forceinline__ void t8_axis2(float4* slotY, int loY, float crY, float sY, bool vY, float4* slotX, int loX,
                                         float crX, bool vX, int R, float sk, float kint, uint32_t swp) {
  const int bY = loY >> 3, bX = loX >> 3;
  const uint32_t MY = (0xFFFFFFFFu >> (32 - R)) << (loY & 7), MX = (0xFFFFFFFFu >> (32 - R)) << (loX & 7);
  const float dY = (float)(loY & ~7) - crY, dX = (float)(loX & ~7) - crX;
#pragma unroll
  for (int c = 0; c < 6; ++c) {
    const uint32_t cc = (uint32_t)c ^ swp;
    const uint32_t mY = MY >> (4 * cc), mX = MX >> (4 * cc);
    float vy[4], vx[4];
    if (!INTEG) {
      const float2 sk2 = make_float2(sk, sk);
      const float by = dY + (float)(4 * cc), bx = dX + (float)(4 * cc);
#pragma unroll
      for (int i = 0; i < 4; i += 2) {
        const float2 off = make_float2((float)i, (float)(i + 1));
        float2 ty = __fmul2_rn(__fadd2_rn(make_float2(by, by), off), sk2);
        float2 tx = __fmul2_rn(__fadd2_rn(make_float2(bx, bx), off), sk2);
        ty = __fmul2_rn(ty, make_float2(-ty.x, -ty.y));
        tx = __fmul2_rn(tx, make_float2(-tx.x, -tx.y));
        const float2 ey = __fmul2_rn(make_float2(ex2_approx(ty.x), ex2_approx(ty.y)), make_float2(sY, sY));
        const float2 ex = make_float2(ex2_approx(tx.x), ex2_approx(tx.y));
        vy[i] = (mY >> i) & 1u ? ey.x : 0.f;
        vy[i + 1] = (mY >> (i + 1)) & 1u ? ey.y : 0.f;
        vx[i] = (mX >> i) & 1u ? ex.x : 0.f;
        vx[i + 1] = (mX >> (i + 1)) & 1u ? ex.y : 0.f;
      }
    } else {
      const float by = dY + (float)(4 * cc), bx = dX + (float)(4 * cc);
      float t = (by - 0.5f) * kint, e = edge_erfc(t), u = (bx - 0.5f) * kint, f = edge_erfc(u);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float tn = (by + (float)i + 0.5f) * kint, en = edge_erfc(tn);
        const float un = (bx + (float)i + 0.5f) * kint, fn = edge_erfc(un);
        vy[i] = (mY >> i) & 1u ? sY * pix_mass(t, e, tn, en) : 0.f;
        vx[i] = (mX >> i) & 1u ? pix_mass(u, f, un, fn) : 0.f;
        t = tn;
        e = en;
        u = un;
        f = fn;
      }
    }
    if (vY) slotY[(2 * bY + (int)cc) & 7] = make_float4(vy[0], vy[1], vy[2], vy[3]);
    if (vX) slotX[(2 * bX + (int)cc) & 7] = make_float4(vx[0], vx[1], vx[2], vx[3]);
  }
}

// a record load the compiler keeps where it is written (ahead of the chunk that uses it)
__device__ __forceinline__ StarRec t8_ldrec(const StarRec* p) {
  StarRec r;
  asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(*reinterpret_cast<uint32_t*>(&r.x)), "=r"(*reinterpret_cast<uint32_t*>(&r.y)),
                 "=r"(*reinterpret_cast<uint32_t*>(&r.s)), "=r"(r.lo)
               : "l"(p)
               : "memory");
  return r;
}

template <bool INTEG>
__device__ void t8_producer(T8Smem& S, const StarRec* __restrict__ srec, const FrameParams& fp,
                            const WorkItem* __restrict__ items, uint32_t nitems, uint32_t* __restrict__ next_ctr,
                            const uint32_t* __restrict__ sbin, const uint32_t* __restrict__ sext, uint32_t items_cap) {
  const int pt = threadIdx.x - T8_CT;
  const int R = fp.R;
  const WorkItem none = {0u, 0u, 0u, ITEM_WHOLE};
  // the CTA's item sequence comes from a global counter (dynamic balance; the image does not depend on it)
  if (pt == 0) S.next_item = atomicAdd(next_ctr, 1u);
  prod_sync();
  uint32_t it = S.next_item;
  WorkItem cur = it < nitems ? items[it] : none;
  // this thread's two words of the next segment's bin-start row (loaded one segment ahead)
  auto bin_row = [&](uint32_t sid, uint32_t& b0, uint32_t& b1) {
    const uint32_t* row = sbin + (size_t)sid * T8_HDR;
    b0 = pt <= T8_NBIN ? __ldcg(&row[pt]) : 0u;
    b1 = pt + T8_PT <= T8_NBIN ? __ldcg(&row[pt + T8_PT]) : 0u;
  };
  uint32_t bA = 0, bB = 0;
  if (it < nitems) bin_row(it, bA, bB);
  uint32_t q = 0;  // global chunk sequence number
  while (it < nitems) {
    const uint32_t nseg = seg_count(cur);
    const int tx = (int)(cur.tile % (uint32_t)fp.ntx), ty = (int)(cur.tile / (uint32_t)fp.ntx);
    const int X0 = tx * TILE_W, IY0 = fp.row0 + ty * TILE_H;
    uint32_t nit = it;
    WorkItem nxt = none;
    for (uint32_t s = 0; s < nseg; ++s) {
      const uint32_t L = seg_len(cur, s);
      const StarRec* rs = srec + cur.jb + s * (uint32_t)T8_SEG;  // this segment, sorted by corner bin
      T8_T(pa);
      prod_sync();  // the previous segment's bin starts have been copied into its stages; S.next_item was read
      if (pt <= T8_NBIN) S.binstart[pt] = bA;
      if (pt + T8_PT <= T8_NBIN) S.binstart[pt + T8_PT] = bB;
      if (s == 0) {
        if (pt == 0) S.next_item = atomicAdd(next_ctr, 1u);
        if (pt < 8) S.gsum[pt] = 0u;
      }
      prod_sync();
      if (s == 0) {
        nit = S.next_item;
        // balance the consumer warps: block (B, Q) = (pt >> 4, pt & 15) has the candidates of its three ranges;
        // the 8 groups of 4 x 4 blocks, sorted by count, are dealt to the 4 warps as (heaviest k, lightest k)
        if (pt < T8_NB * T8_NQ) {
          const int B = pt >> 4, Q = pt & 15;
          uint32_t cnt = 0;
#pragma unroll
          for (int k = 0; k < 3; ++k) {
            const int kb = (Q + k) * T8_KB + B;
            cnt += S.binstart[kb + 3] - S.binstart[kb];
          }
          atomicAdd(&S.gsum[(B >> 2) * 4 + (Q >> 2)], cnt);
        }
      }
      // the segment after this one: the next of this item, else the first of the next item
      if (s + 1 < nseg) {
        bin_row(items_cap + __ldcg(&sext[it]) + s, bA, bB);
      } else if (nit < nitems) {
        nxt = items[nit];
        bin_row(nit, bA, bB);
      }
      if (s == 0) {
        prod_sync();
        if (pt == 0) {
          uint32_t g[8], c[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            g[i] = (uint32_t)i;
            c[i] = S.gsum[i];
          }
#pragma unroll
          for (int i = 1; i < 8; ++i)  // insertion sort, descending count (ties by group index: deterministic)
#pragma unroll
            for (int j = i; j > 0; --j)
              if (c[j] > c[j - 1]) {
                const uint32_t tc = c[j], tg = g[j];
                c[j] = c[j - 1];
                g[j] = g[j - 1];
                c[j - 1] = tc;
                g[j - 1] = tg;
              }
          uint32_t a = 0;
#pragma unroll
          for (int w = 0; w < 4; ++w) a |= (g[w] | g[7 - w] << 4) << (8 * w);
          S.asg = a;
        }
      }
      T8_T(pb);
      T8_ACC(1, pb - pa);
      T8_ACC(5, 1);
      // ---- stratified chunks: chunk c = sorted positions j = c + nch k
      const uint32_t nch = L ? (L + T8_CHUNK - 1) / T8_CHUNK : 1u;
      const uint32_t magic = nch > 1 ? (uint32_t)((0x100000000ull + nch - 1) / nch) : 0u;  // 0: nch == 1
      // star of this thread's row profile: k = pt (consecutive sorted stars per quarter-warp: one corner strip,
      // increasing corner bands -> their ring stores spread over the bank quads); of its column profile: the 8 lanes
      // of a quarter-warp take stars from the 8 eighths of the chunk (different corner strips)
      auto chunk_n = [&](uint32_t c) -> uint32_t {
        return L > c ? (magic ? __umulhi(L - c + nch - 1u, magic) : L - c) : 0u;
      };
      auto kx_of = [&](uint32_t n) -> uint32_t {
        const uint32_t E = (n + 7) / 8, kp = (uint32_t)pt;
        return (kp >> 3) < E ? (kp & 7u) * E + (kp >> 3) : 0xFFFFFFFFu;
      };
      uint32_t n = chunk_n(0), kx = kx_of(n);
      // records of this thread's stars (an invalid one reads position 0 and stores nothing); with 8 producer
      // warps, threads [0, T8_CHUNK) evaluate row profiles and [T8_CHUNK, 2 T8_CHUNK) column profiles
      constexpr bool SPLIT = T8_PT >= 2 * T8_CHUNK;
      const int py = SPLIT ? pt : pt;                       // row-profile star of this thread
      const bool doY = SPLIT ? pt < T8_CHUNK : true, doX = SPLIT ? pt >= T8_CHUNK : true;
      auto kx_of2 = [&](uint32_t nc) -> uint32_t {
        const uint32_t E = (nc + 7) / 8, kp = (uint32_t)(SPLIT ? pt - T8_CHUNK : pt);
        return (kp >> 3) < E ? (kp & 7u) * E + (kp >> 3) : 0xFFFFFFFFu;
      };
      kx = kx_of2(n);
      StarRec ry = {}, rx = {};
      if (L) {
        if (doY) ry = t8_ldrec(rs + ((uint32_t)py < n ? nch * (uint32_t)py : 0u));
        if (doX) rx = t8_ldrec(rs + (kx < n ? nch * kx : 0u));
      }
      for (uint32_t c = 0; c < nch; ++c, ++q) {
        const uint32_t st = q % T8_NS, ph = (q / T8_NS) & 1u;
        T8Stage& T = S.st[st];
        // the next chunk's records, loaded ahead (they do not depend on the stage)
        const uint32_t nn = c + 1 < nch ? chunk_n(c + 1) : 0u, kxn = kx_of2(nn);
        StarRec ryn = ry, rxn = rx;
        if (nn) {
          if (doY) ryn = t8_ldrec(rs + ((uint32_t)py < nn ? c + 1 + nch * (uint32_t)py : 0u));
          if (doX) rxn = t8_ldrec(rs + (kxn < nn ? c + 1 + nch * kxn : 0u));
        }
        T8_T(pe);
        mbar_wait(&S.empty[st], ph ^ 1u);
        T8_T(pf);
#ifndef T8_NOPROF
        if (SPLIT) {
          const uint32_t swp = (uint32_t)(pt >> 2) & 1u;
          if (doY && (uint32_t)py < n)
            t8_axis<INTEG, true>(&T.prof[py][0], lo_y_of(ry.lo) - IY0, ry.y - (float)IY0, ry.s, R, fp.sk, fp.kint, swp);
          if (doX && kx < n)
            t8_axis<INTEG, false>(&T.prof[kx][8], lo_x_of(rx.lo) - X0, rx.x - (float)X0, 1.f, R, fp.sk, fp.kint, swp);
        } else if (n) {
          t8_axis2<INTEG>(&T.prof[pt < T8_CHUNK ? pt : 0][0], lo_y_of(ry.lo) - IY0, ry.y - (float)IY0, ry.s,
                          (uint32_t)pt < n, &T.prof[kx < n ? kx : 0][8], lo_x_of(rx.lo) - X0, rx.x - (float)X0,
                          kx < n, R, fp.sk, fp.kint, (uint32_t)(pt >> 2) & 1u);
        }
#endif
        for (int b = pt; b <= T8_NBIN; b += T8_PT) T.binstart[b] = S.binstart[b];
        if (pt == 0) {
          T.tile = cur.tile;
          T.aux = cur.aux;
          T.flags = (c + 1 == nch ? T8_SEG_LAST : 0u) | (c + 1 == nch && s + 1 == nseg ? T8_ITEM_LAST : 0u);
          T.c = c;
          T.nch = nch;
          T.magic = magic;
          T.seg = s;
          T.asg = S.asg;
        }
        mbar_arrive_warp(&S.full[st]);
        T8_T(pg);
        T8_ACC(3, pf - pe);
        T8_ACC(4, pg - pf);
        T8_ACC(6, 1);
        n = nn;
        kx = kxn;
        ry = ryn;
        rx = rxn;
      }
    }
    it = nit;
    cur = nxt;
  }
  // release the consumers
  const uint32_t st = q % T8_NS, ph = (q / T8_NS) & 1u;
  mbar_wait(&S.empty[st], ph ^ 1u);
  if (pt == 0) S.st[st].flags = T8_STOP;
  mbar_arrive_warp(&S.full[st]);
}

// ------------------------------------------------------------------------------------------------ consumer side

// the lane's pixel row of accumulator row r (0..7); the 16-B halves of the two rings come swapped by sy / sx (the
// bank-quad swizzle): columns of accumulator pair cp are 8 Q + 4 ((cp >> 1) ^ sx) + 2 (cp & 1) + {0, 1}
__device__ __forceinline__ int t8_row(int B, int sy, int r) { return 8 * B + (((r >> 2) ^ sy) << 2) + (r & 3); }

// the lane's 8 values of pixel row 8 B + rr (columns 8 Q .. 8 Q + 7) from its swizzled accumulators: every lane of a
// band then stores the same row in the same instruction (the 4 lanes of a band row of a block group fill one 128-B
// line), instead of rows and halves scattered by the bank-quad swizzle
__device__ __forceinline__ void t8_row_vals(const float2 (&acc)[8][4], int rr, int sy, int sx, float4& lo, float4& hi) {
  float2 a[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) a[k] = sy ? acc[rr ^ 4][k] : acc[rr][k];
  const float4 h0 = make_float4(a[0].x, a[0].y, a[1].x, a[1].y);
  const float4 h1 = make_float4(a[2].x, a[2].y, a[3].x, a[3].y);
  lo = sx ? h1 : h0;
  hi = sx ? h0 : h1;
}

__device__ __forceinline__ void t8_store_fp32(float* __restrict__ out, const FrameParams& fp, const float2 (&acc)[8][4],
                                              int Y0, int X0, int B, int Q, int sy, int sx) {
  const int c0 = X0 + 8 * Q;
  if (c0 >= fp.W) return;
#pragma unroll
  for (int rr = 0; rr < 8; ++rr) {
    const int row = Y0 + 8 * B + rr;
    if (row >= fp.rows) continue;
    float* o = out + (int64_t)row * fp.W + c0;
    float4 lo, hi;
    t8_row_vals(acc, rr, sy, sx, lo, hi);
    if (fp.vec && c0 + 8 <= fp.W) {
      reinterpret_cast<float4*>(o)[0] = lo;
      reinterpret_cast<float4*>(o)[1] = hi;
    } else {
      const float v[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
#pragma unroll
      for (int k = 0; k < 8; ++k)
        if (c0 + k < fp.W) o[k] = v[k];
    }
  }
}

__device__ __forceinline__ void t8_store_gray(void* __restrict__ out_, const FrameParams& fp, const float2 (&acc)[8][4],
                                              int Y0, int X0, int B, int Q, int sy, int sx) {
  const int c0 = X0 + 8 * Q;
  if (c0 >= fp.W) return;
  const float qmax = fp.obits == 8 ? 255.f : 65535.f;
#pragma unroll
  for (int rr = 0; rr < 8; ++rr) {
    const int row = Y0 + 8 * B + rr;
    if (row >= fp.rows) continue;
    float4 lo, hi;
    t8_row_vals(acc, rr, sy, sx, lo, hi);
    const float v[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
    uint32_t g[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) g[k] = quant1(v[k], qmax);
    const int64_t pix = (int64_t)row * fp.W + c0;
    if (fp.obits == 8) {
      uint8_t* o = reinterpret_cast<uint8_t*>(out_) + pix;
      if (fp.vec && c0 + 8 <= fp.W) {
        *reinterpret_cast<uint2*>(o) =
            make_uint2(g[0] | g[1] << 8 | g[2] << 16 | g[3] << 24, g[4] | g[5] << 8 | g[6] << 16 | g[7] << 24);
      } else {
#pragma unroll
        for (int k = 0; k < 8; ++k)
          if (c0 + k < fp.W) o[k] = (uint8_t)g[k];
      }
    } else {
      uint16_t* o = reinterpret_cast<uint16_t*>(out_) + pix;
      if (fp.vec && c0 + 8 <= fp.W) {
        *reinterpret_cast<uint4*>(o) =
            make_uint4(g[0] | g[1] << 16, g[2] | g[3] << 16, g[4] | g[5] << 16, g[6] | g[7] << 16);
      } else {
#pragma unroll
        for (int k = 0; k < 8; ++k)
          if (c0 + k < fp.W) o[k] = (uint16_t)g[k];
      }
    }
  }
}

// the lane's 64 values of a 128 x 64 fp32 tile buffer (partial tiles, the segment scratch): row-major, 8 x 8 block
__device__ __forceinline__ float4* t8_buf_row(float* tb, int B, int Q, int sy, int r) {
  return reinterpret_cast<float4*>(tb + t8_row(B, sy, r) * TILE_W + 8 * Q);
}
__device__ __forceinline__ void t8_buf_write(float* tb, const float2 (&acc)[8][4], int B, int Q, int sy, int sx) {
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    float4* o = t8_buf_row(tb, B, Q, sy, r);
    const float4 h0 = make_float4(acc[r][0].x, acc[r][0].y, acc[r][1].x, acc[r][1].y);
    const float4 h1 = make_float4(acc[r][2].x, acc[r][2].y, acc[r][3].x, acc[r][3].y);
    __stcg(o, sx ? h1 : h0);
    __stcg(o + 1, sx ? h0 : h1);
  }
}
// acc = buf + acc (in the buffer's summation position: earlier segments / parts first)
__device__ __forceinline__ void t8_buf_add(const float* tb, float2 (&acc)[8][4], int B, int Q, int sy, int sx) {
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    const float4* o = t8_buf_row(const_cast<float*>(tb), B, Q, sy, r);
    const float4 a = __ldcg(o), b = __ldcg(o + 1);
    const float4 h0 = sx ? b : a, h1 = sx ? a : b;
    acc[r][0] = __fadd2_rn(make_float2(h0.x, h0.y), acc[r][0]);
    acc[r][1] = __fadd2_rn(make_float2(h0.z, h0.w), acc[r][1]);
    acc[r][2] = __fadd2_rn(make_float2(h1.x, h1.y), acc[r][2]);
    acc[r][3] = __fadd2_rn(make_float2(h1.z, h1.w), acc[r][3]);
  }
}

// The lane's 8 x 8 block: warp w of the consumer warpgroup takes two 4 x 4 block groups of the tile (the item's
// balanced assignment asg: bits [8w, 8w+4) and [8w+4, 8w+8)), lanes 0-15 the first, 16-31 the second; inside a
// group, the diagonal quarter-warp layout (quarter 0: (B, Q) offsets (i, i) and (i, i+2); quarter 1: (i, i+1) and
// (i, i+3)) that makes every LDS.128 phase hit 8 distinct bank quads.
struct T8Geom {
  int B, Q;
};
__device__ __forceinline__ T8Geom t8_geom(uint32_t asg) {
  const int lane = (int)(threadIdx.x & 31u), warp = (int)(threadIdx.x >> 5);
  const int g = (int)((asg >> (8 * warp + 4 * (lane >> 4))) & 15u);
  const int m = lane & 15, qt = m >> 3, i4 = m & 3, e = (m >> 2) & 1;
  T8Geom G;
  G.B = 4 * (g >> 2) + i4;
  G.Q = 4 * (g & 3) + ((i4 + qt + 2 * e) & 3);
  return G;
}

__device__ void t8_consumer(T8Smem& S, const FrameParams& fp, void* __restrict__ out_,
                            const uint2* __restrict__ split_tab, float* __restrict__ part_buf,
                            uint32_t* __restrict__ done, float* __restrict__ seg_scratch) {
  __shared__ int s_last;
  int B = 0, Q = 0, sy = 0, sx = 0;
  uint32_t oy0 = 0, oy1 = 0, ox0 = 0, ox1 = 0;
  float2 acc[8][4];
#pragma unroll
  for (int r = 0; r < 8; ++r)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[r][k] = make_float2(0.f, 0.f);
  for (uint32_t q = 0;; ++q) {
    const uint32_t st = q % T8_NS, ph = (q / T8_NS) & 1u;
    const T8Stage& T = S.st[st];
    T8_T(qa);
    mbar_wait(&S.full[st], ph);
    T8_T(qb);
    T8_ACC(7, qb - qa);
    const uint32_t flags = T.flags;
    if (flags & T8_STOP) break;
    const uint32_t c = T.c, nch = T.nch, magic = T.magic;
    if (c == 0 && T.seg == 0) {  // a new item: this warp's blocks
      const T8Geom G = t8_geom(T.asg);
      B = G.B;
      Q = G.Q;
      sy = (Q >> 1) & 1;
      sx = (B >> 1) & 1;
      oy0 = 32u * (uint32_t)(B & 3) + 16u * (uint32_t)sy;
      oy1 = oy0 ^ 16u;
      ox0 = 128u + 32u * (uint32_t)(Q & 3) + 16u * (uint32_t)sx;
      ox1 = ox0 ^ 16u;
    }
    // the three candidate ranges (corner strips Q-2, Q-1, Q; bands B-2..B each): the segment's sorted bounds, cut
    // to this chunk (sorted positions j = c + nch k)
    uint32_t a[3], L[3];
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      const int kb = (Q + k) * T8_KB + B;
      const uint32_t u0 = T.binstart[kb] + nch - 1u - c, u1 = T.binstart[kb + 3] + nch - 1u - c;  // ceil((j - c) / nch)
      const uint32_t lo = magic ? __umulhi(u0, magic) : u0, hi = magic ? __umulhi(u1, magic) : u1;
      a[k] = lo;
      L[k] = hi - lo;
    }
    const uint32_t L0 = L[0], L01 = L0 + L[1], Lt = L01 + L[2];
#ifdef T8_NOWALK
    const uint32_t steps = 0;
#else
    const uint32_t steps = __reduce_max_sync(0xFFFFFFFFu, Lt);
#endif
    // software-pipelined walk, two steps per iteration on two register sets: the loads of step t + 1 are issued
    // before the 32 FFMA2 of step t; a lane past its ranges reads the stage's zero slot (its FFMA2 add exact zeros;
    // same bank quads, no branch)
    const char* base = reinterpret_cast<const char*>(&T.prof[0][0]);
    const char* zs = reinterpret_cast<const char*>(&T.zero[0]);
    const uint32_t o0 = a[0] * 256u, o1 = (a[1] - L0) * 256u, o2 = (a[2] - L01) * 256u;
    auto slot = [&](uint32_t t) -> const char* {
      return t < Lt ? base + ((t < L0 ? o0 : (t < L01 ? o1 : o2)) + t * 256u) : zs;
    };
    auto fma_step = [&](const float4& ya, const float4& yb, const float4& xa, const float4& xb) {
      const float gy[8] = {ya.x, ya.y, ya.z, ya.w, yb.x, yb.y, yb.z, yb.w};
      const float2 gx[4] = {make_float2(xa.x, xa.y), make_float2(xa.z, xa.w), make_float2(xb.x, xb.y),
                            make_float2(xb.z, xb.w)};
#pragma unroll
      for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[r][k] = __ffma2_rn(make_float2(gy[r], gy[r]), gx[k], acc[r][k]);
    };
#define T8_LD4(P, A, BB, C, D)                                  \
  A = *reinterpret_cast<const float4*>((P) + oy0);               \
  BB = *reinterpret_cast<const float4*>((P) + oy1);              \
  C = *reinterpret_cast<const float4*>((P) + ox0);               \
  D = *reinterpret_cast<const float4*>((P) + ox1)
#ifdef T8_NOPP
#pragma unroll 1
    for (uint32_t t = 0; t < steps; ++t) {
      const char* p = slot(t);
      float4 ya, yb, xa, xb;
      T8_LD4(p, ya, yb, xa, xb);
      fma_step(ya, yb, xa, xb);
    }
    if (false) {
#else
    if (steps) {
#endif
      float4 ya, yb, xa, xb, za, zb, wa, wb;
      const char* p0 = slot(0);
      T8_LD4(p0, ya, yb, xa, xb);
      uint32_t t = 0;
#pragma unroll 1
      for (; t + 2 <= steps; t += 2) {
        const char* p1 = slot(t + 1);
        T8_LD4(p1, za, zb, wa, wb);
        fma_step(ya, yb, xa, xb);
        const char* p2 = slot(t + 2);
        T8_LD4(p2, ya, yb, xa, xb);
        fma_step(za, zb, wa, wb);
      }
      if (t < steps) fma_step(ya, yb, xa, xb);
    }
#undef T8_LD4
    const uint32_t tile = T.tile, aux = T.aux, seg = T.seg;
    mbar_arrive_warp(&S.empty[st]);
    T8_T(qc);
    T8_ACC(8, qc - qb);
    T8_ACC(10, 1);
    if (!(flags & T8_SEG_LAST)) continue;
    float* scratch = seg_scratch + (size_t)blockIdx.x * (TILE_W * TILE_H);
    if (!(flags & T8_ITEM_LAST)) {
      // end of a segment of a long unsplit item: keep the partial sum (earlier segments first) in the CTA's scratch
      if (seg > 0) t8_buf_add(scratch, acc, B, Q, sy, sx);
      t8_buf_write(scratch, acc, B, Q, sy, sx);
#pragma unroll
      for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[r][k] = make_float2(0.f, 0.f);
      continue;
    }
    if (seg > 0) t8_buf_add(scratch, acc, B, Q, sy, sx);
    const int tx = (int)(tile % (uint32_t)fp.ntx), ty = (int)(tile / (uint32_t)fp.ntx);
    bool write = true;
    if (aux != ITEM_WHOLE) {
      // one part of a split heavy tile: partial to the pool; the last part to finish sums the parts in part order
      const uint2 sp = split_tab[aux >> 12];
      t8_buf_write(part_buf + (size_t)(sp.x + (aux & 0xFFFu)) * (TILE_W * TILE_H), acc, B, Q, sy, sx);
      __threadfence();
      cons_sync();
      if (threadIdx.x == 0) s_last = atomicAdd(&done[aux >> 12], 1u) == sp.y - 1;
      cons_sync();
      write = s_last != 0;
      if (write) {
        __threadfence();
#pragma unroll
        for (int r = 0; r < 8; ++r)
#pragma unroll
          for (int k = 0; k < 4; ++k) acc[r][k] = make_float2(0.f, 0.f);
        for (uint32_t k = 0; k < sp.y; ++k)
          t8_buf_add(part_buf + (size_t)(sp.x + k) * (TILE_W * TILE_H), acc, B, Q, sy, sx);
      }
    }
    if (write) {
      if (fp.ndst == 0) {
        if (fp.obits == 0)
          t8_store_fp32(reinterpret_cast<float*>(out_), fp, acc, ty * TILE_H, tx * TILE_W, B, Q, sy, sx);
        else
          t8_store_gray(out_, fp, acc, ty * TILE_H, tx * TILE_W, B, Q, sy, sx);
      } else {
        for (int d = 0; d < fp.ndst; ++d) t8_store_fp32(fp.dst[d], fp, acc, ty * TILE_H, tx * TILE_W, B, Q, sy, sx);
      }
    }
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[r][k] = make_float2(0.f, 0.f);
    T8_T(qd);
    T8_ACC(9, qd - qc);
  }
}

template <bool INTEG>
__global__ void __launch_bounds__(T8_THREADS, 2)
    k_tile8(const StarRec* __restrict__ srec, FrameParams fp, void* __restrict__ out_,
            const WorkItem* __restrict__ items, const uint2* __restrict__ split_tab, float* __restrict__ part_buf,
            uint32_t* __restrict__ done, float* __restrict__ seg_scratch, Header* hdr,
            const uint32_t* __restrict__ sbin, const uint32_t* __restrict__ sext, uint32_t items_cap) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T8Smem& S = *reinterpret_cast<T8Smem*>(smem_raw);
  const int tid = threadIdx.x;
#ifdef T8_TIMING
  if ((tid & 31) == 0)
    for (int k = 0; k < 16; ++k) t8_acc_slot()[k] = 0ull;
#endif
  for (int i = tid; i < T8_NS * 16; i += T8_THREADS) S.st[i / 16].zero[i % 16] = make_float4(0.f, 0.f, 0.f, 0.f);
  if (tid < T8_NS) {
    mbar_init(&S.full[tid], T8_PROD * T8_ARRIVALS_PER_WARP);
    mbar_init(&S.empty[tid], T8_CONS * T8_ARRIVALS_PER_WARP);
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  T8_T(k0);
  const uint32_t nitems = __ldcg(&hdr->nitems);
  // registers: the launch gives every thread 128; the producer warpgroup hands 40 per thread to the consumer
  // warpgroup (64 accumulators + 2 x 16 profile operands per lane live across the software-pipelined walk)
  if (tid >= T8_CT) {
    if (T8_PROD == 8)
      asm volatile("setmaxnreg.dec.sync.aligned.u32 48;" ::: "memory");
    else
      asm volatile("setmaxnreg.dec.sync.aligned.u32 88;" ::: "memory");
    t8_producer<INTEG>(S, srec, fp, items, nitems, &hdr->next_item, sbin, sext, items_cap);
  } else {
    if (T8_PROD == 8)
      asm volatile("setmaxnreg.inc.sync.aligned.u32 144;" ::: "memory");
    else
      asm volatile("setmaxnreg.inc.sync.aligned.u32 168;" ::: "memory");
    t8_consumer(S, fp, out_, split_tab, part_buf, done, seg_scratch);
  }
  T8_T(k1);
  T8_ACC(tid >= T8_CT ? 11 : 12, k1 - k0);
#ifdef T8_TIMING
  if ((tid & 31) == 0)
    for (int k = 0; k < 16; ++k) atomicAdd(&g_t8_prof[k], t8_acc_slot()[k]);
#endif
}

}  // namespace

#ifdef T8_TIMING
extern "C" int starsim_debug_t8_timing(double* out16, int reset) {
  unsigned long long h[16];
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(h, g_t8_prof, sizeof(h));
  for (int i = 0; i < 16; ++i) out16[i] = (double)h[i];
  if (reset) {
    unsigned long long z[16] = {};
    cudaMemcpyToSymbol(g_t8_prof, z, sizeof(z));
  }
  return 0;
}
#endif

size_t tile8_scratch_floats(int num_sms) { return (size_t)4 * num_sms * TILE_W * TILE_H; }  // a slot per CTA

void init_tile8_kernel() {
  cudaFuncSetAttribute(k_tile8<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)T8_SMEM_LAUNCH);
  cudaFuncSetAttribute(k_tile8<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)T8_SMEM_LAUNCH);
}

size_t tile8_sbin_words(int64_t ntiles, int part_cap, int64_t pairs) {
  return (size_t)(ntiles + part_cap + pairs / T8_SEG + 1) * T8_HDR;
}

void launch_t8sort(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, const WorkItem* items,
                   int part_cap, Header* hdr, StarRec* srec, uint32_t* sbin, uint32_t* sext, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  k_t8sort<<<(unsigned)(ntiles + part_cap), TS_THREADS, 0, st>>>(ids, rec, fp, items, hdr, srec, sbin, sext,
                                                                  (uint32_t)(ntiles + part_cap));
}

void launch_tile8(const StarRec* srec, const FrameParams& fp, void* out, const WorkItem* items,
                  const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, float* seg_scratch,
                  Header* hdr, const uint32_t* sbin, const uint32_t* sext, int num_sms, cudaStream_t st) {
  const int64_t ntiles = (int64_t)fp.ntx * fp.nty;
  if (ntiles <= 0) return;
  const int64_t grid = std::min<int64_t>(ntiles + part_cap, (int64_t)2 * num_sms);  // persistent, 2 CTAs per SM
  if (fp.psf)
    k_tile8<true><<<(unsigned)grid, T8_THREADS, T8_SMEM_LAUNCH, st>>>(srec, fp, out, items, split_tab, part_buf, done,
                                                                      seg_scratch, hdr, sbin, sext,
                                                                      (uint32_t)(ntiles + part_cap));
  else
    k_tile8<false><<<(unsigned)grid, T8_THREADS, T8_SMEM_LAUNCH, st>>>(srec, fp, out, items, split_tab, part_buf, done,
                                                                       seg_scratch, hdr, sbin, sext,
                                                                       (uint32_t)(ntiles + part_cap));
}

}  // namespace starsim
