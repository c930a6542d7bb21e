// Pieces shared by the two tile-accumulation kernels (tile.cu: per-block entry lists, any R; tile_sb.cu: sorted
// corner bins, R <= SB_MAXR).  Both use the same lane layout: warp (wx, B) owns the 64 x 16 block at tile columns
// 64 wx, rows 16 B; lane group q = lane/4 owns the 8-column strip Q = 8 wx + q, lane hq = lane%4 the rows
// 16 B + hq + 4 i (tile.cu, CONTIG = false) or 16 B + 4 hq + i (tile_sb.cu, CONTIG = true), i = 0..3, as 4 x 4 float2
// accumulators (columns 8 Q + 2 k, 8 Q + 2 k + 1 in acc[i][k]).
#pragma once
#include "common.cuh"

namespace starsim {

template <bool CONTIG>
__device__ __forceinline__ int lane_row(int B, int hq, int i) { return CONTIG ? 16 * B + 4 * hq + i : 16 * B + hq + 4 * i; }

// Barrier over the threads that own the tile's accumulators: the whole CTA (NBAR = 0), or -- in the warp-specialised
// kernel, whose producer warps never take part -- named barrier 2 over the first NBAR threads.
template <int NBAR>
__device__ __forceinline__ void acc_barrier() {
  if (NBAR == 0)
    __syncthreads();
  else
    asm volatile("bar.sync 2, %0;" ::"n"(NBAR) : "memory");
}

// A whole tile is written to `out` directly; a part of a split heavy tile (wi.aux != ITEM_WHOLE) writes its
// 128 x 64 partial to part_buf, and the last part to finish (per-tile counter) sums the parts in part order -- a
// fixed order, so the image stays deterministic.  Returns false for a part that is not the last one (nothing left
// to write); on true, acc holds the tile's final sums.  Contains barriers (acc_barrier<NBAR>): every accumulating
// thread calls it.
template <bool CONTIG, int NBAR = 0>
__device__ __forceinline__ bool tile_reduce_parts(float2 (&acc)[4][4], const WorkItem& wi,
                                                  const uint2* __restrict__ split_tab, float* __restrict__ part_buf,
                                                  uint32_t* __restrict__ done, int B, int wx, int q, int hq,
                                                  int* s_last) {
  if (wi.aux == ITEM_WHOLE) return true;
  const int tid = threadIdx.x;
  const uint2 sp = split_tab[wi.aux >> 12];
  SS_CHECK((wi.aux & 0xFFFu) < sp.y && sp.x + sp.y <= (uint32_t)PART_CAP);
  float* pbuf = part_buf + (size_t)(sp.x + (wi.aux & 0xFFFu)) * (TILE_W * TILE_H);
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float4* o = reinterpret_cast<float4*>(pbuf + lane_row<CONTIG>(B, hq, i) * TILE_W + 64 * wx + 8 * q);
    o[0] = make_float4(acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y);
    o[1] = make_float4(acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y);
  }
  __threadfence();
  acc_barrier<NBAR>();
  if (tid == 0) *s_last = atomicAdd(&done[wi.aux >> 12], 1u) == sp.y - 1;
  acc_barrier<NBAR>();
  if (!*s_last) return false;
  __threadfence();
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[i][k] = make_float2(0.f, 0.f);
  for (uint32_t k = 0; k < sp.y; ++k) {
    const float* pk = part_buf + (size_t)(sp.x + k) * (TILE_W * TILE_H);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float4* o = reinterpret_cast<const float4*>(pk + lane_row<CONTIG>(B, hq, i) * TILE_W + 64 * wx + 8 * q);
      const float4 u = __ldcg(o), v = __ldcg(o + 1);
      acc[i][0] = __fadd2_rn(acc[i][0], make_float2(u.x, u.y));
      acc[i][1] = __fadd2_rn(acc[i][1], make_float2(u.z, u.w));
      acc[i][2] = __fadd2_rn(acc[i][2], make_float2(v.x, v.y));
      acc[i][3] = __fadd2_rn(acc[i][3], make_float2(v.z, v.w));
    }
  }
  return true;
}

// Segments (reading R19): a work item longer than SPLIT_LEN -- a heavy tile left whole because the part pool would
// overflow -- is summed exactly as its parts would be: the chunks of each SPLIT_LEN segment accumulate from zero, and
// at the end of every segment but the last the partial sum is added to the thread's slot of the CTA's scratch tile
// (the first segment writes it) and reset; the last segment adds the scratch in front, (((p0 + p1) + p2) + ...),
// the order of tile_reduce_parts.  So split and unsplit heavy tiles give the same bits, and the rounding of each
// sequential fp32 chain is that of <= SPLIT_LEN stars.  The scratch slot is thread-private ([k][tid] float4: the
// thread reads back only what it wrote), no barrier.
// (the accumulating threads are threads 0 .. TILE_THREADS - 1 of every kernel that uses this)
__device__ __forceinline__ float4* seg_slot(float* seg_scratch, int k) {
  return reinterpret_cast<float4*>(seg_scratch + (size_t)blockIdx.x * (TILE_W * TILE_H)) + k * TILE_THREADS +
         threadIdx.x;
}
__device__ __forceinline__ void seg_flush(float2 (&acc)[4][4], float* seg_scratch, bool first) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; k += 2) {
      float4* o = seg_slot(seg_scratch, 2 * i + k / 2);
      float2 a = acc[i][k], b = acc[i][k + 1];
      if (!first) {
        const float4 u = __ldcg(o);
        a = __fadd2_rn(make_float2(u.x, u.y), a);
        b = __fadd2_rn(make_float2(u.z, u.w), b);
      }
      __stcg(o, make_float4(a.x, a.y, b.x, b.y));
      acc[i][k] = make_float2(0.f, 0.f);
      acc[i][k + 1] = make_float2(0.f, 0.f);
    }
}
__device__ __forceinline__ void seg_finish(float2 (&acc)[4][4], float* seg_scratch) {
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int k = 0; k < 4; k += 2) {
      const float4 u = __ldcg(seg_slot(seg_scratch, 2 * i + k / 2));
      acc[i][k] = __fadd2_rn(make_float2(u.x, u.y), acc[i][k]);
      acc[i][k + 1] = __fadd2_rn(make_float2(u.z, u.w), acc[i][k + 1]);
    }
}

__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ WorkItem ld_volatile_item(const WorkItem* p) {
  WorkItem w;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(w.tile), "=r"(w.jb), "=r"(w.je), "=r"(w.aux) : "l"(p));
  return w;
}

// Write the lane's 4 rows x 8 columns of the tile (rows Y0 + lane_row(B, hq, i) of the band, columns col0 .. col0+7):
// fp32, or (fused output stage, NEXT-1) the gray value of each pixel exactly as k_quantize computes it from the same
// fp32 sum, as u8 / u16.  Coalesced: the 8 lane groups of a warp store 8 adjacent 8-pixel runs of a row.
template <bool CONTIG, int OB = -1>  // OB: the output bits when fixed at compile time (0, 8, 16), -1: fp.obits
__device__ __forceinline__ void tile_store_one(const float2 (&acc)[4][4], const FrameParams& fp, void* __restrict__ out_,
                                           int Y0, int col0, int B, int hq) {
  const int obits = OB >= 0 ? OB : fp.obits;
  if (obits == 0) {
    float* out = reinterpret_cast<float*>(out_);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = Y0 + lane_row<CONTIG>(B, hq, i);  // band-relative
      if (row >= fp.rows || col0 >= fp.W) continue;
      float* o = out + (int64_t)row * fp.W + col0;
      if (fp.vec32 && col0 + 8 <= fp.W) {
        // the lane's 8 pixels of the row as one 256-bit store: one whole 32-B sector per lane
        asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(o), "f"(acc[i][0].x),
                     "f"(acc[i][0].y), "f"(acc[i][1].x), "f"(acc[i][1].y), "f"(acc[i][2].x), "f"(acc[i][2].y),
                     "f"(acc[i][3].x), "f"(acc[i][3].y)
                     : "memory");
      } else if (fp.vec && col0 + 8 <= fp.W) {
        reinterpret_cast<float4*>(o)[0] = make_float4(acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y);
        reinterpret_cast<float4*>(o)[1] = make_float4(acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y);
      } else {
        const float v[8] = {acc[i][0].x, acc[i][0].y, acc[i][1].x, acc[i][1].y,
                            acc[i][2].x, acc[i][2].y, acc[i][3].x, acc[i][3].y};
#pragma unroll
        for (int k = 0; k < 8; ++k)
          if (col0 + k < fp.W) o[k] = v[k];
      }
    }
  } else {
    const float qmax = obits == 8 ? 255.f : 65535.f;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = Y0 + lane_row<CONTIG>(B, hq, i);
      if (row >= fp.rows || col0 >= fp.W) continue;
      uint32_t g[8];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        g[2 * k] = quant1(acc[i][k].x, qmax);
        g[2 * k + 1] = quant1(acc[i][k].y, qmax);
      }
      const int64_t pix = (int64_t)row * fp.W + col0;
      if (obits == 8) {
        uint8_t* o = reinterpret_cast<uint8_t*>(out_) + pix;
        if (fp.vec && col0 + 8 <= fp.W) {
          *reinterpret_cast<uint2*>(o) = make_uint2(g[0] | g[1] << 8 | g[2] << 16 | g[3] << 24,
                                                    g[4] | g[5] << 8 | g[6] << 16 | g[7] << 24);
        } else {
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (col0 + k < fp.W) o[k] = (uint8_t)g[k];
        }
      } else {
        uint16_t* o = reinterpret_cast<uint16_t*>(out_) + pix;
        if (fp.vec && col0 + 8 <= fp.W) {
          *reinterpret_cast<uint4*>(o) = make_uint4(g[0] | g[1] << 16, g[2] | g[3] << 16, g[4] | g[5] << 16,
                                                    g[6] | g[7] << 16);
        } else {
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (col0 + k < fp.W) o[k] = (uint16_t)g[k];
        }
      }
    }
  }
}


// The fused output stage (NEXT-1) from an fp32 tile staged in shared memory (row-major TILE_W floats per row): thread t quantises
// 4 consecutive pixels of a row (exactly as k_quantize, quant1) and stores them as one u8x4 / u16x4 word when the
// row run is whole and aligned, else pixel by pixel.
__device__ __forceinline__ void tile_store_gray_staged(const float* __restrict__ buf, const FrameParams& fp,
                                                    void* __restrict__ out_, int Y0, int X0, int TWe, int THe) {
  const float qmax = fp.obits == 8 ? 255.f : 65535.f;
  for (int p = threadIdx.x * 4; p < TILE_W * TILE_H; p += TILE_THREADS * 4) {
    const int r = p / TILE_W, c = p % TILE_W;
    if (r >= THe || c >= TWe) continue;
    const float4 v = *reinterpret_cast<const float4*>(buf + p);
    const uint32_t g0 = quant1(v.x, qmax), g1 = quant1(v.y, qmax), g2 = quant1(v.z, qmax), g3 = quant1(v.w, qmax);
    const int64_t pix = (int64_t)(Y0 + r) * fp.W + X0 + c;
    if (fp.obits == 8) {
      uint8_t* o = reinterpret_cast<uint8_t*>(out_) + pix;
      if (fp.vec && c + 4 <= TWe) {
        *reinterpret_cast<uint32_t*>(o) = g0 | g1 << 8 | g2 << 16 | g3 << 24;
      } else {
        if (c < TWe) o[0] = (uint8_t)g0;
        if (c + 1 < TWe) o[1] = (uint8_t)g1;
        if (c + 2 < TWe) o[2] = (uint8_t)g2;
        if (c + 3 < TWe) o[3] = (uint8_t)g3;
      }
    } else {
      uint16_t* o = reinterpret_cast<uint16_t*>(out_) + pix;
      if (fp.vec && c + 4 <= TWe) {
        *reinterpret_cast<uint2*>(o) = make_uint2(g0 | g1 << 16, g2 | g3 << 16);
      } else {
        if (c < TWe) o[0] = (uint16_t)g0;
        if (c + 1 < TWe) o[1] = (uint16_t)g1;
        if (c + 2 < TWe) o[2] = (uint16_t)g2;
        if (c + 3 < TWe) o[3] = (uint16_t)g3;
      }
    }
  }
}

// The epilogue: into `out_`, or (fused band exchange) into each of the fp.ndst destination frames.
template <bool CONTIG, int OB = -1>
__device__ __forceinline__ void tile_store(const float2 (&acc)[4][4], const FrameParams& fp, void* __restrict__ out_,
                                           int Y0, int col0, int B, int hq) {
  if (fp.ndst == 0) {
    tile_store_one<CONTIG, OB>(acc, fp, out_, Y0, col0, B, hq);
    return;
  }
  for (int g = 0; g < fp.ndst; ++g) tile_store_one<CONTIG, OB>(acc, fp, fp.dst[g], Y0, col0, B, hq);
}

}  // namespace starsim
