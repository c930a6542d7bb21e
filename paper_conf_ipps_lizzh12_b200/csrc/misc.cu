// The comparison kernels (the paper's atomic star-centric design and its lookup-table variant), the output quantiser
// and the AoS upload split.
#include "common.cuh"
#include "launch.h"

namespace starsim {

// ---------------------------------------------------------------------------------------------------------------
// k_atomic -- the paper's parallel simulator (Fig. 6) re-shaped for sm_100a: one warp per star
// (the paper used one block per star and one thread per ROI pixel, Fig. 4).  Lane 0 computes the
// brightness once (Fig. 6 step 5) in fp64; the separable profiles gx, s'*gy are staged in shared memory (one
// MUFU.EX2 per ROI column / row instead of one 2-D exp per pixel); each lane then adds g*mu into its ROI pixels with
// a global fp32 reduction (Fig. 6 step 8: atomicAdd -> REDG.E.ADD.F32).  The image must be zeroed first.
// ---------------------------------------------------------------------------------------------------------------
constexpr int ATOM_WARPS = 8;

template <bool CIRC>  // NEXT-3: the pixel circle (reading R21) instead of the square ROI
__global__ void __launch_bounds__(ATOM_WARPS * 32) k_atomic(const float* __restrict__ X, const float* __restrict__ Y,
                                                            const float* __restrict__ M, int64_t n, FrameParams fp,
                                                            float* __restrict__ out) {
  extern __shared__ float s_prof[];  // per warp: gx[R] then gy[R]
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t i = (int64_t)blockIdx.x * ATOM_WARPS + warp;
  if (i >= n) return;
  const float x = X[i], y = Y[i], m = M[i];
  const float R = (float)fp.R;
  if (!(isfinite(x) && isfinite(y) && isfinite(m))) return;
  if (!(x > -R - 2.f && x < (float)fp.W + R + 2.f && y > (float)fp.row0 - R - 2.f &&
        y < (float)(fp.row0 + fp.rows) + R + 2.f))
    return;
  const int lx = roi_lo_exact(x, fp.R), ly = roi_lo_exact(y, fp.R);
  const int cx0 = max(lx, 0), cx1 = min(lx + fp.R - 1, fp.W - 1);
  const int cy0 = max(ly, fp.row0), cy1 = min(ly + fp.R - 1, fp.row0 + fp.rows - 1);
  if (cx0 > cx1 || cy0 > cy1) return;
  const int w = cx1 - cx0 + 1, h = cy1 - cy0 + 1;
  float s = 0.f;
  if (lane == 0) s = (float)(fp.s_scale * pow(2.512, -(double)m));
  s = __shfl_sync(0xffffffffu, s, 0);
  float* gx = s_prof + warp * 2 * fp.R;
  float* gy = gx + fp.R;
  if (!fp.psf) {
    for (int c = lane; c < w; c += 32) {
      const float d = (float)(cx0 + c) - x;
      const float e = d * fp.sk;
      gx[c] = ex2_approx(-(e * e));
    }
    for (int r = lane; r < h; r += 32) {
      const float d = (float)(cy0 + r) - y;
      const float e = d * fp.sk;
      gy[r] = s * ex2_approx(-(e * e));
    }
  } else {  // NEXT-2: pixel-integrated PSF, the pixel's 1-D masses between its edges
    for (int c = lane; c < w; c += 32) {
      const float d = (float)(cx0 + c) - x, ta = (d - 0.5f) * fp.kint, tb = (d + 0.5f) * fp.kint;
      gx[c] = pix_mass(ta, edge_erfc(ta), tb, edge_erfc(tb));
    }
    for (int r = lane; r < h; r += 32) {
      const float d = (float)(cy0 + r) - y, ta = (d - 0.5f) * fp.kint, tb = (d + 0.5f) * fp.kint;
      gy[r] = s * pix_mass(ta, edge_erfc(ta), tb, edge_erfc(tb));
    }
  }
  __syncwarp();
  const float inv_w = 1.0f / (float)w;
  float* o = out + (int64_t)(cy0 - fp.row0) * fp.W + cx0;
  for (int p = lane; p < w * h; p += 32) {
    const int r = __float2int_rz(((float)p + 0.5f) * inv_w);
    const int c = p - r * w;
    if (CIRC && !in_roi_circle(cy0 + r - ly, cx0 + c - lx, fp.R)) continue;  // NEXT-3: the pixel circle
    atomicAdd(o + (int64_t)r * fp.W + c, gy[r] * gx[c]);
  }
}

void launch_atomic(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, float* out,
                   cudaStream_t st) {
  if (n <= 0) return;
  const unsigned blocks = (unsigned)((n + ATOM_WARPS - 1) / ATOM_WARPS);
  const size_t smem = sizeof(float) * 2 * fp.R * ATOM_WARPS;
  if (fp.roi)
    k_atomic<true><<<blocks, ATOM_WARPS * 32, smem, st>>>(x, y, m, n, fp, out);
  else
    k_atomic<false><<<blocks, ATOM_WARPS * 32, smem, st>>>(x, y, m, n, fp, out);
}

// ---------------------------------------------------------------------------------------------------------------
// k_lut -- NEXT-4: the paper's adaptive simulator (Fig. 8) re-shaped for sm_100a.  The paper
// pre-builds a lookup table of a star's intensity matrix over its ROI (per magnitude) and replaces the per-pixel
// evaluation of Eqs. 1-2 by table reads.  Here the R x R matrix of Eq. 2 for a star at the centre of its ROI is
// built once per CTA in shared memory (the magnitude only scales it, so one matrix times the star's s' is the
// paper's 3-D table exactly), and each warp adds s' * LUT[r][c] into its star's ROI pixels with global fp32
// reductions (reading R20: the star sits at its ROI's centre -- exact for stars on pixel centres, odd R).
// ---------------------------------------------------------------------------------------------------------------
template <bool CIRC>
__global__ void __launch_bounds__(ATOM_WARPS * 32) k_lut(const float* __restrict__ X, const float* __restrict__ Y,
                                                         const float* __restrict__ M, int64_t n, FrameParams fp,
                                                         float* __restrict__ out) {
  extern __shared__ float s_lut[];  // [R][R], then the 1-D centred profile [R]
  const int R = fp.R;
  float* g1 = s_lut + R * R;
  const float cen = 0.5f * (float)(R - 1);  // exact
  for (int k = threadIdx.x; k < R; k += blockDim.x) {
    const float d = (float)k - cen;  // exact
    if (!fp.psf) {
      const float e = d * fp.sk;
      g1[k] = ex2_approx(-(e * e));
    } else {
      const float ta = (d - 0.5f) * fp.kint, tb = (d + 0.5f) * fp.kint;
      g1[k] = pix_mass(ta, edge_erfc(ta), tb, edge_erfc(tb));
    }
  }
  __syncthreads();
  for (int k = threadIdx.x; k < R * R; k += blockDim.x) s_lut[k] = g1[k / R] * g1[k % R];
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t i = (int64_t)blockIdx.x * ATOM_WARPS + warp;
  if (i >= n) return;
  const float x = X[i], y = Y[i], m = M[i];
  const float Rf = (float)R;
  if (!(isfinite(x) && isfinite(y) && isfinite(m))) return;
  if (!(x > -Rf - 2.f && x < (float)fp.W + Rf + 2.f && y > (float)fp.row0 - Rf - 2.f &&
        y < (float)(fp.row0 + fp.rows) + Rf + 2.f))
    return;
  const int lx = roi_lo_exact(x, R), ly = roi_lo_exact(y, R);
  const int cx0 = max(lx, 0), cx1 = min(lx + R - 1, fp.W - 1);
  const int cy0 = max(ly, fp.row0), cy1 = min(ly + R - 1, fp.row0 + fp.rows - 1);
  if (cx0 > cx1 || cy0 > cy1) return;
  const int w = cx1 - cx0 + 1, h = cy1 - cy0 + 1;
  float s = 0.f;
  if (lane == 0) s = (float)(fp.s_scale * pow(2.512, -(double)m));  // Eq. 1, the table's magnitude axis
  s = __shfl_sync(0xffffffffu, s, 0);
  const float* lut = s_lut + (cy0 - ly) * R + (cx0 - lx);
  const float inv_w = 1.0f / (float)w;
  float* o = out + (int64_t)(cy0 - fp.row0) * fp.W + cx0;
  for (int p = lane; p < w * h; p += 32) {
    const int r = __float2int_rz(((float)p + 0.5f) * inv_w);
    const int c = p - r * w;
    if (CIRC && !in_roi_circle(cy0 + r - ly, cx0 + c - lx, R)) continue;  // NEXT-3: the pixel circle
    atomicAdd(o + (int64_t)r * fp.W + c, s * lut[r * R + c]);
  }
}

void launch_lut(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, float* out,
                cudaStream_t st) {
  if (n <= 0) return;
  const unsigned blocks = (unsigned)((n + ATOM_WARPS - 1) / ATOM_WARPS);
  const size_t smem = sizeof(float) * (size_t)(fp.R * fp.R + fp.R);
  if (fp.roi)
    k_lut<true><<<blocks, ATOM_WARPS * 32, smem, st>>>(x, y, m, n, fp, out);
  else
    k_lut<false><<<blocks, ATOM_WARPS * 32, smem, st>>>(x, y, m, n, fp, out);
}

// ---------------------------------------------------------------------------------------------------------------
// k_quantize -- the Output stage on an fp32 image: quant1 (common.cuh) per pixel, 4 per thread.
// ---------------------------------------------------------------------------------------------------------------
template <int BITS>
__global__ void k_quantize(const float* __restrict__ img, int64_t npix, void* __restrict__ out) {
  const float qmax = BITS == 8 ? 255.f : 65535.f;
  const int64_t n4 = npix / 4;
  const bool aligned = ((reinterpret_cast<uintptr_t>(img) & 15) == 0) &&
                       ((reinterpret_cast<uintptr_t>(out) & (BITS == 8 ? 3 : 7)) == 0);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (aligned) {
    for (; i < n4; i += stride) {
      const float4 v = reinterpret_cast<const float4*>(img)[i];
      const uint32_t a = quant1(v.x, qmax), b = quant1(v.y, qmax), c = quant1(v.z, qmax), d = quant1(v.w, qmax);
      if (BITS == 8)
        reinterpret_cast<uint32_t*>(out)[i] = a | (b << 8) | (c << 16) | (d << 24);
      else
        reinterpret_cast<uint2*>(out)[i] = make_uint2(a | (b << 16), c | (d << 16));
    }
    i = n4 * 4 + ((int64_t)blockIdx.x * blockDim.x + threadIdx.x);
  } else {
    i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  }
  for (; i < npix; i += stride) {
    const uint32_t q = quant1(img[i], qmax);
    if (BITS == 8) reinterpret_cast<uint8_t*>(out)[i] = (uint8_t)q;
    else reinterpret_cast<uint16_t*>(out)[i] = (uint16_t)q;
  }
}

void launch_quantize(const float* img, int64_t npix, int bits, void* out, int num_sms, cudaStream_t st) {
  if (npix <= 0) return;
  int64_t want = (npix / 4 + 255) / 256 + 1;
  const int64_t cap = (int64_t)num_sms * 16;
  if (want > cap) want = cap;
  if (bits == 8) k_quantize<8><<<(unsigned)want, 256, 0, st>>>(img, npix, out);
  else k_quantize<16><<<(unsigned)want, 256, 0, st>>>(img, npix, out);
}

// ---------------------------------------------------------------------------------------------------------------
// k_split_aos -- the paper's star record {mag, posX, posY} -> device SoA x, y, mag.
// ---------------------------------------------------------------------------------------------------------------
__global__ void k_split_aos(const float* __restrict__ aos, int64_t n, float* __restrict__ x, float* __restrict__ y,
                            float* __restrict__ m) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const float a = aos[3 * i], b = aos[3 * i + 1], c = aos[3 * i + 2];
    m[i] = a;
    x[i] = b;
    y[i] = c;
  }
}

void launch_split_aos(const float* aos, int64_t n, float* x, float* y, float* m, int num_sms, cudaStream_t st) {
  if (n <= 0) return;
  int64_t want = (n + 255) / 256;
  const int64_t cap = (int64_t)num_sms * 16;
  if (want > cap) want = cap;
  k_split_aos<<<(unsigned)want, 256, 0, st>>>(aos, n, x, y, m);
}

}  // namespace starsim
