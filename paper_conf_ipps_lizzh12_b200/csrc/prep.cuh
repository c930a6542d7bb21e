// Per-star preparation shared by the two binning pipelines (bin.cu: atomic slots + per-tile sort; dbin.cu: stable
// counting sort).  Step a1 of DESIGN.md §Path.
#pragma once
#include "common.cuh"

namespace starsim {

// Clipped ROI of a star against the frame columns and the band rows; false if empty.
__device__ __forceinline__ bool clip_roi(const FrameParams& fp, int lx, int ly, int& cx0, int& cx1, int& cy0,
                                         int& cy1) {
  cx0 = max(lx, 0);
  cx1 = min(lx + fp.R - 1, fp.W - 1);
  cy0 = max(ly, fp.row0);
  cy1 = min(ly + fp.R - 1, fp.row0 + fp.rows - 1);
  return cx0 <= cx1 && cy0 <= cy1;
}

// Step a1 for one star: reject non-finite x, y, mag (reading R11); exact ROI origin (reading R7); clip to the frame
// columns and band rows; s' = A 2.512^-m / (2 pi sigma^2) in fp64 (Eq. 1 with the 1/(2 pi sigma^2) of Eq. 2 folded
// in; A only for the integrated PSF), rounded once to fp32.  A culled star gets lo = LO_CULLED, s' = 0; otherwise
// [cx0, cx1] x [cy0, cy1] is its clipped ROI (image columns / rows).
__device__ __forceinline__ StarRec prep_star(float x, float y, float m, const FrameParams& fp, int& cx0, int& cx1,
                                             int& cy0, int& cy1) {
  const float R = (float)fp.R;
  bool ok = isfinite(x) && isfinite(y) && isfinite(m);
  // pre-filter far-off stars (keeps the int conversions exact); the exact test is the clip below
  ok = ok && x > -R - 2.f && x < (float)fp.W + R + 2.f && y > (float)fp.row0 - R - 2.f &&
       y < (float)(fp.row0 + fp.rows) + R + 2.f;
  StarRec r;
  r.x = x;
  r.y = y;
  r.s = 0.f;
  r.lo = LO_CULLED;
  if (ok) {
    const int lx = roi_lo_exact(x, fp.R), ly = roi_lo_exact(y, fp.R);
    if (clip_roi(fp, lx, ly, cx0, cx1, cy0, cy1)) {
      r.lo = ((uint32_t)(uint16_t)(int16_t)lx) | ((uint32_t)(uint16_t)(int16_t)ly << 16);
      r.s = (float)(fp.s_scale * exp2(-(double)m * 1.3288364642295399628));  // 2.512^-m, Eq. 1
    }
  }
  return r;
}

}  // namespace starsim
