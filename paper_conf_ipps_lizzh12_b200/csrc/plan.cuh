// Step a2's per-tile planning (DESIGN.md §Heavy tiles), shared by k_scan_one / k_scan_b (bin.cu) and the fused scan
// of k_dplace (dbin.cu): tile_off, and k_tile's work items -- a tile whose list is longer than SPLIT_LEN becomes
// ceil(len / SPLIT_LEN) items over consecutive star ranges (its parts), every other tile one item; parts come first.
// The split depends only on the tile's own list, so it is the same for any band decomposition.  If the parts would
// need more than `part_cap` partial buffers, nothing is split.
#pragma once
#include "common.cuh"

namespace starsim {

// The planner's argument word: the partial-buffer pool size | the part length (FrameParams::split) << 16.
__host__ __device__ __forceinline__ int plan_word(int part_cap, int split) { return part_cap | split << 16; }
__device__ __forceinline__ int plan_cap(int plan) { return plan & 0xFFFF; }
__device__ __forceinline__ uint32_t plan_split(int plan) { return (uint32_t)plan >> 16; }

__device__ __forceinline__ uint32_t parts_of(uint32_t len, uint32_t split) {
  if (len <= split) return 0u;
  return min((len + split - 1) / split, 4095u);
}

// Per-tile planning counts, scanned over the tiles: (pairs, parts, split tiles, light tiles).
__device__ __forceinline__ uint4 add4(uint4 a, uint4 b) {
  return make_uint4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w);
}
__device__ __forceinline__ uint4 sub4(uint4 a, uint4 b) {
  return make_uint4(a.x - b.x, a.y - b.y, a.z - b.z, a.w - b.w);
}
__device__ __forceinline__ uint4 tile_counts(uint32_t c, uint32_t split) {
  const uint32_t np = parts_of(c, split);
  return make_uint4(c, np, np ? 1u : 0u, c <= (uint32_t)LITE_MAX ? 1u : 0u);
}

__device__ __forceinline__ uint4 warp_incl_scan4(uint4 v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t x = __shfl_up_sync(0xffffffffu, v.x, o), y = __shfl_up_sync(0xffffffffu, v.y, o),
                   z = __shfl_up_sync(0xffffffffu, v.z, o), w = __shfl_up_sync(0xffffffffu, v.w, o);
    if (lane >= o) v = add4(v, make_uint4(x, y, z, w));
  }
  return v;
}

// The header of a plan from the totals ta of tile_counts: parts only if they fit the partial-buffer pool; items =
// parts, then heavy whole tiles, then light whole tiles (from lite0 on).
__device__ __forceinline__ void plan_header(Header* hdr, uint32_t* __restrict__ tile_off, int64_t ntiles, uint4 ta,
                                            int part_cap) {
  const bool split_on = ta.y <= (uint32_t)part_cap;
  const uint32_t nparts = split_on ? ta.y : 0u, nsplit = split_on ? ta.z : 0u;
  hdr->P = ta.x;
  tile_off[ntiles] = ta.x;
  hdr->nitems = nparts + (uint32_t)ntiles - nsplit;
  hdr->nsplit = nsplit;
  hdr->lite0 = nparts + (uint32_t)ntiles - nsplit - ta.w;
  hdr->next_item = 0u;
  hdr->next_seg = 0u;
}

// Tile t with c stars: (run, pb, si, li) = (pairs, parts, split tiles, light tiles) of the tiles before it on entry,
// after it on return.  Writes tile_off[t], its items (and split table entry, zeroed completion counter, if it is
// split).  Light tiles (c <= LITE_MAX: never split) take the items from lite0 = nparts + heavy whole tiles on.
__device__ __forceinline__ void plan_tile(uint32_t t, uint32_t c, uint32_t& run, uint32_t& pb, uint32_t& si,
                                          uint32_t& li, uint32_t nparts, uint32_t lite0, bool split_on,
                                          uint32_t* __restrict__ tile_off, WorkItem* __restrict__ items,
                                          uint2* __restrict__ split_tab, uint32_t* __restrict__ done,
                                          uint32_t split) {
  tile_off[t] = run;
  const uint32_t np = split_on ? parts_of(c, split) : 0u;
  if (np) {
    split_tab[si] = make_uint2(pb, np);
    done[si] = 0u;  // the parts' completion counter (k_tile)
    // parts start at multiples of split from the list start: the same boundaries at which a tile kernel that
    // processes the whole (unsplit) list cuts it into segments, so split and unsplit give the same sums
    for (uint32_t j = 0; j < np; ++j)
      items[pb + j] = WorkItem{t, run + j * split, min(run + c, run + (j + 1) * split), (si << 12) | j};
    pb += np;
    ++si;
  } else if (c <= (uint32_t)LITE_MAX) {
    items[lite0 + li] = WorkItem{t, run, run + c, ITEM_WHOLE};
    ++li;
  } else {
    // heavy whole tiles follow the parts, in tile order: index = nparts + (tiles before t neither split nor light)
    items[nparts + t - (split_on ? si : 0u) - li] = WorkItem{t, run, run + c, ITEM_WHOLE};
  }
  run += c;
}

}  // namespace starsim
