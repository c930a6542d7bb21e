// Host-side launchers of the sm_100a kernels (internal to libstarsim.so).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

namespace starsim {

void init_kernels();
void init_tile_kernel();
void init_tile_sb_kernel();
void init_tile_ws_kernel();
void init_tile_wide_kernel();
bool wide_ok(int R);  // k_tile_wide serves this ROI side (SB_MAXR < R <= WIDE_MAXR)
void init_tile8_kernel();
size_t tile8_scratch_floats(int num_sms);
void init_dbin_kernels();
size_t dbin_smem(int ntiles);
int dbin_ctas(int64_t n);          // rows of the count matrix (4,096-star blocks; 1,024-star blocks for small n)
bool dfused_block_ok(int64_t n);  // k_dfused applies (it bins 4,096-star blocks only)
bool dsmall_ok(int64_t n);  // k_dsmall applies (at most DB_CTA stars)
int dfused_max_grid(int num_sms);
cudaError_t launch_dfused(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp,
                          StarRec* rec, uint32_t* C, uint32_t* cnt, int ntiles, uint32_t* tile_off, Header* hdr,
                          WorkItem* items, uint2* split_tab, int part_cap, uint32_t* done, uint32_t* ids,
                          uint32_t* bar, cudaStream_t st);
void launch_dsmall(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                   int ntiles, uint32_t* tile_off, Header* hdr, WorkItem* items, uint2* split_tab, int part_cap,
                   uint32_t* done, uint32_t* ids, cudaStream_t st);
void launch_dcount(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                   uint32_t* codes, uint32_t* C, int ntiles, cudaStream_t st);
void launch_dcolscan(uint32_t* C, int64_t n, int ntiles, uint32_t* cnt, int cstride, const uint32_t* n_dev,
                     cudaStream_t st);
void launch_dplace(const uint32_t* codes, int64_t n, const FrameParams& fp, const uint32_t* C, int ntiles,
                   const uint32_t* cnt, uint32_t* tile_off, Header* hdr, WorkItem* items, uint2* split_tab,
                   int part_cap, uint32_t* done, uint32_t* ids, cudaStream_t st);
void launch_prep(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                 uint32_t* cnt, uint32_t* slots, int tps, cudaStream_t st);
int scan_launches(int64_t ntiles);  // kernels launch_scan enqueues (1 or 2)
void launch_scan(const uint32_t* cnt, int64_t ntiles, uint32_t* tile_off, Header* hdr, WorkItem* items,
                 uint2* split_tab, int part_cap, void* partial, uint32_t* done, cudaStream_t st);
void launch_scatter(const StarRec* rec, int64_t n, const FrameParams& fp, const uint32_t* slots, int tps,
                    const uint32_t* tile_off, uint32_t* ids, cudaStream_t st);
void launch_sortlists(uint32_t* ids, uint32_t* tmp, const uint32_t* tile_off, int64_t ntiles, int64_t n,
                      cudaStream_t st);
void launch_tile(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                 const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                 cudaStream_t st, float* seg_scratch, const uint32_t* tile_off, const StarRec* ws_srec,
                 const uint16_t* ws_cbin);
void launch_tile_sb(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                    const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                    cudaStream_t st, float* seg_scratch, const uint32_t* tile_off);
void launch_tile_ws(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                    const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                    cudaStream_t st, float* seg_scratch, const StarRec* srec, const uint16_t* cbin);
void launch_tile_wide(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, void* out, const WorkItem* items,
                      const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, Header* hdr, int num_sms,
                      cudaStream_t st, float* seg_scratch);
size_t chsort_slots(int64_t ntiles, int64_t pmax);  // rows of k_chsort's bin-start table
size_t chsort_words16();                            // u16 per row
void launch_chsort(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, const WorkItem* items, int part_cap,
                   const Header* hdr, StarRec* srec, uint16_t* cbin, cudaStream_t st);
size_t tile8_sbin_words(int64_t ntiles, int part_cap, int64_t pairs);
void launch_t8sort(const uint32_t* ids, const StarRec* rec, const FrameParams& fp, const WorkItem* items,
                   int part_cap, Header* hdr, StarRec* srec, uint32_t* sbin, uint32_t* sext, cudaStream_t st);
void launch_tile8(const StarRec* srec, const FrameParams& fp, void* out, const WorkItem* items,
                  const uint2* split_tab, float* part_buf, int part_cap, uint32_t* done, float* seg_scratch,
                  Header* hdr, const uint32_t* sbin, const uint32_t* sext, int num_sms, cudaStream_t st);
void launch_atomic(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, float* out,
                   cudaStream_t st);
void launch_lut(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, float* out,
                cudaStream_t st);
void launch_quantize(const float* img, int64_t npix, int bits, void* out, int num_sms, cudaStream_t st);
size_t route_blocks(int64_t n);
void launch_route(const float* x, const float* y, const float* m, int64_t n, int32_t row0, int32_t rows, int32_t R,
                  uint32_t* blk, float* xo, float* yo, float* mo, uint32_t* n_out, cudaStream_t st);
bool sparse_ok(int64_t n, int64_t ntiles);
void launch_srec(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                 uint32_t* box, cudaStream_t st);
void launch_tile_sparse(const StarRec* rec, const uint32_t* box, int64_t n, const FrameParams& fp, void* out,
                        float* seg_scratch, cudaStream_t st);
void launch_split_aos(const float* aos, int64_t n, float* x, float* y, float* m, int num_sms, cudaStream_t st);

}  // namespace starsim
