// Host-side launchers of the sm_100a kernels (internal to libstarsim.so).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

namespace starsim {

void init_kernels();
void launch_bin(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, StarRec* rec,
                uint64_t* pairs, Header* hdr, unsigned long long* status, int bits0, int bits1, cudaStream_t st);
void launch_radix(const uint64_t* in, uint64_t* out, Header* hdr, int pass, int shift, int bits,
                  unsigned long long* status, int64_t pmax, cudaStream_t st);
void launch_offsets(const uint64_t* sorted, const Header* hdr, uint32_t ntiles, uint32_t* tile_off, uint32_t* ids,
                    int64_t pmax, int num_sms, cudaStream_t st);
void launch_tile(const uint32_t* ids, const uint32_t* tile_off, const StarRec* rec, const FrameParams& fp,
                 float* out, cudaStream_t st);
void launch_atomic(const float* x, const float* y, const float* m, int64_t n, const FrameParams& fp, float* out,
                   cudaStream_t st);
void launch_quantize(const float* img, int64_t npix, int bits, void* out, int num_sms, cudaStream_t st);
void launch_split_aos(const float* aos, int64_t n, float* x, float* y, float* m, int num_sms, cudaStream_t st);

}  // namespace starsim
