// Microbenchmark for the round-2 tile-kernel redesign: SM-cycles per warp step of an 8 x 8
// lane-block walk (4 x LDS.128 of ring-slot profiles + 32 FFMA2 per candidate star), for several lane -> block
// mappings and shared-memory layouts, at 4..16 warps per SM; plus producer-style STS.128 patterns.
//
//   L0 diag   quarter-warp = 4 bands x 4 strips on two diagonals; gy half swizzled by Q bit 1, gx by B bit 1
//   L1 row    quarter-warp = 1 band x 8 strips; gy half swizzled by Q bit 0, gx by B bit 0
//   L2 rand   per-lane random chunk offsets inside the star slot (fully random quads)
//   L3 same   every lane of the warp reads the same star (broadcast upper bound)
//   S0..S2    STS.128 of 12 chunks per lane: conflict-free rotation / random quads / all lanes same quad
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o walk8 walk8.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ float g_sink[1 << 16];

constexpr int NSTAR = 512;             // star slots of 256 B (128 KB)
constexpr int STEPS = 4096;

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

template <int L>
__global__ void __launch_bounds__(512) k_walk(int steps, unsigned long long* cyc) {
  extern __shared__ __align__(16) unsigned char sm[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < NSTAR * 64; i += blockDim.x) reinterpret_cast<float*>(sm)[i] = 1e-3f * (i & 63);
  __syncthreads();
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  int B, Q;
  if (L == 0) {  // two 4x4 groups; quarter 0: Q-B in {0,2}, quarter 1: Q-B in {1,3}
    const int g = lane >> 4, m = lane & 15, qt = m >> 3, i = m & 3, e = (m >> 2) & 1;
    B = i;
    Q = 4 * g + ((i + qt + 2 * e) & 3);
  } else {
    B = lane >> 3;
    Q = lane & 7;
  }
  uint32_t oy0, oy1, ox0, ox1;
  if (L == 0) {
    const uint32_t sy = (Q >> 1) & 1, sx = (B >> 1) & 1;
    oy0 = 32 * (B & 3) + 16 * sy; oy1 = 32 * (B & 3) + 16 * (sy ^ 1);
    ox0 = 128 + 32 * (Q & 3) + 16 * sx; ox1 = 128 + 32 * (Q & 3) + 16 * (sx ^ 1);
  } else if (L == 1 || L == 3) {
    const uint32_t sy = Q & 1, sx = B & 1;
    oy0 = 32 * (B & 3) + 16 * sy; oy1 = 32 * (B & 3) + 16 * (sy ^ 1);
    ox0 = 128 + 32 * (Q & 3) + 16 * sx; ox1 = 128 + 32 * (Q & 3) + 16 * (sx ^ 1);
  } else {
    const uint32_t h = hash32(threadIdx.x * 7 + 1);
    oy0 = 16 * (h & 7); oy1 = 16 * ((h >> 3) & 7); ox0 = 16 * ((h >> 6) & 15); ox1 = 16 * ((h >> 10) & 15);
  }
  uint32_t s = (L == 3) ? (hash32(w + 11) & (NSTAR - 1)) : (hash32(threadIdx.x + 977 * blockIdx.x) & (NSTAR - 1));
  uint32_t p = s * 256u;
  float2 acc[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) acc[i] = make_float2(0.f, 0.f);
  __syncthreads();
  const unsigned long long t0 = clock64();
#pragma unroll 2
  for (int t = 0; t < steps; ++t) {
    float4 ya, yb, xa, xb;
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(ya.x), "=f"(ya.y), "=f"(ya.z), "=f"(ya.w) : "r"(base + p + oy0));
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(yb.x), "=f"(yb.y), "=f"(yb.z), "=f"(yb.w) : "r"(base + p + oy1));
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(xa.x), "=f"(xa.y), "=f"(xa.z), "=f"(xa.w) : "r"(base + p + ox0));
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(xb.x), "=f"(xb.y), "=f"(xb.z), "=f"(xb.w) : "r"(base + p + ox1));
    const float gy[8] = {ya.x, ya.y, ya.z, ya.w, yb.x, yb.y, yb.z, yb.w};
    const float2 gx[4] = {make_float2(xa.x, xa.y), make_float2(xa.z, xa.w), make_float2(xb.x, xb.y), make_float2(xb.z, xb.w)};
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int c = 0; c < 4; ++c) acc[4 * r + c] = __ffma2_rn(make_float2(gy[r], gy[r]), gx[c], acc[4 * r + c]);
    p = (p + 256u) & (NSTAR * 256u - 1u);
  }
  const unsigned long long t1 = clock64();
  float sum = 0.f;
#pragma unroll
  for (int i = 0; i < 32; ++i) sum += acc[i].x + acc[i].y;
  g_sink[(blockIdx.x * blockDim.x + threadIdx.x) & 0xFFFF] = sum;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// producer-style stores: each lane writes 12 chunks (16 B) of its star slot
template <int S>
__global__ void __launch_bounds__(512) k_store(int steps, unsigned long long* cyc) {
  extern __shared__ __align__(16) unsigned char sm[];
  const int lane = threadIdx.x & 31;
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  uint32_t j = (threadIdx.x * 5u) & (NSTAR - 1);
  const uint32_t b0 = hash32(threadIdx.x) & 3;
  __syncthreads();
  const unsigned long long t0 = clock64();
  float v = 1.f;
  for (int t = 0; t < steps; ++t) {
#pragma unroll
    for (int c = 0; c < 12; ++c) {
      uint32_t q;
      if (S == 0) q = (c + lane) & 7;                        // rotated: conflict-free
      else if (S == 1) q = (2 * ((b0 + (c >> 1)) & 3) + (c & 1)) & 7;  // static order, random b0
      else q = c & 7;                                        // all lanes the same quad
      const uint32_t a = base + j * 256u + (c >= 6 ? 128u : 0u) + 16u * q;
      asm volatile("st.shared.v4.f32 [%0], {%1,%1,%1,%1};" ::"r"(a), "f"(v) : "memory");
      v += 1.f;
    }
    j = (j + 32u) & (NSTAR - 1);
  }
  const unsigned long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <typename K>
double run(K kern, int warps, int steps, const char* name, double per) {
  const int threads = 32 * warps;
  const size_t smem = NSTAR * 256;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  unsigned long long* d;
  cudaMalloc(&d, 148 * sizeof(unsigned long long));
  kern<<<148, threads, smem>>>(steps / 4, d);
  kern<<<148, threads, smem>>>(steps, d);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  cudaFree(d);
  double mx = 0;
  for (int i = 0; i < 148; ++i) mx = mx > (double)h[i] ? mx : (double)h[i];
  const double v = mx / ((double)steps * warps) * per;
  printf("{\"test\": \"%s\", \"warps_per_sm\": %d, \"sm_cycles_per_warp_step\": %.3f, \"err\": \"%s\"}\n", name, warps, v,
         cudaGetErrorString(e));
  return v;
}

int main() {
  for (int w : {4, 8, 12, 16}) {
    run(k_walk<0>, w, STEPS, "walk L0 diag", 1.0);
    run(k_walk<1>, w, STEPS, "walk L1 row", 1.0);
    run(k_walk<2>, w, STEPS, "walk L2 rand", 1.0);
    run(k_walk<3>, w, STEPS, "walk L3 same-star", 1.0);
  }
  for (int w : {4, 8}) {
    run(k_store<0>, w, 512, "sts12 S0 rotated (per warp-chunk of 32 stars)", 1.0);
    run(k_store<1>, w, 512, "sts12 S1 static random b0", 1.0);
    run(k_store<2>, w, 512, "sts12 S2 same quad", 1.0);
  }
  return 0;
}
