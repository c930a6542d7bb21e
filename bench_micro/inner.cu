// Microbenchmark of candidate tile-kernel inner loops: SM-cycles per warp step for the ways of
// delivering row factors (gy, broadcast from shared memory) and column factors (gx, lane-varying) to the FFMA2s.
// Each warp walks a list of star-slot entries in shared memory and updates a fixed register window.
//   D1: 1 star/step,  lane=(c16,h): 2x LDS.128 (2 addr), 1x LDS.64 lane-var, 8 FFMA2 (gy,gy)x(gxA,gxB)
//   D2: 2 stars/step, lane=(c16,p): 4x LDS.128 (2 addr), 1x LDS.32 lane-var, 8 FFMA2 (gy0,gy1)x(gx,gx)
//   D3: 2 stars/step, lane=(c8,h,p): 2x LDS.128 (4 addr), 1x LDS.64 lane-var, 8 FFMA2 (gy,gy)x(gxA,gxB)
//   D4: 4 stars/step, lane=(c8,p4): 4x LDS.128 (4 addr), 1x LDS.32 lane-var, 8 FFMA2 (gy0,gy1)x(gx,gx)
//   D5: like D2 but the 16 row factors come as 2x LDS.128 of 8 (gy pairs packed as float2 of 2 rows) -- n/a
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o inner inner.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ unsigned long long g_cyc[4096];
__device__ float g_sink[1 << 16];

constexpr int NSLOT = 16;   // star slots per warp
constexpr int NENT = 256;   // entries per warp list

template <int D>
__global__ void __launch_bounds__(256) k_inner(int iters) {
  __shared__ __align__(16) float s_gy[8][NSLOT][16];
  __shared__ __align__(16) float s_gx[8][NSLOT][48];
  __shared__ uint32_t s_ent[8][NENT];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int i = lane; i < NSLOT * 16; i += 32) (&s_gy[w][0][0])[i] = 1e-3f * (i & 15);
  for (int i = lane; i < NSLOT * 48; i += 32) (&s_gx[w][0][0])[i] = 1e-3f * (i % 48);
  for (int i = lane; i < NENT; i += 32) {
    uint32_t a = (i * 7 + 3) % NSLOT, b = (i * 13 + 5) % NSLOT, c = (i * 29 + 1) % NSLOT, d = (i * 31 + 9) % NSLOT;
    uint32_t off = (i * 5) & 15;
    s_ent[w][i] = a | (b << 6) | (c << 12) | (d << 18) | (off << 24);
  }
  __syncwarp();
  float2 acc[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) acc[i] = make_float2(0.f, 0.f);
  const uint32_t gyb = (uint32_t)__cvta_generic_to_shared(&s_gy[w][0][0]);
  const uint32_t gxb = (uint32_t)__cvta_generic_to_shared(&s_gx[w][0][0]);
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll 2
    for (int e = 0; e < NENT; ++e) {
      const uint32_t ent = s_ent[w][e];
      int sel;
      if (D == 1) sel = 0;
      else if (D == 2) sel = lane >> 4;
      else if (D == 3) sel = lane >> 4;
      else sel = lane >> 3;
      const uint32_t slot = (ent >> (6 * sel)) & 15u;
      const uint32_t off = ent >> 24;
      if (D == 1 || D == 3) {
        const int c = (D == 1) ? (lane & 15) : (lane & 7);
        const int h = (D == 1) ? (lane >> 4) : ((lane >> 3) & 1);
        float4 g0, g1; float2 gx;
        uint32_t ay = gyb + (slot * 16 + h * 8) * 4;
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g0.x), "=f"(g0.y), "=f"(g0.z), "=f"(g0.w) : "r"(ay));
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g1.x), "=f"(g1.y), "=f"(g1.z), "=f"(g1.w) : "r"(ay + 16));
        uint32_t ax = gxb + (slot * 48 + 2 * (c + off)) * 4;
        asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(gx.x), "=f"(gx.y) : "r"(ax));
        const float g[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[4 + j] = __ffma2_rn(make_float2(g[j], g[j]), gx, acc[4 + j]);
      } else {
        const int c = (D == 2) ? (lane & 15) : (lane & 7);
        float4 g[4]; float gx;
        uint32_t ay = gyb + slot * 64;
#pragma unroll
        for (int q = 0; q < 4; ++q)
          asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(g[q].x), "=f"(g[q].y), "=f"(g[q].z), "=f"(g[q].w) : "r"(ay + 16 * q));
        uint32_t ax = gxb + (slot * 48 + c + off) * 4;
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(gx) : "r"(ax));
        const float2 gx2 = make_float2(gx, gx);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          acc[4 + 2 * q] = __ffma2_rn(make_float2(g[q].x, g[q].y), gx2, acc[4 + 2 * q]);
          acc[5 + 2 * q] = __ffma2_rn(make_float2(g[q].z, g[q].w), gx2, acc[5 + 2 * q]);
        }
      }
    }
  }
  unsigned long long t1 = clock64();
  float s = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += acc[i].x + acc[i].y;
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cyc[blockIdx.x] = t1 - t0;
}

static int n_sm;

// D5/D6/D7: the W8 phase-D step: 8 lane groups (4 lanes: cx, h) each take a star from their own list; per lane:
// LDS.U8 list entry -> LDS.64 info -> 2x LDS.128 gy (slot stride GYS floats) + 1x LDS.128 gx (8-float slots),
// 16 FFMA2 (gy,gy)x(gxA,gxB).  D5: gy stride 16 floats; D6: gy stride 20 floats (bank rotation); D7: like D5 but all
// lane groups read the same star (1 star/step, conflict-free reference).
template <int D>
__global__ void __launch_bounds__(256) k_w8(int iters) {
  constexpr int GYS = (D == 6) ? 20 : 16;
  __shared__ __align__(16) float s_gy[256 * GYS];
  __shared__ __align__(16) float s_gx[512 * 8];
  __shared__ __align__(8) int2 s_info[256];
  __shared__ uint8_t s_list[32][256];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 256 * GYS; i += 256) s_gy[i] = 1e-3f * (i & 31);
  for (int i = threadIdx.x; i < 512 * 8; i += 256) s_gx[i] = 1e-3f * (i & 15);
  for (int i = threadIdx.x; i < 256; i += 256) s_info[i] = make_int2((i * 37) & 127, (i * 53) & 255);
  for (int i = threadIdx.x; i < 32 * 256; i += 256) s_list[i >> 8][i & 255] = (uint8_t)((i * 97 + (i >> 8) * 31) & 255);
  __syncthreads();
  const int q = lane >> 2, cx = (lane >> 1) & 1, h = lane & 1;
  const int B = warp >> 1, Q = 8 * (warp & 1) + q;
  const int p = (D == 7) ? (B * 8) : (B * 8 + q);
  float2 acc[8][2];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc[i][0] = acc[i][1] = make_float2(0.f, 0.f);
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll 2
    for (int t = 0; t < 256; ++t) {
      const int s = s_list[p][t];
      const int2 inf = s_info[s];
      const float4* gya = reinterpret_cast<const float4*>(&s_gy[(inf.x + B) * GYS + h * 8]);
      const float4* gxa = reinterpret_cast<const float4*>(&s_gx[(inf.y + (D == 7 ? 0 : Q)) * 8 + cx * 4]);
      const float4 g0 = gya[0], g1 = gya[1], x4 = gxa[0];
      const float2 gA = make_float2(x4.x, x4.y), gB = make_float2(x4.z, x4.w);
      const float g[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        acc[i][0] = __ffma2_rn(make_float2(g[i], g[i]), gA, acc[i][0]);
        acc[i][1] = __ffma2_rn(make_float2(g[i], g[i]), gB, acc[i][1]);
      }
    }
  }
  unsigned long long t1 = clock64();
  float sum = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) sum += acc[i][0].x + acc[i][0].y + acc[i][1].x + acc[i][1].y;
  if (sum == 1234.5f) g_sink[threadIdx.x] = sum;
  if (threadIdx.x == 0) g_cyc[blockIdx.x] = t1 - t0;
}

template <int D>
static void run_w8(const char* name, int blocks_per_sm) {
  const int iters = 100;
  const int B = n_sm * blocks_per_sm;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k_w8<D><<<B, 256>>>(2);
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  k_w8<D><<<B, 256>>>(iters);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long cyc[4096]; cudaMemcpyFromSymbol(cyc, g_cyc, sizeof(unsigned long long) * B);
  double mx = 0; for (int i = 0; i < B; ++i) mx = cyc[i] > mx ? (double)cyc[i] : mx;
  double steps_per_sm = (double)iters * 256 * 8 * blocks_per_sm;
  double cyc_per_step = mx / steps_per_sm;
  printf("{\"design\": \"%s\", \"warps_per_sm\": %d, \"sm_cycles_per_step\": %.3f, \"sm_cycles_per_visit\": %.3f, \"ms\": %.3f, \"err\": \"%s\"}\n",
         name, 8 * blocks_per_sm, cyc_per_step, cyc_per_step / (D == 7 ? 1 : 8), ms, cudaGetErrorString(cudaGetLastError()));
}

template <int D>
static void run(const char* name, int blocks_per_sm, int stars_per_step) {
  const int iters = 200;
  const int B = n_sm * blocks_per_sm;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k_inner<D><<<B, 256>>>(2);
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  k_inner<D><<<B, 256>>>(iters);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long cyc[4096]; cudaMemcpyFromSymbol(cyc, g_cyc, sizeof(unsigned long long) * B);
  double mx = 0; for (int i = 0; i < B; ++i) mx = cyc[i] > mx ? (double)cyc[i] : mx;
  double steps_per_sm = (double)iters * NENT * 8 * blocks_per_sm;
  double cyc_per_step = mx / steps_per_sm;
  printf("{\"design\": \"%s\", \"warps_per_sm\": %d, \"sm_cycles_per_step\": %.3f, \"sm_cycles_per_star\": %.3f, \"ms\": %.3f, \"err\": \"%s\"}\n",
         name, 8 * blocks_per_sm, cyc_per_step, cyc_per_step / stars_per_step, ms, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0); n_sm = p.multiProcessorCount;
  for (int bps = 1; bps <= 3; ++bps) {
    run_w8<5>("W8 random slots gy16", bps);
    run_w8<6>("W8 random slots gy20", bps);
    run_w8<7>("W8 same star all groups", bps);
  }
  for (int bps = 1; bps <= 3; ++bps) {
    run<1>("D1 1star c16xh  2xLDS128(2a)+LDS64", bps, 1);
    run<2>("D2 2star c16xp  4xLDS128(2a)+LDS32", bps, 2);
    run<3>("D3 2star c8xhxp 2xLDS128(4a)+LDS64", bps, 2);
    run<4>("D4 4star c8xp4  4xLDS128(4a)+LDS32", bps, 4);
  }
  return 0;
}
