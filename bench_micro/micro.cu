// Microbenchmarks for the roofline denominators of the star-image tile kernel.
// Measures per-SM throughput of FFMA, FFMA2, MUFU.EX2, LDS variants, SHFL and HBM read/write bandwidth on the
// device it runs on. Output: one JSON object on stdout. Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

__device__ unsigned long long g_cycles[4096];
__device__ float g_sink[1 << 16];

__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }

// ---- FFMA: 8 independent accumulators, shared multiplicand (reuse-friendly, like acc += g*gx) ----
__global__ void k_ffma(int iters, float a, float b) {
  float acc[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc[i] = threadIdx.x * 0.001f + i;
  float m = a + threadIdx.x * 1e-7f;
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = fmaf(acc[i], m, b);
    }
  }
  unsigned long long t1 = clock64();
  float s = 0; for (int i = 0; i < 8; ++i) s += acc[i];
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- FFMA, 3 distinct register sources per instruction (acc = x*y + acc with x,y varying) ----
__global__ void k_ffma3(int iters, float a, float b) {
  float acc[8], x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { acc[i] = threadIdx.x * 0.001f + i; x[i] = a + i * 1e-3f; }
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = fmaf(x[i], x[(i + j + 1) & 7], acc[i]);
    }
  }
  unsigned long long t1 = clock64();
  float s = 0; for (int i = 0; i < 8; ++i) s += acc[i];
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- FFMA2 on float2 (2 FMAs per lane per instruction) ----
__global__ void k_ffma2(int iters, float a, float b) {
  float2 acc[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) acc[i] = make_float2(threadIdx.x * 0.001f + i, i * 0.5f);
  float2 m = make_float2(a + threadIdx.x * 1e-7f, a), bb = make_float2(b, b);
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = __ffma2_rn(acc[i], m, bb);
    }
  }
  unsigned long long t1 = clock64();
  float s = 0; for (int i = 0; i < 8; ++i) s += acc[i].x + acc[i].y;
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- MUFU.EX2 ----
__global__ void k_ex2(int iters, float a) {
  float v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = -(threadIdx.x * 1e-3f + i * 0.1f);
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int i = 0; i < 8; ++i) v[i] = ex2(v[i]) - a;
    }
  }
  unsigned long long t1 = clock64();
  float s = 0; for (int i = 0; i < 8; ++i) s += v[i];
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- LDS variants. mode: 0 = LDS.32 lane-varying conflict-free, 1 = LDS.32 uniform,
//      2 = LDS.128 uniform, 3 = LDS.128 lane-varying (consecutive), 4 = LDS.128 2 addresses (half-warps),
//      5 = LDS.128 4 addresses, 6 = LDS.128 8 addresses, 7 = LDS.64 uniform ----
template <int MODE>
__global__ void k_lds(int iters) {
  __shared__ __align__(16) float sm[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) sm[i] = i * 1e-6f;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  unsigned base = 0;
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      unsigned step = (unsigned)(it * 16 + j) * 64u;
      if (MODE == 0) {
        unsigned addr = ((step + lane) & 8191u) * 4u + (unsigned)__cvta_generic_to_shared(sm);
        float v; asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr)); a0 += v;
      } else if (MODE == 1) {
        unsigned addr = ((step) & 8191u) * 4u + (unsigned)__cvta_generic_to_shared(sm);
        float v; asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr)); a0 += v;
      } else if (MODE == 7) {
        unsigned addr = ((step) & 8190u) * 4u + (unsigned)__cvta_generic_to_shared(sm);
        float v, w; asm volatile("ld.shared.v2.f32 {%0,%1}, [%2];" : "=f"(v), "=f"(w) : "r"(addr)); a0 += v; a1 += w;
      } else {
        unsigned off;
        if (MODE == 2) off = 0; else if (MODE == 3) off = lane * 4; else if (MODE == 4) off = (lane >> 4) * 4;
        else if (MODE == 5) off = (lane >> 3) * 4; else off = (lane >> 2) * 4;
        unsigned addr = ((step + off) & 8188u) * 4u + (unsigned)__cvta_generic_to_shared(sm);
        float v0, v1, v2, v3;
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v0), "=f"(v1), "=f"(v2), "=f"(v3) : "r"(addr));
        a0 += v0; a1 += v1; a2 += v2; a3 += v3;
      }
    }
  }
  unsigned long long t1 = clock64();
  float s = a0 + a1 + a2 + a3 + base;
  if (s == 1234.5f) g_sink[threadIdx.x] = s;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- SHFL.IDX with lane-varying source ----
__global__ void k_shfl(int iters) {
  const int lane = threadIdx.x & 31;
  float v0 = lane * 0.5f, v1 = lane * 0.25f, acc = 0;
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      float a = __shfl_sync(0xffffffffu, (j & 1) ? v0 : v1, (lane + j + it) & 31);
      acc += a;
    }
  }
  unsigned long long t1 = clock64();
  if (acc == 1234.5f) g_sink[threadIdx.x] = acc;
  if (threadIdx.x == 0) g_cycles[blockIdx.x] = t1 - t0;
}
// ---- HBM: write-only, read-only, copy with 16-B vectors, grid-stride ----
__global__ void k_write(float4* __restrict__ dst, size_t n4, float v) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
    dst[i] = make_float4(v, v, v, v);
}
__global__ void k_read(const float4* __restrict__ src, size_t n4, float* out) {
  float s = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
    float4 v = __ldcs(src + i); s += v.x + v.y + v.z + v.w;
  }
  if (s == 1234.5f) out[0] = s;
}
__global__ void k_copy(const float4* __restrict__ src, float4* __restrict__ dst, size_t n4) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
    dst[i] = __ldcs(src + i);
}

static int n_sm = 0;

template <typename F>
static double run_compute(const char* name, F launch, int blocks, int threads, double ops_per_thread_iter, int iters,
                          bool first) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  launch(blocks, threads, 2);  // warm
  cudaDeviceSynchronize();
  cudaEventRecord(e0); launch(blocks, threads, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long cyc[4096]; cudaMemcpyFromSymbol(cyc, g_cycles, sizeof(unsigned long long) * blocks);
  double mx = 0; for (int i = 0; i < blocks; ++i) mx = cyc[i] > mx ? (double)cyc[i] : mx;
  double total_ops = ops_per_thread_iter * iters * (double)blocks * threads;
  double per_s = total_ops / (ms * 1e-3);
  // ops per SM per clock, from the in-kernel cycle count of the slowest block (blocks per SM are co-resident)
  int bps = (blocks + n_sm - 1) / n_sm;
  double per_sm_clk = ops_per_thread_iter * iters * (double)threads * bps / mx;
  double clk_ghz = mx / (ms * 1e-3) / 1e9;
  printf("%s  \"%s\": {\"ops_per_s\": %.4e, \"ops_per_sm_clk\": %.2f, \"eff_clk_ghz\": %.3f, \"ms\": %.3f}\n",
         first ? "" : ",", name, per_s, per_sm_clk, clk_ghz, ms);
  return per_sm_clk;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0)); n_sm = p.multiProcessorCount;
  int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  printf("{\"device\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, \"clock_rate_khz\": %d, \"smem_per_block_optin\": %zu,\n",
         p.name, n_sm, p.l2CacheSize, clk_khz, p.sharedMemPerBlockOptin);
  const int T = 256, B = n_sm * 4;  // 32 warps / SM
  run_compute("ffma_reuse", [&](int b, int t, int it) { k_ffma<<<b, t>>>(it, 1.0001f, 0.5f); }, B, T, 128, 2000, true);
  run_compute("ffma_3reg", [&](int b, int t, int it) { k_ffma3<<<b, t>>>(it, 1.0001f, 0.5f); }, B, T, 128, 2000, false);
  run_compute("ffma2_fmas", [&](int b, int t, int it) { k_ffma2<<<b, t>>>(it, 1.0001f, 0.5f); }, B, T, 256, 2000, false);
  run_compute("mufu_ex2", [&](int b, int t, int it) { k_ex2<<<b, t>>>(it, 0.5f); }, B, T, 128, 400, false);
  run_compute("lds32_lanevar", [&](int b, int t, int it) { k_lds<0><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds32_uniform", [&](int b, int t, int it) { k_lds<1><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds64_uniform", [&](int b, int t, int it) { k_lds<7><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds128_uniform", [&](int b, int t, int it) { k_lds<2><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds128_lanevar", [&](int b, int t, int it) { k_lds<3><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds128_2addr", [&](int b, int t, int it) { k_lds<4><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds128_4addr", [&](int b, int t, int it) { k_lds<5><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("lds128_8addr", [&](int b, int t, int it) { k_lds<6><<<b, t>>>(it); }, B, T, 16, 2000, false);
  run_compute("shfl_idx", [&](int b, int t, int it) { k_shfl<<<b, t>>>(it); }, B, T, 16, 2000, false);

  // HBM
  size_t bytes = (size_t)2 << 30;  // 2 GiB per buffer (>> L2)
  float4 *a, *b; float* o;
  CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes)); CK(cudaMalloc(&o, 64));
  size_t n4 = bytes / 16;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int gb = n_sm * 8, gt = 512;
  for (int mode = 0; mode < 3; ++mode) {
    float best = 1e30f;
    for (int rep = 0; rep < 6; ++rep) {
      cudaEventRecord(e0);
      if (mode == 0) k_write<<<gb, gt>>>(a, n4, 1.0f);
      else if (mode == 1) k_read<<<gb, gt>>>(a, n4, o);
      else k_copy<<<gb, gt>>>(a, b, n4);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (rep > 0 && ms < best) best = ms;
    }
    double moved = (mode == 2 ? 2.0 : 1.0) * bytes;
    printf(", \"%s_GBps\": %.1f\n", mode == 0 ? "hbm_write" : (mode == 1 ? "hbm_read" : "hbm_copy"),
           moved / (best * 1e-3) / 1e9);
  }
  // write of a 67 MB image (fits in L2): what a single-frame fp32 image store sees
  {
    size_t ib = (size_t)4096 * 4096 * 4; size_t in4 = ib / 16; float best = 1e30f;
    for (int rep = 0; rep < 8; ++rep) {
      k_read<<<gb, gt>>>(b, n4, o);  // evict with clean lines
      cudaEventRecord(e0); k_write<<<gb, gt>>>(a, in4, 2.0f); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (rep > 0 && ms < best) best = ms;
    }
    printf(", \"write_67MB_after_clean_flush_GBps\": %.1f, \"write_67MB_us\": %.2f\n", ib / (best * 1e-3) / 1e9, best * 1e3);
    best = 1e30f;
    for (int rep = 0; rep < 8; ++rep) {
      k_write<<<gb, gt>>>(b, n4, 3.0f);  // evict with dirty lines
      cudaEventRecord(e0); k_write<<<gb, gt>>>(a, in4, 2.0f); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (rep > 0 && ms < best) best = ms;
    }
    printf(", \"write_67MB_after_dirty_flush_GBps\": %.1f, \"write_67MB_dirty_us\": %.2f\n", ib / (best * 1e-3) / 1e9, best * 1e3);
    // empty-kernel launch cadence
    float ms; cudaEventRecord(e0);
    for (int i = 0; i < 1000; ++i) k_write<<<1, 32>>>(a, 0, 0.f);
    cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
    printf(", \"empty_launch_us\": %.3f\n", ms);
  }
  printf("}\n");
  CK(cudaGetLastError());
  return 0;
}
