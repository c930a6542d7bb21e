// Microbenchmark: throughput of global integer atomics on a small counter array (the binning pattern: P random
// increments over ntiles counters), with and without a used return value, and of a plain streaming kernel of the
// same shape for reference.  Prints one JSON object.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

__global__ void k_red(uint32_t* cnt, uint32_t ntiles, int n, int per) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint32_t h = hash32(i);
  for (int k = 0; k < per; ++k) atomicAdd(&cnt[(h + k * 7919u) % ntiles], 1u);
}
__global__ void k_atom(uint32_t* cnt, uint32_t ntiles, int n, int per, uint32_t* out) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint32_t h = hash32(i), s = 0;
  uint32_t r[4];
#pragma unroll
  for (int k = 0; k < 4; ++k) r[k] = k < per ? atomicAdd(&cnt[(h + k * 7919u) % ntiles], 1u) : 0u;
#pragma unroll
  for (int k = 0; k < 4; ++k) s += r[k];
  out[i] = s;
}
__global__ void k_stream(const float4* in, float4* out, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float4 v = in[i];
  out[i] = make_float4(v.x + 1, v.y, v.z, v.w);
}
__global__ void k_empty() {}

int main() {
  const int n = 1 << 20;
  uint32_t *cnt, *out;
  float4 *a, *b;
  cudaMalloc(&cnt, 1 << 22);
  cudaMalloc(&out, n * 4);
  cudaMalloc(&a, n * 16);
  cudaMalloc(&b, n * 16);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  printf("{");
  const char* sep = "";
  for (uint32_t ntiles : {8192u, 16384u, 262144u}) {
    for (int per : {2, 4}) {
      for (int mode = 0; mode < 2; ++mode) {
        float best = 1e9f;
        for (int rep = 0; rep < 5; ++rep) {
          cudaMemset(cnt, 0, ntiles * 4);
          cudaEventRecord(e0);
          if (mode == 0) k_red<<<(n + 255) / 256, 256>>>(cnt, ntiles, n, per);
          else k_atom<<<(n + 255) / 256, 256>>>(cnt, ntiles, n, per, out);
          cudaEventRecord(e1);
          cudaEventSynchronize(e1);
          float ms;
          cudaEventElapsedTime(&ms, e0, e1);
          if (ms < best) best = ms;
        }
        printf("%s\"%s_t%u_p%d_us\": %.2f", sep, mode ? "atom_ret" : "red", ntiles, per, best * 1e3);
        sep = ", ";
      }
    }
  }
  float best = 1e9f;
  for (int rep = 0; rep < 5; ++rep) {
    cudaEventRecord(e0);
    k_stream<<<(n + 255) / 256, 256>>>(a, b, n);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf(", \"stream_1M_float4_us\": %.2f", best * 1e3);
  best = 1e9f;
  for (int rep = 0; rep < 5; ++rep) {
    cudaEventRecord(e0);
    k_empty<<<1, 32>>>();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  printf(", \"empty_kernel_us\": %.2f", best * 1e3);
  // back-to-back dependent empty kernels in a graph-less stream: per-launch device gap
  cudaEventRecord(e0);
  for (int i = 0; i < 100; ++i) k_empty<<<148, 128>>>();
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  printf(", \"empty_148x128_x100_per_launch_us\": %.2f", ms * 10);
  // same via a CUDA graph
  cudaStream_t s;
  cudaStreamCreate(&s);
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < 100; ++i) k_empty<<<148, 128, 0, s>>>();
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaGraphLaunch(ge, s);
  cudaStreamSynchronize(s);
  cudaEventRecord(e0, s);
  cudaGraphLaunch(ge, s);
  cudaEventRecord(e1, s);
  cudaEventSynchronize(e1);
  cudaEventElapsedTime(&ms, e0, e1);
  printf(", \"graph_empty_148x128_x100_per_launch_us\": %.2f}\n", ms * 10);
  return 0;
}
