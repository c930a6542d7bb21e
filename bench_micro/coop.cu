// probe: a cooperative launch (cudaLaunchAttributeCooperative) captured into a CUDA graph, with a hand-rolled
// grid barrier (atomic counter, zeroed by a memset node each replay)
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(unsigned* bar, int* out, int n) {
  __shared__ int s;
  if (threadIdx.x == 0) {
    out[blockIdx.x] = blockIdx.x;
    __threadfence();
    atomicAdd(bar, 1u);
    unsigned v;
    do { asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(v) : "l"(bar)); } while (v < gridDim.x);
    int sum = 0;
    for (int i = 0; i < (int)gridDim.x; ++i) sum += out[i];
    s = sum;
  }
  __syncthreads();
  if (threadIdx.x == 0) out[gridDim.x + blockIdx.x] = s;
}
int main() {
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  int nb = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k, 1024, 0);
  int grid = nb * nsm;
  printf("sms %d blocks/sm %d grid %d\n", nsm, nb, grid);
  unsigned* bar; int* out; cudaMalloc(&bar, 4); cudaMalloc(&out, 8 * grid * 4);
  cudaStream_t st; cudaStreamCreate(&st);
  cudaLaunchConfig_t cfg = {}; cfg.gridDim = grid; cfg.blockDim = 1024; cfg.stream = st;
  cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeCooperative; at[0].val.cooperative = 1;
  cfg.attrs = at; cfg.numAttrs = 1;
  cudaGraph_t g; cudaGraphExec_t ge;
  cudaError_t e = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  printf("begin %s\n", cudaGetErrorString(e));
  cudaMemsetAsync(bar, 0, 4, st);
  e = cudaLaunchKernelEx(&cfg, k, bar, out, grid);
  printf("launch in capture %s\n", cudaGetErrorString(e));
  e = cudaStreamEndCapture(st, &g); printf("end %s\n", cudaGetErrorString(e));
  e = cudaGraphInstantiate(&ge, g, 0); printf("inst %s\n", cudaGetErrorString(e));
  for (int r = 0; r < 3; ++r) { e = cudaGraphLaunch(ge, st); }
  e = cudaStreamSynchronize(st); printf("run %s\n", cudaGetErrorString(e));
  int h[2]; cudaMemcpy(h, out + grid, 8, cudaMemcpyDeviceToHost);
  printf("sum %d expect %d\n", h[0], grid * (grid - 1) / 2);
  // too-large cooperative grid must fail cleanly
  cfg.gridDim = grid + 1; e = cudaLaunchKernelEx(&cfg, k, bar, out, grid + 1);
  printf("oversize %s\n", cudaGetErrorString(e)); cudaGetLastError();
  return 0;
}
