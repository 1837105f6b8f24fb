// Microbenchmark (round 2): the fixed costs of a small single build on B200 -- per-kernel launch gap
// inside a CUDA graph, a cooperative launch, and grid.sync() with 120 CTAs x 256 threads.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o tools/sync_overhead tools/sync_overhead.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__global__ void empty_kernel(int *p) {
  if (p && threadIdx.x == 0 && blockIdx.x == 0) p[0] += 1;
}
template <int NS>
__global__ void sync_kernel(int *p) {
  cg::grid_group g = cg::this_grid();
#pragma unroll 1
  for (int i = 0; i < NS; i++) {
    if (threadIdx.x == 0) atomicAdd(p + blockIdx.x % 32, 1);
    g.sync();
  }
}

template <class L>
float time_graph(cudaStream_t st, int reps, L launch) {
  cudaGraph_t gr;
  cudaGraphExec_t ex;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < reps; i++) launch();
  cudaStreamEndCapture(st, &gr);
  cudaGraphInstantiate(&ex, gr, 0);
  cudaGraphLaunch(ex, st);
  cudaStreamSynchronize(st);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, st);
  for (int k = 0; k < 10; k++) cudaGraphLaunch(ex, st);
  cudaEventRecord(b, st);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  cudaGraphExecDestroy(ex);
  cudaGraphDestroy(gr);
  return ms * 1e3f / (10 * reps);   // us per kernel
}

template <int NS>
float coop(cudaStream_t st, int *d, int grid) {
  return time_graph(st, 100, [&] {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, sync_kernel<NS>, d);
  });
}

int main() {
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  int *d;
  cudaMalloc(&d, 1024);
  cudaMemset(d, 0, 1024);
  printf("{\"empty_kernel_1cta_us\": %.2f, ", time_graph(st, 100, [&] { empty_kernel<<<1, 32, 0, st>>>(d); }));
  printf("\"empty_kernel_120x256_us\": %.2f, ", time_graph(st, 100, [&] { empty_kernel<<<120, 256, 0, st>>>(d); }));
  printf("\"coop_0sync_us\": %.2f, ", coop<0>(st, d, 120));
  printf("\"coop_1sync_us\": %.2f, ", coop<1>(st, d, 120));
  printf("\"coop_5sync_us\": %.2f, ", coop<5>(st, d, 120));
  printf("\"coop_20sync_us\": %.2f, ", coop<20>(st, d, 120));
  printf("\"coop_20sync_148_us\": %.2f}\n", coop<20>(st, d, 148));
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
  return 0;
}
