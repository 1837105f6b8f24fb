// FP64 tensor-core (mma.sync m8n8k4 f64) throughput on this GPU: every warp runs independent chains of
// DMMA on register fragments.  nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/dmma_peak tools/dmma_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};\n"
               : "+d"(d0), "+d"(d1)
               : "d"(a), "d"(b));
}

template <int CH>
__global__ void dmma_loop(double *out, int iters, double a0, double b0) {
  double d[CH][2];
  for (int c = 0; c < CH; c++) d[c][0] = d[c][1] = 0.0;
  double a = a0 + threadIdx.x * 1e-9, b = b0 - threadIdx.x * 1e-9;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int c = 0; c < CH; c++) dmma(d[c][0], d[c][1], a, b);
  }
  double s = 0.0;
  for (int c = 0; c < CH; c++) s += d[c][0] + d[c][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int CH>
__global__ void dfma_loop(double *out, int iters, double a0, double b0) {
  double d[CH];
  for (int c = 0; c < CH; c++) d[c] = c;
  const double a = a0 + threadIdx.x * 1e-9, b = b0;
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int c = 0; c < CH; c++) d[c] = fma(a, d[c], b);
  }
  double s = 0.0;
  for (int c = 0; c < CH; c++) s += d[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double *out;
  cudaMalloc(&out, sizeof(double) * sms * 8 * 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 4000;
  for (int warps = 4; warps <= 16; warps *= 2) {
    const int grid = sms * 2, block = 32 * warps / 2;
    dmma_loop<8><<<grid, block>>>(out, 10, 1.0, 1.0);
    cudaEventRecord(e0);
    dmma_loop<8><<<grid, block>>>(out, iters, 1.0, 1.0);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    const double flop = 2.0 * 256 * 8.0 * iters * (double)grid * block / 32;
    printf("{\"op\": \"dmma_m8n8k4\", \"warps_per_sm\": %d, \"tflops\": %.2f}\n", warps, flop / (ms * 1e-3) / 1e12);
    dfma_loop<8><<<grid, block>>>(out, 10, 1.0, 1.0);
    cudaEventRecord(e0);
    dfma_loop<8><<<grid, block>>>(out, iters * 8, 1.0, 1.0);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    const double flop2 = 2.0 * 8.0 * iters * 8 * (double)grid * block;
    printf("{\"op\": \"dfma\", \"warps_per_sm\": %d, \"tflops\": %.2f}\n", warps, flop2 / (ms * 1e-3) / 1e12);
  }
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) printf("error %s\n", cudaGetErrorString(err));
  return 0;
}
