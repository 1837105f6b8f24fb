// fp64_peak.cu -- measures the B200 FP64 (DFMA) issue rate: lanes per SM per clock and TFLOP/s.
// Used once to pin the roofline denominator of the inner-integral kernel.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/fp64_peak tools/fp64_peak.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int CHAINS = 8;
constexpr int ITERS = 4096;

__global__ void dfma_kernel(double *out, double a, double b, long long *cycles) {
  double x[CHAINS];
#pragma unroll
  for (int c = 0; c < CHAINS; c++) x[c] = threadIdx.x * 1e-3 + c;
  long long t0 = clock64();
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < CHAINS; c++) x[c] = fma(x[c], a, b);
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int c = 0; c < CHAINS; c++) s += x[c];
  if (s == 1.2345) out[0] = s;
  if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  double *out;
  long long *cyc;
  const int threads = 512, blocks_per_sm = 4, blocks = sms * blocks_per_sm;
  cudaMalloc(&out, 8);
  cudaMalloc(&cyc, sizeof(long long) * blocks);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int w = 0; w < 3; w++) dfma_kernel<<<blocks, threads>>>(out, 0.999999, 1e-7, cyc);
  cudaEventRecord(e0);
  const int reps = 20;
  for (int r = 0; r < reps; r++) dfma_kernel<<<blocks, threads>>>(out, 0.999999, 1e-7, cyc);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  long long *hc = new long long[blocks];
  cudaMemcpy(hc, cyc, sizeof(long long) * blocks, cudaMemcpyDeviceToHost);
  double cmax = 0;
  for (int i = 0; i < blocks; i++) cmax = hc[i] > cmax ? hc[i] : cmax;
  const double dfma_total = (double)reps * blocks * threads * ITERS * CHAINS;
  const double tflops = 2.0 * dfma_total / (ms * 1e-3) / 1e12;
  // per SM per clock: blocks_per_sm co-resident blocks share the SM during the cycle window
  const double lanes = (double)blocks_per_sm * threads * ITERS * CHAINS / cmax;
  printf("{\"sms\": %d, \"clock_rate_mhz\": %.0f, \"dfma_tflops\": %.3f, \"dfma_lanes_per_sm_per_clk\": %.2f, "
         "\"implied_clock_mhz\": %.0f}\n",
         sms, clk / 1e3, tflops, lanes, tflops * 1e12 / (2.0 * sms * lanes) / 1e6);
  return 0;
}
