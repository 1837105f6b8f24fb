// fp64_lat.cu -- single-warp dependent-chain latencies on this GPU (DFMA, DMUL, MUFU.RCP64H + fix-up,
// LDS round trip), in SM cycles.  Informs the inner kernel's ILP budget.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void lat(double *out, long long *cyc, double a, double b) {
  __shared__ double sm[64];
  double x = threadIdx.x * 1e-9 + 1.0;
  sm[threadIdx.x] = x;
  __syncwarp();
  long long t0, t1;
  // DFMA chain
  t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < 1024; i++) { x = fma(x, a, b); x = fma(x, a, b); x = fma(x, a, b); x = fma(x, a, b); }
  t1 = clock64();
  cyc[0] = t1 - t0;
  // DMUL chain
  t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < 1024; i++) { x = x * a; x = x * b; x = x * a; x = x * b; }
  t1 = clock64();
  cyc[1] = t1 - t0;
  // MUFU.RCP64H chain
  t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < 1024; i++) {
    double y;
    asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    x = y + 1.0;
  }
  t1 = clock64();
  cyc[2] = t1 - t0;
  // LDS round trip (address depends on the loaded value)
  int idx = threadIdx.x;
  t0 = clock64();
#pragma unroll 1
  for (int i = 0; i < 1024; i++) { double v = sm[idx]; idx = ((int)v + threadIdx.x) & 31; }
  t1 = clock64();
  cyc[3] = t1 - t0;
  out[threadIdx.x] = x + idx;
}

int main() {
  double *o; long long *c, h[4];
  cudaMalloc(&o, 64 * 8); cudaMalloc(&c, 4 * 8);
  for (int w = 0; w < 2; w++) lat<<<1, 32>>>(o, c, 0.9999999, 1e-9);
  cudaMemcpy(h, c, 32, cudaMemcpyDeviceToHost);
  printf("{\"dfma_latency_cyc\": %.2f, \"dmul_latency_cyc\": %.2f, \"rcp64h_plus_dadd_latency_cyc\": %.2f, \"lds_dep_latency_cyc\": %.2f}\n",
         h[0] / 4096.0, h[1] / 4096.0, h[2] / 1024.0, h[3] / 1024.0);
  return 0;
}
