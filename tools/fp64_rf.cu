// fp64_rf.cu -- DFMA issue rate vs operand sources (register-file bank pressure test).
//  v0: x = fma(x, a, b), a/b the same values every time (uniform -> UR or reuse cache)
//  v1: x[c] = fma(x[c], y[c], z[c]) with per-chain distinct registers y, z (3 distinct R operands)
//  v2: x[c] = fma(x[c], y[c], b) (2 distinct R + 1 uniform)
#include <cstdio>
#include <cuda_runtime.h>
constexpr int CH = 8, IT = 2048;
template <int V>
__global__ void k(double *out, double a, double b, long long *cyc) {
  double x[CH], y[CH], z[CH];
#pragma unroll
  for (int c = 0; c < CH; c++) { x[c] = threadIdx.x * 1e-3 + c; y[c] = 0.999 + threadIdx.x * 1e-9 * c; z[c] = 1e-7 * (c + 1) + threadIdx.x * 1e-12; }
  long long t0 = clock64();
  for (int i = 0; i < IT; i++) {
#pragma unroll
    for (int c = 0; c < CH; c++) {
      if (V == 0) x[c] = fma(x[c], a, b);
      if (V == 1) x[c] = fma(x[c], y[c], z[c]);
      if (V == 2) x[c] = fma(x[c], y[c], b);
      if (V == 3) x[c] = fma(y[0], x[c], z[c]);   // shared multiplier (operand reuse), distinct addend
      if (V == 4) x[c] = x[c] * y[c];              // DMUL, two distinct registers
      if (V == 5) x[c] = fma(x[c], y[c], x[c]);    // three operands, two distinct registers
    }
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int c = 0; c < CH; c++) s += x[c] + y[c] + z[c];
  if (s == 1.2345) out[0] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int V> void run(double *o, long long *c, int sms) {
  const int threads = 256, bps = 4;   // 32 warps / SM
  for (int w = 0; w < 2; w++) k<V><<<sms * bps, threads>>>(o, 0.999999, 1e-7, c);
  cudaDeviceSynchronize();
  long long h[1024]; cudaMemcpy(h, c, 8 * sms * bps, cudaMemcpyDeviceToHost);
  double mx = 0; for (int i = 0; i < sms * bps; i++) mx = h[i] > mx ? h[i] : mx;
  double lanes = (double)bps * threads * IT * CH / mx;
  printf("\"v%d_lanes_per_sm_clk\": %.2f%s", V, lanes, V == 5 ? "" : ", ");
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double *o; long long *c; cudaMalloc(&o, 8); cudaMalloc(&c, 8 * 1024);
  printf("{"); run<0>(o, c, sms); run<1>(o, c, sms); run<2>(o, c, sms); run<3>(o, c, sms); run<4>(o, c, sms);
  run<5>(o, c, sms); printf("}\n");
}
