// kernels_band.cuh -- NEXT-2 of SURVEY.md §8(f): the paper's batched band LU for the implicit step
// (PAPER.md:1@24330-26180, §III-G): A = shift M - J per species block, reverse Cuthill-McKee order,
// band storage with B = UBW = LBW, outer-product band LU without pivoting (Golub-Van Loan Alg.
// 4.3.1), then forward/backward substitution.  (included once, by landau.cu)
//
// Band storage of one matrix: n rows x W = 2B + 1, row-major, A(i, j) at i W + (j - i + B).
#pragma once
#include <cstdint>

namespace landau {

// A = shift M - J scattered into the (zeroed) band storage of one species block, every batch item
__global__ void band_fill_kernel(int64_t nslots, const int32_t *__restrict__ band_slot, const double *__restrict__ M,
                                 const double *__restrict__ J, int64_t J_bstride, int64_t J_off, double shift,
                                 double *__restrict__ band, int64_t band_bstride, int64_t band_off, int nbatch) {
  const int64_t total = nslots * nbatch;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / nslots, s = k % nslots;
    band[b * band_bstride + band_off + band_slot[s]] = fma(shift, M[s], -J[b * J_bstride + J_off + s]);
  }
}

struct BandDesc {   // per species block
  int64_t off;      // offset of the block inside one batch item's band storage
  int n, B;
};

// One CTA per (batch item, species block).  Step k: multipliers l_i = A(i,k) / A(k,k) for the B rows
// below, then the B x B outer-product update A(i,j) -= l_i A(k,j); threads run along j (contiguous).
__global__ void __launch_bounds__(1024) band_factor_kernel(double *__restrict__ band, int64_t band_bstride,
                                                           const BandDesc *__restrict__ desc, int nsp) {
  extern __shared__ double mult[];   // [B]
  const int b = blockIdx.x / nsp, a = blockIdx.x % nsp;
  const BandDesc d = desc[a];
  double *A = band + (int64_t)b * band_bstride + d.off;
  const int n = d.n, B = d.B, W = 2 * B + 1;
  for (int k = 0; k < n - 1; k++) {
    const int m = min(B, n - 1 - k);
    const double ip = 1.0 / A[(int64_t)k * W + B];
    for (int t = threadIdx.x; t < m; t += blockDim.x) {
      const int64_t at = (int64_t)(k + 1 + t) * W + (B - 1 - t);   // A(k+1+t, k)
      const double l = A[at] * ip;
      mult[t] = l;
      A[at] = l;
    }
    __syncthreads();
    const double *rowk = A + (int64_t)k * W + B;   // rowk[c + 1] = A(k, k + 1 + c)
    for (int idx = threadIdx.x; idx < m * m; idx += blockDim.x) {
      const int r = idx / m, c = idx % m;
      // A(k+1+r, k+1+c) at row k+1+r, offset c - r + B
      A[(int64_t)(k + 1 + r) * W + (c - r + B)] -= mult[r] * rowk[c + 1];
    }
    __syncthreads();
  }
}

// One warp per (batch item, species block): x = U^-1 L^-1 P b in the RCM order, then un-permuted.
// y is the permuted right-hand side, worked in place in scratch (global), lanes split each row's dot
// product over its band and reduce with shuffles.
__global__ void band_solve_kernel(const double *__restrict__ band, int64_t band_bstride, const BandDesc *__restrict__ desc,
                                  const int32_t *__restrict__ perm_all, const int64_t *__restrict__ perm_off,
                                  const int64_t *__restrict__ vec_off, int64_t ndof, const double *__restrict__ rhs,
                                  double *__restrict__ scratch, double *__restrict__ x, int nsp, int nbatch) {
  const int lane = threadIdx.x & 31;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (w >= (int64_t)nbatch * nsp) return;
  const int b = (int)(w / nsp), a = (int)(w % nsp);
  const BandDesc d = desc[a];
  const double *A = band + (int64_t)b * band_bstride + d.off;
  const int32_t *perm = perm_all + perm_off[a];   // new -> old (within the species block)
  const int n = d.n, B = d.B, W = 2 * B + 1;
  const double *bb = rhs + (int64_t)b * ndof + vec_off[a];
  double *y = scratch + (int64_t)b * ndof + vec_off[a];
  double *xb = x + (int64_t)b * ndof + vec_off[a];
  for (int i = lane; i < n; i += 32) y[i] = bb[perm[i]];
  __syncwarp();
  for (int i = 0; i < n; i++) {   // forward: unit lower L
    double s = 0.0;
    const int j0 = max(0, i - B);
    for (int j = j0 + lane; j < i; j += 32) s = fma(A[(int64_t)i * W + (j - i + B)], y[j], s);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) y[i] -= s;
    __syncwarp();
  }
  for (int i = n - 1; i >= 0; i--) {   // backward: U
    double s = 0.0;
    const int j1 = min(n - 1, i + B);
    for (int j = i + 1 + lane; j <= j1; j += 32) s = fma(A[(int64_t)i * W + (j - i + B)], y[j], s);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) y[i] = (y[i] - s) / A[(int64_t)i * W + B];
    __syncwarp();
  }
  for (int i = lane; i < n; i += 32) xb[perm[i]] = y[i];
}

}  // namespace landau
