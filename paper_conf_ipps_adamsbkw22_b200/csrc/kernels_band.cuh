// kernels_band.cuh -- NEXT-2 of SURVEY.md §8(f): the paper's batched band LU for the implicit step
// (PAPER.md:1@24330-26180, §III-G): A = shift M - J per species block, reverse Cuthill-McKee order,
// half-bandwidth B, outer-product band LU without pivoting (Golub-Van Loan Alg. 4.3.1), then
// forward/backward substitution.  (included once, by landau.cu)
//
// Factor storage of one matrix, "step-major": n rows of W = 2B + 1 doubles; row k holds what step k
// of the elimination produces:
//   LU[k][0] = U(k, k) (the pivot),  LU[k][t] = U(k, k + t) (t = 1..B),  LU[k][B + t] = L(k + t, k)
// (entries past n - 1 are zero).  Both substitutions then read one contiguous row per step.
#pragma once
#include <cstdint>

namespace landau {

// register window: each thread owns an R x C tile of the (B+1) x (B+1) active square, at most 256
// threads per CTA: 4 x 8 tiles for B + 1 <= 88 (two CTAs per SM), 8 x 8 tiles for B + 1 <= 128
constexpr int kBandD = 6;        // cp.async prefetch distance, in elimination steps
constexpr int kBandMaxP = 128;

struct BandDesc {             // per species block
  int64_t off;                // offset of the block in one batch item's LU storage
  int64_t aoff;               // offset of the block in one batch item's entry-value list (Aent)
  const int32_t *ent_ptr;     // [n+1] entering-row entry lists of the block's grid (host_setup.h)
  const uint16_t *ent_pos;    // [nent] position in the entering row: 0..B row part, B+1..2B column part
  int n, B, Pp, nent;         // B: the half-bandwidth padded so that Pp = B + 1 is a multiple of 8
};

// Aent[b][aoff + e] = shift M[slot e] - J[b][J_off + slot e]: the block's entries in consumption order
__global__ void band_gather_kernel(int64_t nent, const int32_t *__restrict__ ent_slot, const double *__restrict__ M,
                                   const double *__restrict__ J, int64_t J_bstride, int64_t J_off, double shift,
                                   double *__restrict__ Aent, int64_t ent_bstride, int64_t aoff, int nbatch) {
  const int64_t total = nent * nbatch;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / nent, e = k % nent;
    const int32_t s = ent_slot[e];
    Aent[b * ent_bstride + aoff + e] = fma(shift, M[s], -J[b * J_bstride + J_off + s]);
  }
}

__device__ __forceinline__ void cp_async8(void *smem, const void *gmem) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// band_lu_kernel, warp 0: issue the entry values of entering row e into ring slot e mod (D+1) (an
// empty commit group past n keeps one group per step)
__device__ __forceinline__ void band_issue(int e, int n, const int32_t *sptr, const double *ae, double *ring, int W,
                                           int lane) {
  if (e < n) {
    const int q0 = sptr[e], cnt = sptr[e + 1] - q0;
    double *dst = ring + (e % (kBandD + 1)) * W;
    for (int q = lane; q < cnt; q += 32) cp_async8(dst + q, ae + q0 + q);
  }
  cp_async_commit();
}

// One CTA per (batch item, species block).  The P x P active square (P = B + 1, B the padded
// half-bandwidth, P a multiple of 8) of the outer-product elimination lives in REGISTERS, cut into
// R x C tiles, one per thread, addressed circularly: logical row/column i sits in physical
// row/column i mod P.  Step k (pk = k mod P):
//   b) the owners of physical row/column pk publish U(k, .), A(., k) and the pivot in shared memory;
//   c) every thread applies the rank-1 update to its tile (the retiring row/column see zero
//      multipliers) and threads 0..2B write one value each of the factor row LU[k]; warp 0 stages
//      the entering row/column e = k + P: its entry values arrive by cp.async kBandD steps ahead and
//      are scattered into a dense buffer (after the entries of row e - 2 are scattered back to zero);
//   d) the owners of the retiring physical row/column load the entering one.
// The step loop is unrolled by 8 (P is a multiple of 8, so pk mod R and pk mod C are compile-time
// constants in each copy): the owners index their registers statically.  Two barriers per step,
// FP64 FMAs on register operands, no integer division.  Steps k = -P .. -1 only load the window.
template <int kBandR, int kBandC, int MINB>
__global__ void __launch_bounds__(256, MINB) band_lu_kernel(const double *__restrict__ Aent, int64_t ent_bstride,
                                                        double *__restrict__ LU, int64_t lu_bstride,
                                                        const BandDesc *__restrict__ desc, int nsp) {
  static_assert(8 % kBandR == 0 || kBandR % 8 == 0, "tile rows divide or are divided by the unroll");
  static_assert(kBandC == 8, "tile columns = the unroll");
  extern __shared__ double smem[];
  const int bi = blockIdx.x / nsp, a = blockIdx.x % nsp;
  const BandDesc d = desc[a];
  const int n = d.n, B = d.B, P = B + 1, W = 2 * B + 1;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int ntc = P / kBandC;
  const int tr = tid / ntc, tc = tid % ntc;
  const bool owner = tr < P / kBandR;
  const int pr0 = tr * kBandR, pc0 = tc * kBandC;
  // shared layout
  double *a_s = smem;                       // [P]  column k (raw); the retiring entry is zero
  double *u_s = a_s + P;                    // [P]  row k
  double *piv_s = u_s + P;                  // [2]  pivot, 1 / pivot
  double *dbuf = piv_s + 2;                 // [2][W] entering row (dense)
  double *ring = dbuf + 2 * W;              // [kBandD + 1][W] entry values in flight
  int32_t *sptr = (int32_t *)(ring + (kBandD + 1) * W);   // [n + 1]
  uint16_t *spos = (uint16_t *)(sptr + n + 1);             // [nent]
  for (int i = tid; i < 2 * P; i += blockDim.x) a_s[i] = 0.0;
  for (int i = tid; i < 2 * W; i += blockDim.x) dbuf[i] = 0.0;
  for (int i = tid; i <= n; i += blockDim.x) sptr[i] = d.ent_ptr[i];
  for (int i = tid; i < d.nent; i += blockDim.x) spos[i] = d.ent_pos[i];
  const double *ae = Aent + (int64_t)bi * ent_bstride + d.aoff;
  double *lu = LU + (int64_t)bi * lu_bstride + d.off;
  __syncthreads();
  if (warp == 0)
    for (int e = 0; e < kBandD; e++) band_issue(e, n, sptr, ae, ring, W, lane);
  double cell[kBandR][kBandC];
#pragma unroll
  for (int r = 0; r < kBandR; r++)
#pragma unroll
    for (int c = 0; c < kBandC; c++) cell[r][c] = 0.0;
  // the thread's entry of the factor row LU[k] (t = tid < W): a U entry (physical column pk + t) or
  // an L entry (physical row pk + t - B), both modulo P by one conditional subtraction
  const int tw = tid < W ? (tid <= B ? tid : tid - B) : 0;

  int pkb = 0;   // (k mod P) of the first step of the unrolled group
  for (int kb = -P; kb < n; kb += 8) {
#pragma unroll
    for (int u = 0; u < 8; u++) {
      const int k = kb + u, pk = pkb + u;
      const int rr = u % kBandR, cc = u % kBandC;   // compile-time after unrolling
      const bool rowown = owner && tr == (pkb + u - rr) / kBandR;
      const bool colown = owner && tc == pkb / kBandC;
      const bool live = k >= 0 && k < n;
      if (live) {   // b) publish the pivot row and column
        if (rowown) {
#pragma unroll
          for (int c = 0; c < kBandC; c++) u_s[pc0 + c] = (colown && c == cc) ? 0.0 : cell[rr][c];
          if (colown) {
            piv_s[0] = cell[rr][cc];
            piv_s[1] = __drcp_rn(cell[rr][cc]);
          }
        }
        if (colown) {
#pragma unroll
          for (int r = 0; r < kBandR; r++) a_s[pr0 + r] = (rowown && r == rr) ? 0.0 : cell[r][cc];
        }
      }
      __syncthreads();
      const int e = k + P;   // entering row
      double *db = dbuf + (e & 1) * W;
      if (warp == 0) {   // stage the entering row: clear row e - 2's entries, wait for row e's, scatter
        if (e >= 2 && e - 2 < n)
          for (int q = sptr[e - 2] + lane; q < sptr[e - 1]; q += 32) db[spos[q]] = 0.0;
        band_issue(e + kBandD, n, sptr, ae, ring, W, lane);
        cp_async_wait<kBandD>();
        __syncwarp();
        if (e < n) {
          const int q0 = sptr[e], cnt = sptr[e + 1] - q0;
          const double *src = ring + (e % (kBandD + 1)) * W;
          for (int q = lane; q < cnt; q += 32) db[spos[q0 + q]] = src[q];
        }
      }
      if (live) {   // c) rank-1 update of the tile; threads 0..2B write step k's factor row
        const double rinv = piv_s[1];
        if (owner) {
          double l[kBandR], uu[kBandC];
#pragma unroll
          for (int r = 0; r < kBandR; r++) l[r] = a_s[pr0 + r] * rinv;
#pragma unroll
          for (int c = 0; c < kBandC; c++) uu[c] = u_s[pc0 + c];
#pragma unroll
          for (int r = 0; r < kBandR; r++)
#pragma unroll
            for (int c = 0; c < kBandC; c++) cell[r][c] = fma(-l[r], uu[c], cell[r][c]);
        }
        if (tid < W) {
          int j = pk + tw;
          j -= j >= P ? P : 0;
          lu[(int64_t)k * W + tid] = tid == 0 ? piv_s[0] : tid <= B ? u_s[j] : a_s[j] * rinv;
        }
      }
      __syncthreads();
      // d) the retiring physical row/column pk takes the entering row/column e = k + P; offset 0 of
      //    the entering row is logical index k + 1, i.e. physical pk + 1 (mod P)
      const int pk1 = pk + 1 == P ? 0 : pk + 1;
      if (colown) {
        int o = pr0 - pk1;   // offset of physical row pr0 in the entering column
        o += o < 0 ? P : 0;
#pragma unroll
        for (int r = 0; r < kBandR; r++) {
          const int orr = o + r >= P ? o + r - P : o + r;
          if (!(rowown && r == rr)) cell[r][cc] = db[B + 1 + orr];
        }
      }
      if (rowown) {
        int o = pc0 - pk1;
        o += o < 0 ? P : 0;
#pragma unroll
        for (int c = 0; c < kBandC; c++) {
          const int oc = o + c >= P ? o + c - P : o + c;
          cell[rr][c] = db[oc];
        }
      }
    }
    pkb += 8;
    pkb -= pkb == P ? P : 0;
  }
}

// One warp per (batch item, species block): x = U^-1 L^-1 (P b) in the RCM order, un-permuted on
// the way out.  y lives in shared memory; the factor rows stream through a per-warp cp.async ring
// kBandD steps ahead (each step is a short dependent chain, so the loads must not sit on it).
// Forward substitution is column-oriented (step k updates y[k+1..k+B] with L(., k)), backward
// substitution row-oriented (a dot product with U(k, .) reduced by shuffles).
__global__ void band_solve_kernel(const double *__restrict__ LU, int64_t lu_bstride, const BandDesc *__restrict__ desc,
                                  const int32_t *__restrict__ perm_all, const int64_t *__restrict__ perm_off,
                                  const int64_t *__restrict__ vec_off, int64_t ndof, int nmax, int Bmax,
                                  const double *__restrict__ rhs, double *__restrict__ x, int nsp, int nbatch) {
  extern __shared__ double sm[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (w >= (int64_t)nbatch * nsp) return;
  const int b = (int)(w / nsp), a = (int)(w % nsp);
  const BandDesc d = desc[a];
  const double *A = LU + (int64_t)b * lu_bstride + d.off;
  const int32_t *perm = perm_all + perm_off[a];   // new -> old (within the species block)
  const int n = d.n, B = d.B, W = 2 * B + 1;
  const int RW = Bmax + 1;                        // ring row width
  const double *bb = rhs + (int64_t)b * ndof + vec_off[a];
  double *xb = x + (int64_t)b * ndof + vec_off[a];
  double *y = sm + (int64_t)wib * (nmax + Bmax + 1 + (kBandD + 1) * RW);
  double *ring = y + nmax + Bmax + 1;
  for (int i = lane; i < n + B + 1; i += 32) y[i] = i < n ? bb[perm[i]] : 0.0;   // zero pads past n
  // forward: ring rows hold L(k+1..k+B, k) = LU[k][B+1..2B]
  auto issue_f = [&](int k) {
    if (k < n)
      for (int t = lane; t < B; t += 32) cp_async8(ring + (k % (kBandD + 1)) * RW + t, A + (int64_t)k * W + B + 1 + t);
    cp_async_commit();
  };
  for (int k = 0; k < kBandD; k++) issue_f(k);
  for (int k = 0; k < n; k++) {
    issue_f(k + kBandD);
    cp_async_wait<kBandD>();
    __syncwarp();
    const double *row = ring + (k % (kBandD + 1)) * RW;
    const double yk = y[k];
    for (int t = lane; t < B; t += 32) y[k + 1 + t] = fma(-row[t], yk, y[k + 1 + t]);   // pads absorb t >= n-1-k
    __syncwarp();
  }
  cp_async_wait<0>();
  __syncwarp();
  for (int i = n + lane; i < n + B + 1; i += 32) y[i] = 0.0;
  // backward: ring rows hold U(k, k..k+B) = LU[k][0..B], k descending
  auto issue_b = [&](int s) {   // s-th backward step, k = n - 1 - s
    const int k = n - 1 - s;
    if (k >= 0)
      for (int t = lane; t <= B; t += 32) cp_async8(ring + (s % (kBandD + 1)) * RW + t, A + (int64_t)k * W + t);
    cp_async_commit();
  };
  for (int s = 0; s < kBandD; s++) issue_b(s);
  for (int s = 0; s < n; s++) {
    const int k = n - 1 - s;
    issue_b(s + kBandD);
    cp_async_wait<kBandD>();
    __syncwarp();
    const double *row = ring + (s % (kBandD + 1)) * RW;
    double acc = 0.0;
    for (int t = 1 + lane; t <= B; t += 32) acc = fma(row[t], y[k + t], acc);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) y[k] = (y[k] - acc) / row[0];
    __syncwarp();
  }
  for (int i = lane; i < n; i += 32) xb[perm[i]] = y[i];
}

}  // namespace landau
