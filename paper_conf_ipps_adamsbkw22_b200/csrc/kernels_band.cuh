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
#ifndef LANDAU_BAND_D
#define LANDAU_BAND_D 6
#endif
constexpr int kBandD = LANDAU_BAND_D;   // cp.async prefetch distance, in elimination steps
constexpr int kBandMaxP = 128;

struct BandDesc {             // per species block
  int64_t off;                // offset of the block in one batch item's LU storage
  int64_t aoff;               // offset of the block in one batch item's entry-value list (Aent)
  const int32_t *ent_ptr;     // [n+1] entering-row entry lists of the block's grid (host_setup.h)
  const uint16_t *ent_pos;    // [nent] position in the entering row: 0..B row part, B+1..2B column part
  int n, B, Pp, nent;         // B: the half-bandwidth padded so that Pp = B + 1 is a multiple of 8
};

// Aent[b][aoff + e] = shift M[s] + eta A_E[s] - J[b][J_off + s], s = slot of entry e: the block's
// entries in consumption order (eta = E_z e_a / m_a, the advection term of Eq. 4; 0 without a field)
__global__ void band_gather_kernel(int64_t nent, const int32_t *__restrict__ ent_slot, const double *__restrict__ M,
                                   const double *__restrict__ AE, double eta, const double *__restrict__ J,
                                   int64_t J_bstride, int64_t J_off, double shift, double *__restrict__ Aent,
                                   int64_t ent_bstride, int64_t aoff, int nbatch) {
  const int64_t total = nent * nbatch;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / nent, e = k % nent;
    const int32_t s = ent_slot[e];
    Aent[b * ent_bstride + aoff + e] = fma(shift, M[s], fma(eta, AE[s], -J[b * J_bstride + J_off + s]));
  }
}

__device__ __forceinline__ void cp_async8(void *smem, const void *gmem) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

constexpr int kBandE = 2;   // entry values per thread and group of 8 entering rows (host-checked)

// 1 / a for a normal pivot: MUFU seed, one cubically convergent correction y (1 + e + e^2)
// (seed error ~2^-22 -> ~2^-66; three dependent FP64 operations instead of four)
__device__ __forceinline__ double rcp_newton(double a) {
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(a));
  const double e = fma(-a, y, 1.0);
  return fma(fma(e, e, e), y, y);
}

// One CTA per (batch item, species block).  The P x P active square (P = B + 1, B the padded
// half-bandwidth, P a multiple of 8) of the outer-product elimination lives in REGISTERS, cut into
// R x C tiles, one per thread, addressed circularly: logical row/column i sits in physical
// row/column i mod P.  Per step: the owners of the retiring physical row/column publish them in
// shared memory, every thread applies the update to its tile (the retiring row/column see zero
// multipliers), threads 0..2B write the factor rows, and the owners of the retiring row/column load
// the entering row/column k + P from a dense buffer.  Steps run in groups of 8 (P is a multiple of
// 8, so the owners index their registers statically in each unrolled copy).  The 8 rows entering in
// group g are staged in bulk, once per group: their entry values (contiguous in Aent) are loaded
// into registers two groups ahead, scattered into dense buffer set g mod 3 at the first step of
// group g - 1, and scattered back to zero at the first step of group g + 2; each entering row is
// stored twice (row part at [0, P) and [P, 2P), column part at [2P, 3P) and [3P, 4P)) so the
// circular window offsets need no modulo.  Groups of steps k < 0 only load the window.
// Elimination steps k, k+1 (k even) share one barrier.  The owners of the two
// retiring rows / columns (same tile row and tile column, since k is even and R, C are even) publish
// them raw; the owner of the 2 x 2 corner publishes the pivots and L(k+1, k); every thread then
// forms, for its own rows and columns,
//   l0 = A(., k) / p0,  l1 = (A(., k+1) - l0 A(k, k+1)) / p1,  u0 = A(k, .),  u1 = A(k+1, .) - L(k+1,k) u0
// and applies cell -= l0 u0 + l1 u1 (the same outer-product elimination, two steps fused).  Needs the
// half-bandwidth padding B + 2 <= P so row k+1's band (to column k+1+B_true) lies in the window.
template <int kBandR, int kBandC, int MINB>
__global__ void __launch_bounds__(256, MINB) band_lu2_kernel(const double *__restrict__ Aent, int64_t ent_bstride,
                                                         double *__restrict__ LU, int64_t lu_bstride,
                                                         const BandDesc *__restrict__ desc, int nsp) {
  static_assert(kBandR % 2 == 0 && (8 % kBandR == 0 || kBandR % 8 == 0), "tile rows: even, divide the group");
  static_assert(kBandC == 8, "tile columns = the group");
  extern __shared__ double smem[];
  const int bi = blockIdx.x / nsp, a = blockIdx.x % nsp;
  const BandDesc d = desc[a];
  const int n = d.n, B = d.B, P = B + 1, W = 2 * B + 1;
  const int tid = threadIdx.x, T = blockDim.x;
  const int ntc = P / kBandC;
  const int tr = tid / ntc, tc = tid % ntc;
  const bool owner = tr < P / kBandR;
  const int pr0 = tr * kBandR, pc0 = tc * kBandC;
  // shared layout, double-buffered by pair parity: column k, column k+1 (raw), row k, row k+1 (raw,
  // padded: physical column j at upos(j) = j + 2 (j / 8), so the 16-byte loads of the tile columns
  // hit distinct banks), corner scalars (p0, 1/p0, L(k+1,k), p1, 1/p1, U(k,k+1), -, -)
  const int PU = P / 8 * 10, SHW = 2 * P + 2 * PU + 8, W4 = 4 * P;
  auto upos = [](int j) { return j + (j >> 3) * 2; };
  double *sh0 = smem;
  // [3][8][4P] entering rows (dense), one set per group: row part [0, P) and column part [2P, 3P),
  // each stored twice (copy at +P) so the circular window offsets need no modulo
  double *dbuf = sh0 + 2 * SHW;
  int32_t *sptr = (int32_t *)(dbuf + 24 * W4);             // [n + 1]
  uint16_t *spos = (uint16_t *)(sptr + n + 1);             // [nent] base position in a 4P row
  for (int i = tid; i < 2 * SHW; i += T) sh0[i] = 0.0;
  for (int i = tid; i < 24 * W4; i += T) dbuf[i] = 0.0;
  for (int i = tid; i <= n; i += T) sptr[i] = d.ent_ptr[i];
  for (int i = tid; i < d.nent; i += T) spos[i] = d.ent_pos[i];
  const double *ae = Aent + (int64_t)bi * ent_bstride + d.aoff;
  double *lu = LU + (int64_t)bi * lu_bstride + d.off;
  const int ngroups = (n + 7) / 8;
  auto grange = [&](int g, int &q0, int &q1) {
    q0 = g < ngroups ? sptr[8 * g] : 0;
    q1 = g < ngroups ? sptr[min(8 * g + 8, n)] : 0;
  };
  double vin[kBandE];
  __syncthreads();
  {
    int q0, q1;
    grange(0, q0, q1);
#pragma unroll
    for (int m = 0; m < kBandE; m++)
      if (q0 + tid + m * T < q1) {
        const int q = spos[q0 + tid + m * T];
        dbuf[q] = dbuf[q + P] = ae[q0 + tid + m * T];
      }
    grange(1, q0, q1);
#pragma unroll
    for (int m = 0; m < kBandE; m++) vin[m] = q0 + tid + m * T < q1 ? ae[q0 + tid + m * T] : 0.0;
  }
  double cell[kBandR][kBandC];
#pragma unroll
  for (int r = 0; r < kBandR; r++)
#pragma unroll
    for (int c = 0; c < kBandC; c++) cell[r][c] = 0.0;
  // writer: thread t < W writes entry t of LU[k] and of LU[k+1]; U entries sit at physical column
  // pk + t, L entries at physical row pk + t - B (mod P)
  const int tw = tid < W ? (tid <= B ? tid : tid - B) : 0;

  int pkb = 0;
  for (int kb = -P, g = 0; kb < n; kb += 8, g++) {
    const double *dset = dbuf + (g % 3) * 8 * W4;
#pragma unroll
    for (int u = 0; u < 8; u += 2) {
      const int k = kb + u, pk = pkb + u;
      const int rr = u % kBandR, cc = u % kBandC;   // rows rr, rr+1 / columns cc, cc+1 of the tile
      const bool rowown = owner && tr == (pkb + u - rr) / kBandR;
      const bool colown = owner && tc == pkb / kBandC;
      const bool live0 = k >= 0 && k < n, live1 = k + 1 < n;
      double *sh = sh0 + ((u >> 1) & 1) * SHW;
      double *a0_s = sh, *a1_s = sh + P, *u0_s = sh + 2 * P, *u1_s = sh + 2 * P + PU, *sc = sh + 2 * P + 2 * PU;
      if (u == 0 && g >= 2) {   // clear group g - 2's rows from set (g + 1) mod 3
        int q0, q1;
        grange(g - 2, q0, q1);
        double *ds = dbuf + ((g + 1) % 3) * 8 * W4;
#pragma unroll
        for (int m = 0; m < kBandE; m++)
          if (q0 + tid + m * T < q1) {
            const int q = spos[q0 + tid + m * T];
            ds[q] = ds[q + P] = 0.0;
          }
      }
      if (live0) {   // b) publish rows k, k+1 and columns k, k+1 (zero at the retiring positions)
        if (rowown) {
#pragma unroll
          for (int c = 0; c < kBandC; c++) {
            const bool ret = colown && (c == cc || c == cc + 1);
            u0_s[tc * 10 + c] = ret ? 0.0 : cell[rr][c];
            u1_s[tc * 10 + c] = ret ? 0.0 : cell[rr + 1][c];
          }
          if (colown) {   // the 2 x 2 corner: p1 = det / p0 and 1 / p1 = p0 / det, so both
                          // reciprocals start at once (shorter serial chain before the barrier)
            const double p0 = cell[rr][cc], ukk1 = cell[rr][cc + 1], c10 = cell[rr + 1][cc];
            const double det = fma(p0, cell[rr + 1][cc + 1], -(c10 * ukk1));
            const double r0 = rcp_newton(p0);
            const double rdet = live1 ? rcp_newton(det) : 0.0;
            sc[0] = p0;
            sc[1] = r0;
            sc[2] = c10 * r0;
            sc[3] = det * r0;
            sc[4] = p0 * rdet;
            sc[5] = ukk1;
          }
        }
        if (colown) {
#pragma unroll
          for (int r = 0; r < kBandR; r++) {
            const bool ret = rowown && (r == rr || r == rr + 1);
            a0_s[pr0 + r] = ret ? 0.0 : cell[r][cc];
            a1_s[pr0 + r] = ret ? 0.0 : cell[r][cc + 1];
          }
        }
      }
      __syncthreads();
      if (u == 0) {   // scatter group g + 1 into set (g + 1) mod 3; load group g + 2
        int q0, q1;
        grange(g + 1, q0, q1);
        double *ds = dbuf + ((g + 1) % 3) * 8 * W4;
#pragma unroll
        for (int m = 0; m < kBandE; m++)
          if (q0 + tid + m * T < q1) {
            const int q = spos[q0 + tid + m * T];
            ds[q] = ds[q + P] = vin[m];
          }
        grange(g + 2, q0, q1);
#pragma unroll
        for (int m = 0; m < kBandE; m++) vin[m] = q0 + tid + m * T < q1 ? ae[q0 + tid + m * T] : 0.0;
      }
      if (live0) {   // c) rank-2 update; threads 0..2B write LU[k] and LU[k+1]
        const double r0 = sc[1], l10 = sc[2], r1 = sc[4], ukk1 = sc[5];
        if (owner) {
          double l0[kBandR], l1[kBandR], u0[kBandC], u1[kBandC];
          const double2 *a02 = reinterpret_cast<const double2 *>(a0_s + pr0);
          const double2 *a12 = reinterpret_cast<const double2 *>(a1_s + pr0);
#pragma unroll
          for (int r = 0; r < kBandR / 2; r++) {
            const double2 x0 = a02[r], x1 = a12[r];
            l0[2 * r] = x0.x * r0;
            l0[2 * r + 1] = x0.y * r0;
            l1[2 * r] = fma(-l0[2 * r], ukk1, x1.x) * r1;
            l1[2 * r + 1] = fma(-l0[2 * r + 1], ukk1, x1.y) * r1;
          }
          const double2 *u02 = reinterpret_cast<const double2 *>(u0_s + tc * 10);
          const double2 *u12 = reinterpret_cast<const double2 *>(u1_s + tc * 10);
#pragma unroll
          for (int c = 0; c < kBandC / 2; c++) {
            const double2 y0 = u02[c], y1 = u12[c];
            u0[2 * c] = y0.x;
            u0[2 * c + 1] = y0.y;
            u1[2 * c] = fma(-l10, y0.x, y1.x);
            u1[2 * c + 1] = fma(-l10, y0.y, y1.y);
          }
#pragma unroll
          for (int r = 0; r < kBandR; r++)
#pragma unroll
            for (int c = 0; c < kBandC; c++) cell[r][c] = fma(-l1[r], u1[c], fma(-l0[r], u0[c], cell[r][c]));
        }
        if (tid < W) {
          int j = pk + tw;
          j -= j >= P ? P : 0;
          double v0, v1;
          if (tid == 0) {
            v0 = sc[0];
            v1 = sc[3];
          } else if (tid <= B) {   // U(k, k+t) and U(k+1, k+1+t): physical columns j and j + 1
            int j1 = j + 1;
            j1 -= j1 >= P ? P : 0;
            v0 = tid == 1 ? ukk1 : u0_s[upos(j)];
            v1 = fma(-l10, u0_s[upos(j1)], u1_s[upos(j1)]);
          } else {                 // L(k+t, k) and L(k+1+t, k+1): physical rows j and j + 1
            int j1 = j + 1;
            j1 -= j1 >= P ? P : 0;
            v0 = tid == B + 1 ? l10 : a0_s[j] * r0;
            v1 = fma(-a0_s[j1] * r0, ukk1, a1_s[j1]) * r1;
          }
          lu[(int64_t)k * W + tid] = v0;
          if (live1) lu[(int64_t)(k + 1) * W + tid] = v1;
        }
      }
      // d) the retiring physical rows/columns pk, pk+1 take the entering rows/columns k+P, k+P+1
      //    (rows u, u+1 of the group's set), in that order
#pragma unroll
      for (int h = 0; h < 2; h++) {
        const double *db = dset + (u + h) * W4;
        const int pkh = pk + h;
        const int pk1 = pkh + 1 == P ? 0 : pkh + 1;
        const int rh = rr + h, ch = cc + h;
        if (colown) {
          int o = pr0 - pk1;
          o += o < 0 ? P : 0;
          const double *dc = db + 2 * P + o;   // duplicated column part: no wrap
#pragma unroll
          for (int r = 0; r < kBandR; r++)
            if (!(rowown && r == rh)) cell[r][ch] = dc[r];
        }
        if (rowown) {
          int o = pc0 - pk1;
          o += o < 0 ? P : 0;
          const double *dr = db + o;           // duplicated row part: no wrap
#pragma unroll
          for (int c = 0; c < kBandC; c++) cell[rh][c] = dr[c];
        }
      }
    }
    pkb += 8;
    pkb -= pkb == P ? P : 0;
  }
}

// ---- column-warp factorisation with look-ahead (round 2) ------------------------------------------
// The same outer-product band LU (Golub-Van Loan Alg. 4.3.1, rank-1 steps) and the same step-major
// factor rows as band_lu2_kernel, with the P x P window (P = 8 NC, a template constant) distributed so
// that the per-step synchronisation is a producer/consumer hand-off instead of a CTA barrier:
//   * warp w owns the physical columns w + 8 c (c < NC: cyclic, so consecutive pivots belong to
//     different warps); lane l owns the physical rows l + 32 m (m < MR = ceil(P / 32)):
//     cell[m][c] = window(l + 32 m, w + 8 c);
//   * step k (pivot at physical index pk = k mod P) needs the multipliers l_k (P values) from the
//     warp owning column pk, and the pivot row's values in each warp's own columns, which the warp's
//     lane pk mod 32 holds -- so only l_k crosses warps, through a shared-memory ring, guarded by the
//     named barrier 1 + k mod 9: its producer bar.arrive()s, the other warps bar.sync();
//   * look-ahead: during step k the owner of column pk + 1 applies step k to that column first, forms
//     l_{k+1} = column / pivot and publishes it before updating its other columns, so the next step's
//     hand-off overlaps the current step's rank-1 update;
//   * every 8 steps one CTA barrier stages the next group's entering rows (dense, indexed by physical
//     position, three sets) and writes the previous group's factor rows from the l / u rings
//     (coalesced); it also bounds how far any warp runs ahead (9 barrier ids, 16 ring slots suffice).
// Retiring row pk: l_k = 0 there, so the update leaves the entering row (written just before) intact;
// retiring column pk: updated like the others, then overwritten by the entering column.
constexpr int kCwRing = 16;   // ring slots of l_k / row-k values (>= 8 steps of a group + look-ahead + lag)

__device__ __forceinline__ void named_sync(int id, int cnt) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(cnt) : "memory"); }
__device__ __forceinline__ void named_arrive(int id, int cnt) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(cnt) : "memory"); }

template <int NC>
__global__ void __launch_bounds__(256, 2) band_lu_cw_kernel(const double *__restrict__ Aent, int64_t ent_bstride,
                                                            double *__restrict__ LU, int64_t lu_bstride,
                                                            const BandDesc *__restrict__ desc, int nsp) {
  constexpr int P = 8 * NC, W = 2 * P - 1, MR = (P + 31) / 32, T = 256;
  extern __shared__ double smem[];
  const int bi = blockIdx.x / nsp, a = blockIdx.x % nsp;
  const BandDesc d = desc[a];   // d.B + 1 == P (host-checked)
  const int n = d.n;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  double *Lr = smem;                      // [kCwRing][P] l_k by physical row (0 at the pivot row)
  double *Ur = Lr + kCwRing * P;          // [kCwRing][P] row k, warp-major: column w + 8 c at w NC + c
  double *eb = Ur + kCwRing * P;          // [3][8][2P] entering rows: row part [0, P) warp-major, column part [P, 2P)
  const double *ae = Aent + (int64_t)bi * ent_bstride + d.aoff;
  double *lu = LU + (int64_t)bi * lu_bstride + d.off;
  const int ngroups = (n + 7) / 8;
  for (int i = tid; i < 3 * 16 * P; i += T) eb[i] = 0.0;
  // an entry of group g (entering rows 8g..8g+7): its dense index from the band_lu2 position code
  // (ri 4P + (row part: p | column part: 2P + p - P)), whose logical index is ni + p - 2B - 1 (column
  // part) or ni + p - B (row part) with B = P - 1, i.e. physical (ni + p + 1) mod P either way
  auto stage = [&](int g, double *v, int *ix) {
#pragma unroll
    for (int m = 0; m < kBandE; m++) {
      v[m] = 0.0;
      ix[m] = -1;
    }
    if (g >= ngroups) return;
    const int q0 = d.ent_ptr[8 * g], q1 = d.ent_ptr[min(8 * g + 8, n)];
#pragma unroll
    for (int m = 0; m < kBandE; m++) {
      const int q = q0 + tid + m * T;
      if (q < q1) {
        const int code = d.ent_pos[q];
        const int ri = code / (4 * P), qq = code - ri * 4 * P;
        const bool isrow = qq < P;
        const int pp = isrow ? qq : qq - P;
        const int phys = (8 * g + ri + pp + 1) % P;   // row part stored warp-major: (phys % 8) NC + phys / 8
        ix[m] = ri * 2 * P + (isrow ? (phys & 7) * NC + (phys >> 3) : P + phys);
        v[m] = ae[q];
      }
    }
  };
  double vin[kBandE];
  int vix[kBandE];
  __syncthreads();
  for (int g0 = 0; g0 < 2; g0++) {   // groups 0 and 1 into sets 0 and 1; group 2 waits in registers
    stage(g0, vin, vix);
#pragma unroll
    for (int m = 0; m < kBandE; m++)
      if (vix[m] >= 0) eb[g0 * 16 * P + vix[m]] = vin[m];
  }
  stage(2, vin, vix);
  // factor rows of steps [k0, k0 + 8) from the rings: t < P: U(k, k + t), t >= P: L(k + t - P + 1, k)
  auto write_rows = [&](int k0) {
    for (int r = 0; r < 8; r++) {
      const int kk = k0 + r;
      if (kk < 0 || kk >= n) continue;
      const int pkk = kk % P, sl = kk & (kCwRing - 1);
      for (int t = tid; t < W; t += T) {
        int j = pkk + (t < P ? t : t - P + 1);
        j -= j >= P ? P : 0;
        lu[(int64_t)kk * W + t] = t < P ? Ur[sl * P + (j & 7) * NC + (j >> 3)] : Lr[sl * P + j];
      }
    }
  };
  auto group_barrier = [&](int g, int kb) {   // stage group g + 1, clear set (g + 2) % 3, rows of group g - 1
    __syncthreads();
#pragma unroll
    for (int m = 0; m < kBandE; m++)
      if (vix[m] >= 0) eb[((g + 1) % 3) * 16 * P + vix[m]] = vin[m];
    double2 *cs = reinterpret_cast<double2 *>(eb + ((g + 2) % 3) * 16 * P);
    for (int i = tid; i < 8 * P; i += T) cs[i] = make_double2(0.0, 0.0);
    stage(g + 2, vin, vix);
    write_rows(kb - 8);
    __syncthreads();
  };

  double cell[MR][NC];
#pragma unroll
  for (int m = 0; m < MR; m++)
#pragma unroll
    for (int c = 0; c < NC; c++) cell[m][c] = 0.0;
  const int c0 = w * NC;   // this warp's segment of a warp-major row (Ur, entering row parts)
  // the pivot row's values of this warp's columns -> ring slot sl (lane rl of slot rm holds them)
  // (16-byte accesses for even NC: c0, the ring rows and the dense rows are 16-byte aligned)
  auto put_row = [&](double *dst, int rl, int rm) {
#pragma unroll
    for (int m = 0; m < MR; m++)
      if (m == rm && lane == rl) {
        if constexpr (NC % 2 == 0) {
#pragma unroll
          for (int c = 0; c < NC; c += 2) reinterpret_cast<double2 *>(dst)[c / 2] = make_double2(cell[m][c], cell[m][c + 1]);
        } else {
#pragma unroll
          for (int c = 0; c < NC; c++) dst[c] = cell[m][c];
        }
      }
  };
  auto take_row = [&](const double *src, int rl, int rm) {   // the entering row into lane rl, slot rm
#pragma unroll
    for (int m = 0; m < MR; m++)
      if (m == rm && lane == rl) {
        if constexpr (NC % 2 == 0) {
#pragma unroll
          for (int c = 0; c < NC; c += 2) {
            const double2 v = reinterpret_cast<const double2 *>(src)[c / 2];
            cell[m][c] = v.x;
            cell[m][c + 1] = v.y;
          }
        } else {
#pragma unroll
          for (int c = 0; c < NC; c++) cell[m][c] = src[c];
        }
      }
  };
  auto take_col = [&](const double *src, int oc, int pk) {    // the entering column into column oc
#pragma unroll
    for (int c = 0; c < NC; c++)
      if (c == oc) {
#pragma unroll
        for (int m = 0; m < MR; m++) {
          const int row = lane + 32 * m;
          if ((m < MR - 1 || row < P) && row != pk) cell[m][c] = src[row];
        }
      }
  };
  // l_{k+1} from column pn (physical) with step k applied: multipliers l, the old pivot row's value at
  // column pn from lane rl (slot rm), whose row is the entering row from this step on (value ev)
  auto produce = [&](const double *l, int pn, int rl, int rm, double ev, double *dst) {
    const int nc = pn >> 3;
#pragma unroll
    for (int c = 0; c < NC; c++)
      if (c == nc) {
        double uv = cell[0][c];
#pragma unroll
        for (int m = 1; m < MR; m++) uv = rm == m ? cell[m][c] : uv;
        uv = __shfl_sync(0xffffffffu, uv, rl);
        double t[MR];
#pragma unroll
        for (int m = 0; m < MR; m++) t[m] = (m == rm && lane == rl) ? ev : fma(-l[m], uv, cell[m][c]);
        const int prm = pn >> 5;
        double tv = t[0];
#pragma unroll
        for (int m = 1; m < MR; m++) tv = prm == m ? t[m] : tv;
        const double pv = __shfl_sync(0xffffffffu, tv, pn & 31);
        const double r = rcp_newton(pv);
#pragma unroll
        for (int m = 0; m < MR; m++) {
          const int row = lane + 32 * m;
          if (m < MR - 1 || row < P) dst[row] = row == pn ? 0.0 : t[m] * r;
        }
      }
  };

  // ---- steps k = -P .. -1: the first P rows / columns enter the window; l_0 at the end ----
  int pk = 0, g = 0;
  for (int kb = -P; kb < 0; kb += 8, g++) {
    if (g > 0) group_barrier(g, kb);
    else __syncthreads();
    const double *es = eb + (g % 3) * 16 * P;
#pragma unroll 1
    for (int u = 0; u < 8; u++, pk++) {   // pk = k + P < P
      take_row(es + u * 2 * P + c0, pk & 31, pk >> 5);
      if (w == (pk & 7)) take_col(es + u * 2 * P + P, pk >> 3, pk);
    }
  }
  pk = 0;
  if (w == 0 && n > 0) {   // l_0 (column 0 belongs to warp 0); nothing to apply yet
    const double z[MR] = {};
    produce(z, 0, 32, MR, 0.0, Lr);
    __syncwarp();
    named_arrive(1, T);
  }
  // ---- steps k = 0 .. n - 1 ----
  int bid = 1;   // named barrier of step k: 1 + k mod 9
  for (int kb = 0; kb < n; kb += 8, g++) {
    group_barrier(g, kb);
    const double *es = eb + (g % 3) * 16 * P;
#pragma unroll 1
    for (int u = 0; u < 8; u++) {
      const int k = kb + u;
      if (k >= n) break;
      const int ow = pk & 7, oc = pk >> 3;         // owner warp / column slot of the retiring column
      const int rl = pk & 31, rm = pk >> 5;        // owner lane / slot of the retiring row
      const int sl = k & (kCwRing - 1);
      const int pn = pk + 1 == P ? 0 : pk + 1;
      const int bid1 = bid == 9 ? 1 : bid + 1;
      if (w != ow) named_sync(bid, T);
      double l[MR], uu[NC];
#pragma unroll
      for (int m = 0; m < MR; m++) {
        const int row = lane + 32 * m;
        l[m] = (m < MR - 1 || row < P) ? Lr[sl * P + row] : 0.0;
      }
      if (k + 1 < n && w == (pn & 7)) {   // look-ahead first: l_{k+1} (the next step's only hand-off)
        produce(l, pn, rl, rm, es[u * 2 * P + (pn & 7) * NC + (pn >> 3)], Lr + ((k + 1) & (kCwRing - 1)) * P);
        __syncwarp();
        named_arrive(bid1, T);
      }
      put_row(Ur + sl * P + c0, rl, rm);
      __syncwarp();
#pragma unroll
      for (int c = 0; c < NC; c++) uu[c] = Ur[sl * P + c0 + c];
      take_row(es + u * 2 * P + c0, rl, rm);   // the entering row k + P takes physical row pk
#pragma unroll
      for (int m = 0; m < MR; m++)             // rank-1 update (column pn again: the same fma)
#pragma unroll
        for (int c = 0; c < NC; c++) cell[m][c] = fma(-l[m], uu[c], cell[m][c]);
      if (w == ow) take_col(es + u * 2 * P + P, oc, pk);   // the entering column k + P
      pk = pn;
      bid = bid1;
    }
  }
  __syncthreads();
  write_rows(8 * ((n - 1) / 8));   // the last group's rows
}

// One warp per (batch item, species block): x = U^-1 L^-1 (P b) in the RCM order, un-permuted on
// the way out.  y lives in shared memory; the factor rows stream through a per-warp cp.async ring
// kBandD steps ahead (each step is a short dependent chain, so the loads must not sit on it).
// Forward substitution is column-oriented (step k updates y[k+1..k+B] with L(., k)), backward
// substitution row-oriented (a dot product with U(k, .) reduced by shuffles).
__global__ void band_solve_kernel(const double *__restrict__ LU, int64_t lu_bstride, const BandDesc *__restrict__ desc,
                                  const int32_t *__restrict__ perm_all, const int64_t *__restrict__ perm_off,
                                  const int64_t *__restrict__ vec_off, int64_t ndof, int nmax, int Bmax,
                                  const double *__restrict__ rhs, double *__restrict__ x, int nsp, int nbatch,
                                  const double *__restrict__ yfwd) {
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
  if (yfwd) {   // the fused factorisation already eliminated forward: y = L^-1 b (RCM order)
    const double *yb = yfwd + (int64_t)b * ndof + vec_off[a];
    for (int i = lane; i < n + B + 1; i += 32) y[i] = i < n ? yb[i] : 0.0;
  } else {
    for (int i = lane; i < n + B + 1; i += 32) y[i] = i < n ? bb[perm[i]] : 0.0;   // zero pads past n
  }
  // forward: ring rows hold L(k+1..k+B, k) = LU[k][B+1..2B]
  auto issue_f = [&](int k) {
    if (k < n)
      for (int t = lane; t < B; t += 32) cp_async8(ring + (k % (kBandD + 1)) * RW + t, A + (int64_t)k * W + B + 1 + t);
    cp_async_commit();
  };
  const int nf = yfwd ? 0 : n;   // forward steps
  for (int k = 0; k < kBandD; k++) issue_f(k < nf ? k : n);
  for (int k = 0; k < nf; k++) {
    issue_f(k + kBandD < nf ? k + kBandD : n);
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
