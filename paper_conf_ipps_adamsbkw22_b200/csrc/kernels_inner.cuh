// kernels_inner.cuh -- the inner integral (a-2): directed and symmetric pair kernels, split-j and slot reductions, tensor-cache fill
// (split out of landau.cu; included once, by landau.cu)
#pragma once
#include <cstdint>

#include "kernels.cuh"

namespace landau {

// build-time tuning knobs of the symmetric inner kernel (defaults = measured best on B200)
#ifndef LANDAU_SYM_UNROLL
#define LANDAU_SYM_UNROLL 2
#endif
constexpr int kSymUnroll = LANDAU_SYM_UNROLL;
#ifndef LANDAU_MIR_UNROLL
#define LANDAU_MIR_UNROLL 1
#endif
constexpr int kMirUnroll = LANDAU_MIR_UNROLL;
#ifndef LANDAU_SYM_WARPS
#define LANDAU_SYM_WARPS 8   // measured (mirror kernel, C4): 8 warps x 1 block 2.89 ms, 4 x 2 3.13, 2 x 4 3.16
#endif
#ifndef LANDAU_SYM_MINB
#define LANDAU_SYM_MINB 1
#endif
#ifndef LANDAU_MIR_UNROLL
#define LANDAU_MIR_UNROLL 1
#endif

// ------------------------------------------------------------------------------------------------
// N2: inner integral.  Work is warp-granular: a warp owns 32*TPT consecutive targets of one batch
// item and one split of the source range (split-j), so the target tiling never pads across batch
// items.  Sources are staged per warp through shared memory, 32 at a time (one per lane), and every
// lane then reads the same source (broadcast LDS.128).  Coefficients of the elliptic fits live in
// registers (see kernels.cuh).  out = [batch][nsplit][5][nt] partials (or G when nsplit == 1).
// ------------------------------------------------------------------------------------------------
constexpr int kInnerTB = 128;
constexpr int kInnerWarps = kInnerTB / 32;

template <int TPT, int MINB>
__global__ void __launch_bounds__(kInnerTB, MINB) inner_kernel(int64_t N, int64_t t0, int64_t nt, int64_t split_len,
                                                             int nsplit, int64_t wtiles, int64_t nitems,
                                                             const double *__restrict__ pr, const double *__restrict__ pz,
                                                             const double *__restrict__ wT, double *__restrict__ out,
                                                             int64_t out_bstride) {
  __shared__ double2 s_rz[kInnerWarps][32], s_w[kInnerWarps][32], s_wz[kInnerWarps][32];   // (wkz, rb^2)
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  stage_pair_coef(s_coef, s_ltab);
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t item = (int64_t)blockIdx.x * kInnerWarps + wid;
  if (item >= nitems) return;   // whole warp: no block-level barrier follows
  const int64_t b = item / (nsplit * wtiles);
  const int64_t rem = item % (nsplit * wtiles);
  const int split = (int)(rem / wtiles);
  const int64_t wt = rem % wtiles;
  const double *wb = wT + b * 3 * N;
  int64_t ti[TPT];
  double tr[TPT], tz[TPT], tr2[TPT];
  Acc5 acc[TPT];
#pragma unroll
  for (int t = 0; t < TPT; t++) {
    ti[t] = wt * 32 * TPT + t * 32 + lane;
    const int64_t gi = t0 + (ti[t] < nt ? ti[t] : nt - 1);
    tr[t] = pr[gi];
    tz[t] = pz[gi];
    tr2[t] = tr[t] * tr[t];
    acc[t] = Acc5{0.0, 0.0, 0.0, 0.0, 0.0};
  }
  const int64_t j0 = (int64_t)split * split_len;
  const int64_t j1 = min(N, j0 + split_len);
  for (int64_t jt = j0; jt < j1; jt += 32) {
    const int64_t j = jt + lane;
    __syncwarp();
    if (j < j1) {
      const double rj = pr[j];
      s_rz[wid][lane] = make_double2(rj, pz[j]);
      s_w[wid][lane] = make_double2(wb[j], wb[N + j]);
      s_wz[wid][lane] = make_double2(wb[2 * N + j], rj * rj);
    }
    __syncwarp();
    const int n = (int)min((int64_t)32, j1 - jt);
#pragma unroll 2
    for (int k = 0; k < n; k++) {
      const double2 rz = s_rz[wid][k], w = s_w[wid][k], wz = s_wz[wid][k];
#pragma unroll
      for (int t = 0; t < TPT; t++) landau_pair(tr[t], tz[t], tr2[t], rz.x, rz.y, wz.y, w.x, w.y, wz.x, cf, acc[t]);
    }
  }
  double *o = out + b * out_bstride + (int64_t)split * 5 * nt;
#pragma unroll
  for (int t = 0; t < TPT; t++) {
    if (ti[t] < nt) {
      o[ti[t]] = acc[t].drr;
      o[nt + ti[t]] = acc[t].drz;
      o[2 * nt + ti[t]] = acc[t].dzz;
      o[3 * nt + ti[t]] = acc[t].kr;
      o[4 * nt + ti[t]] = acc[t].kz;
    }
  }
}

// ------------------------------------------------------------------------------------------------
// N2 (symmetric): each unordered pair of points is evaluated once.  The points
// are cut into T tiles of 32.  A warp item is one j-tile b (its 32 points and their reverse-sum
// accumulators in warp-private shared memory) against one or two i-tiles a1 < a2 < b, or the
// diagonal item (b, b).  Lane L holds target i = a*32 + L (forward sums in registers); at step k it
// pairs with j = b*32 + ((L + k) mod 32), so the 32 lanes touch 32 distinct j each step
// (conflict-free, no atomics).  Diagonal items run k = 1..16 (lanes < 16 only at k = 16) so every
// unordered pair is visited exactly once.  Two i-tiles per item give two independent pair chains
// per lane (the FP64 pipe needs the ILP) and share one accumulator update per step.
// Every item writes 32-point partial "slots"; reduce_sym_kernel sums, for each tile, its slots in a
// fixed host-built order -> bitwise reproducible.  part = [batch][nslots][5][32].
// ------------------------------------------------------------------------------------------------
constexpr int kSymWarps = LANDAU_SYM_WARPS;
#ifndef LANDAU_SYM_NI
#define LANDAU_SYM_NI 2
#endif
constexpr int kSymNI = LANDAU_SYM_NI;   // max i-tiles per item (independent pair chains per lane)
static_assert(kSymNI >= 1 && kSymNI <= 3, "sym items carry 1..3 i-tiles");

struct SymItem {   // host-built, see landau_create
  int a[3];        // i-tiles (n of them, all < b); n == 0: the diagonal item (b, b)
  int b, n;
  int slot;        // first of the item's consecutive partial slots: one per i-tile (or the diagonal's
                   // forward sums), then the j-tile's reverse sums
};

__device__ __forceinline__ void sym_load_i(const double *pr, const double *pz, const double *wb, int64_t N, int64_t i,
                                           double zpad, double &r, double &z, double &wd, double &wkr, double &wkz) {
  const bool v = i < N;   // padding: far away, zero weights -- contributes nothing, never read back
  r = v ? pr[i] : 1.0;
  z = v ? pz[i] : zpad;
  wd = v ? wb[i] : 0.0;
  wkr = v ? wb[N + i] : 0.0;
  wkz = v ? wb[2 * N + i] : 0.0;
}

__device__ __forceinline__ void sym_store(double *o, int lane, const Acc5 &a) {
  o[lane] = a.drr;
  o[32 + lane] = a.drz;
  o[64 + lane] = a.dzz;
  o[96 + lane] = a.kr;
  o[128 + lane] = a.kz;
}

// NI i-tiles against the warp's j-tile (NI independent pair chains per lane and step); DIAG: the
// tile against itself, k = 1..16 (lanes < 16 only at k = 16) -- every unordered pair exactly once.
// The reverse sums travel with their j: at step k lane L holds the accumulator of j = (L + k) mod 32
// and hands it to lane L - 1 by a shuffle, so consecutive steps carry no memory fence and their
// (long, independent) pair evaluations overlap; the j data itself is read-only shared memory.
template <int NI, bool DIAG, bool MASK>
__device__ __forceinline__ void sym_run(const SymItem &it, const double *pr, const double *pz, const double *wb,
                                        int64_t N, int lane, const double2 *s_rz, const double2 *s_w,
                                        const double2 *s_wz, const PairCoef &cf, double *o) {
  double r[NI], z[NI], r2[NI], wd[NI], wkr[NI], wkz[NI];
  Acc5 ai[NI];
#pragma unroll
  for (int t = 0; t < NI; t++) {
    sym_load_i(pr, pz, wb, N, (int64_t)(DIAG ? it.b : it.a[t]) * 32 + lane, 1.0e6 + 64.0 * t + lane, r[t], z[t], wd[t],
               wkr[t], wkz[t]);
    r2[t] = r[t] * r[t];
    ai[t] = Acc5{0.0, 0.0, 0.0, 0.0, 0.0};
  }
  constexpr int k0 = DIAG ? 1 : 0, k1 = DIAG ? 17 : 32;
  const int src = (lane + 1) & 31;
  Acc5 aj{0.0, 0.0, 0.0, 0.0, 0.0};
  // diagonal items: steps 1..15 are unmasked, step 16 (lanes >= 16 would double-count) is peeled
  constexpr int kmain = DIAG ? 16 : 32;
#pragma unroll kSymUnroll
  for (int k = k0; k < kmain; k++) {
    const int jj = (lane + k) & 31;
    const double2 rz = s_rz[jj], w = s_w[jj], wz = s_wz[jj];
#pragma unroll
    for (int t = 0; t < NI; t++)
      landau_pair_sym<MASK>(r[t], z[t], r2[t], wd[t], wkr[t], wkz[t], rz.x, rz.y, wz.y, w.x, w.y, wz.x, true, cf,
                                ai[t], aj);
    aj.drr = __shfl_sync(0xffffffffu, aj.drr, src);
    aj.drz = __shfl_sync(0xffffffffu, aj.drz, src);
    aj.dzz = __shfl_sync(0xffffffffu, aj.dzz, src);
    aj.kr = __shfl_sync(0xffffffffu, aj.kr, src);
    aj.kz = __shfl_sync(0xffffffffu, aj.kz, src);
  }
  if constexpr (DIAG) {
    const int jj = (lane + 16) & 31;
    const double2 rz = s_rz[jj], w = s_w[jj], wz = s_wz[jj];
    landau_pair_sym<true>(r[0], z[0], r2[0], wd[0], wkr[0], wkz[0], rz.x, rz.y, wz.y, w.x, w.y, wz.x, lane < 16, cf,
                              ai[0], aj);
    aj.drr = __shfl_sync(0xffffffffu, aj.drr, src);
    aj.drz = __shfl_sync(0xffffffffu, aj.drz, src);
    aj.dzz = __shfl_sync(0xffffffffu, aj.dzz, src);
    aj.kr = __shfl_sync(0xffffffffu, aj.kr, src);
    aj.kz = __shfl_sync(0xffffffffu, aj.kz, src);
  }
#pragma unroll
  for (int t = 0; t < NI; t++) sym_store(o + t * 160, lane, ai[t]);
  // after the last hand-over lane L holds the reverse sums of j = (L + k1) mod 32
  const int jf = (lane + k1) & 31;
  double *oj = o + (DIAG ? 1 : NI) * 160;
  oj[jf] = aj.drr;
  oj[32 + jf] = aj.drz;
  oj[64 + jf] = aj.dzz;
  oj[96 + jf] = aj.kr;
  oj[128 + jf] = aj.kz;
}

template <int MINB, bool MASK>
__global__ void __launch_bounds__(32 * kSymWarps, MINB) inner_sym_kernel(int64_t N, int64_t nitems_b, int64_t nslots,
                                                                         int64_t nitems,
                                                                         const SymItem *__restrict__ items,
                                                                         const double *__restrict__ pr,
                                                                         const double *__restrict__ pz,
                                                                         const double *__restrict__ wT,
                                                                         double *__restrict__ part) {
  __shared__ double2 s_rz[kSymWarps][32], s_w[kSymWarps][32], s_wz[kSymWarps][32];   // (wkz, rb^2)
__shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  stage_pair_coef(s_coef, s_ltab);
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  // persistent warps: grid-stride over the (batch item, work item) list
  for (int64_t item = (int64_t)blockIdx.x * kSymWarps + wid; item < nitems; item += (int64_t)gridDim.x * kSymWarps) {
  const int64_t bb = item / nitems_b;
  const SymItem it = items[item % nitems_b];
  const double *wb = wT + bb * 3 * N;
  __syncwarp();   // the previous item's readers are done with the warp's j-tile buffer
  {
    double r, z, wd, wkr, wkz;
    sym_load_i(pr, pz, wb, N, (int64_t)it.b * 32 + lane, 2.0e6 + lane, r, z, wd, wkr, wkz);
    s_rz[wid][lane] = make_double2(r, z);
    s_w[wid][lane] = make_double2(wd, wkr);
    s_wz[wid][lane] = make_double2(wkz, r * r);
  }
  __syncwarp();
  double *o = part + (bb * nslots + it.slot) * 160;
  switch (it.n) {
    case 0: sym_run<1, true, MASK>(it, pr, pz, wb, N, lane, s_rz[wid], s_w[wid], s_wz[wid], cf, o); break;
    case 1: sym_run<1, false, MASK>(it, pr, pz, wb, N, lane, s_rz[wid], s_w[wid], s_wz[wid], cf, o); break;
    case 2:
      if constexpr (kSymNI >= 2) sym_run<2, false, MASK>(it, pr, pz, wb, N, lane, s_rz[wid], s_w[wid], s_wz[wid], cf, o);
      break;
    default:
      if constexpr (kSymNI >= 3)
        sym_run<kSymNI, false, MASK>(it, pr, pz, wb, N, lane, s_rz[wid], s_w[wid], s_wz[wid], cf, o);
      break;
  }
  }
}

// G[b][c][i] = sum of the partial slots of tile t = i / 32 in the fixed order of tile_slots.
__global__ void reduce_sym_kernel(int64_t N, int64_t nslots, const int32_t *__restrict__ tile_ptr,
                                  const int32_t *__restrict__ tile_slots, const double *__restrict__ part,
                                  double *__restrict__ G, int64_t G_bstride, int nbatch) {
  const int64_t total = (int64_t)nbatch * 5 * N;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / (5 * N), c = (k / N) % 5, i = k % N;
    const int t = (int)(i / 32), lane = (int)(i % 32);
    const double *pb = part + b * nslots * 160 + c * 32 + lane;
    double s = 0.0;
    for (int q = tile_ptr[t]; q < tile_ptr[t + 1]; q++) s += pb[(int64_t)tile_slots[q] * 160];
    G[b * G_bstride + c * N + i] = s;
  }
}

// ------------------------------------------------------------------------------------------------
// N2 (mirror-symmetric): meshes symmetric under v_par -> -v_par (z -> -z; every configuration of
// SURVEY §8(d)) pair each point u of the upper half U (z > 0) with its mirror u' (detected and
// symmetrised at create).  Reflection keeps lambda+-, x, m and every J integral and flips the sign of
// the off-diagonal components:  U(i', j') = F U(i, j) F,  F = diag(1, -1) on (r, z).  So with
//   A(u)  = (wT_D, wT_Kr, wT_Kz)(u),     Bf(u) = F-flipped weights of u' = (wT_D, wT_Kr, -wT_Kz)(u'),
//   G(u) = Ga(u),  G(u') = F Gb(u)      (F on G: negate the rz and K_z components),
// and U(i, j) the same-side tensor, V(i, j) = U(i, j') the cross tensor (source mirrored),
//   Ga(i) = sum_j U(i,j) A(j) + V(i,j) F Bf(j),     Gb(i) = sum_j U(i,j) Bf(j) + V(i,j) F A(j).
// One tensor evaluation serves four ordered interactions (the i <-> j symmetry of the symmetric
// kernel on top): N^2 / 4 evaluations per build instead of N^2 / 2.  The reverse direction of a V
// evaluation is F rev(V(i,j)) F, so V items accumulate it F-flipped (sources R1 = Bf(i), R2 = A(i))
// and flip it when storing.  Items and slots as in inner_sym_kernel over the tiles of U, each item
// once as a U item and once as a V item (it.v); a V diagonal item also pairs every point with its own
// mirror (step 0, forward only).  part = [batch][nslots][2][5][32] (Ga, Gb).
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ void mir_weights(const double *wb, int64_t N, int64_t H, const int32_t *pu,
                                            const int32_t *pm, int64_t u, double A[3], double Bf[3]) {
  if (u < H) {
    const int64_t p = pu[u], q = pm[u];
    A[0] = wb[p];
    A[1] = wb[N + p];
    A[2] = wb[2 * N + p];
    Bf[0] = wb[q];
    Bf[1] = wb[N + q];
    Bf[2] = -wb[2 * N + q];
  } else {
    A[0] = A[1] = A[2] = Bf[0] = Bf[1] = Bf[2] = 0.0;
  }
}

__device__ __forceinline__ void acc_shfl(Acc5 &a, int src) {
  a.drr = __shfl_sync(0xffffffffu, a.drr, src);
  a.drz = __shfl_sync(0xffffffffu, a.drz, src);
  a.dzz = __shfl_sync(0xffffffffu, a.dzz, src);
  a.kr = __shfl_sync(0xffffffffu, a.kr, src);
  a.kz = __shfl_sync(0xffffffffu, a.kz, src);
}

// store 5 x 32 sums at lane position pos; flip = negate the rz and K_z components (F)
__device__ __forceinline__ void mir_store(double *o, int pos, const Acc5 &a, bool flip) {
  const double sg = flip ? -1.0 : 1.0;
  o[pos] = a.drr;
  o[32 + pos] = sg * a.drz;
  o[64 + pos] = a.dzz;
  o[96 + pos] = a.kr;
  o[128 + pos] = sg * a.kz;
}

// ------------------------------------------------------------------------------------------------
// N2 (mirror-symmetric, one CTA per batch item): for batches of small meshes (C4) the whole G of a
// vertex fits in shared memory (Ga, Gb: 80 B per upper-half point), so a persistent CTA owns one
// vertex at a time and accumulates there -- no partial slots in HBM and no reduction kernel.
// Work items are tile pairs (a, b), each evaluating BOTH tensors of every (i in a, j in b): the
// same-side U(i, j) and the cross V(i, j) = U(i, j') -- two independent pair chains per lane that
// share the j-tile staging and the reverse-sum shuffles, with one set of accumulators: forward
// Ga(i) += U A(j) + V F Bf(j), Gb(i) += U Bf(j) + V F A(j); reverse (F-flipped for V, see
// inner_mir_kernel) Ga(j) += rev(U) A(i) + F rev(V) Bf(i), Gb(j) += rev(U) Bf(i) + F rev(V) A(i).
// The host schedules the items in rounds whose tile sets are disjoint (round-robin tournament of
// the tiles, then rounds of diagonal items), so the warps of a CTA add their sums into shared memory
// without atomics and every target's partial sums arrive in a fixed order: bitwise reproducible.
// ------------------------------------------------------------------------------------------------
// One U+V step in sum/difference form.  Every accumulated term has the shape
//   Ga += A U + B (s X),   Gb += B U + A (s X)      (U: same-side tensor, X: cross tensor, s = +-1),
// so with hp = (A + B)/2, hm = (A - B)/2 the pair is carried as P += hp (U + s X), M += hm (U - s X)
// (Ga = P + M, Gb = P - M at the end of the item).  The reverse sums have the same shape with the i
// weights, and the nine (U, X, s) combinations of the 5 + 5 + reverse tensor components reduce to six
// sums/differences (S2 = D5, S3 = D7, ...): 12 DADD + 28 DFMA per step instead of 56 DFMA, and half
// the DFMAs that read three distinct registers (register-file bank reads).
// j-data: (rj, zj, rj^2) and its staged weights hp(j) = (p01.x, p01.y, p2m0.x), hm(j) = (p2m0.y, m12.x,
// m12.y); i weights hpi, hmi.  msk scales both tensors (diagonal-step masks); REV = false: forward only.
template <bool MASK, bool REV, bool UON>
__device__ __forceinline__ void vtx_step(double r, double z, double r2, const double hpi[3], const double hmi[3],
                                         double rj, double zj, double rj2, double2 p01, double2 p2m0, double2 m12,
                                         const PairCoef &cf, double msk, Acc5 &P, Acc5 &M, Acc5 &PJ, Acc5 &MJ) {
  bool oku = true, okv;
  double Udrr = 0.0, Udrz = 0.0, Udzz = 0.0, Ukrr = 0.0, Ukzr = 0.0, Vdrr = 0.0;
  double Xdrr, Xdrz, Xdzz, Xkrr, Xkzr, Ydrr;
  if constexpr (UON) pair_tensors<MASK>(r, z, r2, rj, zj, rj2, cf, oku, Udrr, Udrz, Udzz, Ukrr, Ukzr, Vdrr);
  pair_tensors<MASK>(r, z, r2, rj, -zj, rj2, cf, okv, Xdrr, Xdrz, Xdzz, Xkrr, Xkzr, Ydrr);
  const double mu = (!MASK || oku) ? msk : 0.0, mv = (!MASK || okv) ? msk : 0.0;
  Udrr *= mu; Udrz *= mu; Udzz *= mu; Ukrr *= mu; Ukzr *= mu; Vdrr *= mu;
  Xdrr *= mv; Xdrz *= mv; Xdzz *= mv; Xkrr *= mv; Xkzr *= mv; Ydrr *= mv;
  const double S1 = Udrr + Xdrr, D1 = Udrr - Xdrr;   // (drr, +)
  const double S2 = Udrz + Xdrz, D2 = Udrz - Xdrz;   // (drz, +); (drz, -) = (D2, S2)
  const double S3 = Udzz + Xdzz, D3 = Udzz - Xdzz;   // (dzz, +); (dzz, -) = (D3, S3)
  const double S4 = Ukrr + Xkrr, D4 = Ukrr - Xkrr;   // (krr, +)
  const double S6 = Ukzr + Xkzr, D6 = Ukzr - Xkzr;   // (kzr, +); (kzr, -) = (D6, S6)
  // forward: weights of j
  P.drr = fma(p01.x, S1, P.drr);
  M.drr = fma(p2m0.y, D1, M.drr);
  P.drz = fma(p01.x, S2, P.drz);
  M.drz = fma(p2m0.y, D2, M.drz);
  P.dzz = fma(p01.x, S3, P.dzz);
  M.dzz = fma(p2m0.y, D3, M.dzz);
  P.kr = fma(p01.y, S4, fma(p2m0.x, D2, P.kr));
  M.kr = fma(m12.x, D4, fma(m12.y, S2, M.kr));
  P.kz = fma(p01.y, S6, fma(p2m0.x, D3, P.kz));
  M.kz = fma(m12.x, D6, fma(m12.y, S3, M.kz));
  if constexpr (REV) {   // reverse: weights of i
    const double S8 = Vdrr + Ydrr, D8 = Vdrr - Ydrr;   // (rev drr, +)
    PJ.drr = fma(hpi[0], S8, PJ.drr);
    MJ.drr = fma(hmi[0], D8, MJ.drr);
    PJ.drz = fma(hpi[0], D6, PJ.drz);
    MJ.drz = fma(hmi[0], S6, MJ.drz);
    PJ.dzz = fma(hpi[0], S3, PJ.dzz);
    MJ.dzz = fma(hmi[0], D3, MJ.dzz);
    PJ.kr = fma(hpi[1], S4, fma(hpi[2], S6, PJ.kr));
    MJ.kr = fma(hmi[1], D4, fma(hmi[2], D6, MJ.kr));
    PJ.kz = fma(hpi[1], D2, fma(hpi[2], D3, PJ.kz));
    MJ.kz = fma(hmi[1], S2, fma(hmi[2], S3, MJ.kz));
  }
}

__device__ __forceinline__ void vtx_add(double *sG, int64_t Hp, int64_t pos, const Acc5 &a) {
  sG[pos] += a.drr;
  sG[Hp + pos] += a.drz;
  sG[2 * Hp + pos] += a.dzz;
  sG[3 * Hp + pos] += a.kr;
  sG[4 * Hp + pos] += a.kz;
}

// Ga = P + M into sGa, Gb = P - M into sGb
__device__ __forceinline__ void vtx_add_pm(double *sGa, double *sGb, int64_t Hp, int64_t pos, const Acc5 &P,
                                           const Acc5 &M) {
  vtx_add(sGa, Hp, pos, Acc5{P.drr + M.drr, P.drz + M.drz, P.dzz + M.dzz, P.kr + M.kr, P.kz + M.kz});
  vtx_add(sGb, Hp, pos, Acc5{P.drr - M.drr, P.drz - M.drz, P.dzz - M.dzz, P.kr - M.kr, P.kz - M.kz});
}

// One (a, b) item: lane L's target i = 32 a + L against j = 32 b + (L + k) mod 32, both tensor families;
// returns the forward sums of i (P, M) and the reverse sums of j = 32 b + (L + kend(DIAG)) mod 32
// (PJ, MJ), kend = 17 for the diagonal item and 32 (i.e. L) otherwise.  s_j: the warp's staged j-tile b
// as (r, z), (hp_d, hp_kr), (hp_kz, hm_d), (hm_kr, hm_kz), (r^2, -).
template <bool DIAG, bool MASK, bool RESET_J = true>
__device__ __forceinline__ void vtx_item(int a, const double *rU, const double *zU, const double *wb, int64_t N,
                                         int64_t H, const int32_t *pu, const int32_t *pm, int lane,
                                         const double2 *s_j, const PairCoef &cf, Acc5 &P, Acc5 &M, Acc5 &PJ,
                                         Acc5 &MJ) {
  const int64_t i = (int64_t)a * 32 + lane;
  double Ai[3], Bi[3], hpi[3], hmi[3];
  mir_weights(wb, N, H, pu, pm, i, Ai, Bi);
#pragma unroll
  for (int c = 0; c < 3; c++) {
    hpi[c] = 0.5 * (Ai[c] + Bi[c]);
    hmi[c] = 0.5 * (Ai[c] - Bi[c]);
  }
  const double r = i < H ? rU[i] : 1.0;
  const double z = i < H ? zU[i] : 1.0e6 + lane;   // padding: far away, zero weights
  const double r2 = r * r;
  P = M = Acc5{0.0, 0.0, 0.0, 0.0, 0.0};
  if constexpr (RESET_J) PJ = MJ = Acc5{0.0, 0.0, 0.0, 0.0, 0.0};   // else: the j-tile's sums carry on
  const int src = (lane + 1) & 31;
  if constexpr (DIAG) {   // step 0: each point with its own mirror (V forward only; U is the self pair)
    const double2 rz = s_j[lane * 5], p01 = s_j[lane * 5 + 1], p2m0 = s_j[lane * 5 + 2], m12 = s_j[lane * 5 + 3],
                  rr2 = s_j[lane * 5 + 4];
    vtx_step<MASK, false, false>(r, z, r2, hpi, hmi, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, 1.0, P, M, PJ, MJ);
  }
  constexpr int k0 = DIAG ? 1 : 0, kmain = DIAG ? 16 : 32;
#pragma unroll kMirUnroll
  for (int k = k0; k < kmain; k++) {
    const int jj = (lane + k) & 31;
    const double2 rz = s_j[jj * 5], p01 = s_j[jj * 5 + 1], p2m0 = s_j[jj * 5 + 2], m12 = s_j[jj * 5 + 3],
                  rr2 = s_j[jj * 5 + 4];
    vtx_step<MASK, true, true>(r, z, r2, hpi, hmi, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, 1.0, P, M, PJ, MJ);
    acc_shfl(PJ, src);
    acc_shfl(MJ, src);
  }
  if constexpr (DIAG) {   // step 16: lanes >= 16 would double-count
    const int jj = (lane + 16) & 31;
    const double2 rz = s_j[jj * 5], p01 = s_j[jj * 5 + 1], p2m0 = s_j[jj * 5 + 2], m12 = s_j[jj * 5 + 3],
                  rr2 = s_j[jj * 5 + 4];
    vtx_step<true, true, true>(r, z, r2, hpi, hmi, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, lane < 16 ? 1.0 : 0.0, P,
                               M, PJ, MJ);
    acc_shfl(PJ, src);
    acc_shfl(MJ, src);
  }
}

// stage j-tile b of batch item wb into the warp's buffer (see vtx_item)
__device__ __forceinline__ void vtx_stage_j(int b, const double *rU, const double *zU, const double *wb, int64_t N,
                                            int64_t H, const int32_t *pu, const int32_t *pm, int lane, double2 *d) {
  const int64_t j = (int64_t)b * 32 + lane;
  double A[3], Bf[3];
  mir_weights(wb, N, H, pu, pm, j, A, Bf);
  const double r = j < H ? rU[j] : 1.0;
  const double z = j < H ? zU[j] : 2.0e6 + lane;
  d += lane * 5;   // (r, z), hp = (A + Bf)/2, hm = (A - Bf)/2, (r^2, -)
  d[0] = make_double2(r, z);
  d[1] = make_double2(0.5 * (A[0] + Bf[0]), 0.5 * (A[1] + Bf[1]));
  d[2] = make_double2(0.5 * (A[2] + Bf[2]), 0.5 * (A[0] - Bf[0]));
  d[3] = make_double2(0.5 * (A[1] - Bf[1]), 0.5 * (A[2] - Bf[2]));
  d[4] = make_double2(r * r, 0.0);
}

// N2 (mirror-symmetric, partial-sum slots): the per-vertex kernel's (a, b) U + V items spread over every
// warp of the GPU (batches below one vertex per SM, single large meshes such as C5).  An item is a
// j-tile b with a run of na consecutive i-tiles a0 .. a0+na-1 < b, evaluated one after the other: the
// j-tile is staged once and its reverse sums carry on in registers across the run (after 32 steps
// every lane holds its own j again), so the item writes na forward slots and one reverse slot
// (slot0 .. slot0+na); na = 0 is the diagonal item (b, b) with slots slot0 (forward), slot0+1
// (reverse).  reduce_mir_kernel sums each tile's slots in a fixed host-built order.
// part = [batch][nslots][2][5][32].
__device__ __forceinline__ void mir_store_pm(double *o, int pos, const Acc5 &P, const Acc5 &M) {
  mir_store(o, pos, Acc5{P.drr + M.drr, P.drz + M.drz, P.dzz + M.dzz, P.kr + M.kr, P.kz + M.kz}, false);
  mir_store(o + 160, pos, Acc5{P.drr - M.drr, P.drz - M.drz, P.dzz - M.dzz, P.kr - M.kr, P.kz - M.kz}, false);
}

template <int MINB, bool MASK>
__global__ void __launch_bounds__(32 * kSymWarps, MINB) inner_mir_kernel(int64_t N, int64_t H, int64_t nitems_b,
                                                                         int64_t nslots, int64_t nitems,
                                                                         const int4 *__restrict__ items,
                                                                         const double *__restrict__ rU,
                                                                         const double *__restrict__ zU,
                                                                         const int32_t *__restrict__ pu,
                                                                         const int32_t *__restrict__ pm,
                                                                         const double *__restrict__ wT,
                                                                         double *__restrict__ part) {
  __shared__ double2 s_j[kSymWarps][32 * 5];
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  stage_pair_coef(s_coef, s_ltab);
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int64_t item = (int64_t)blockIdx.x * kSymWarps + wid; item < nitems; item += (int64_t)gridDim.x * kSymWarps) {
    const int64_t bb = item / nitems_b, q = item % nitems_b;
    const int4 it = items[q];   // (a0, na, b, slot0)
    const double *wb = wT + bb * 3 * N;
    __syncwarp();   // the previous item's readers are done with the warp's j-tile buffer
    vtx_stage_j(it.z, rU, zU, wb, N, H, pu, pm, lane, s_j[wid]);
    __syncwarp();
    double *o = part + (bb * nslots + it.w) * 320;
    Acc5 P, M, PJ, MJ;
    if (it.y == 0) {   // the diagonal item (b, b)
      vtx_item<true, MASK>(it.z, rU, zU, wb, N, H, pu, pm, lane, s_j[wid], cf, P, M, PJ, MJ);
      mir_store_pm(o, lane, P, M);
      mir_store_pm(o + 320, (lane + 17) & 31, PJ, MJ);
    } else {
      vtx_item<false, MASK>(it.x, rU, zU, wb, N, H, pu, pm, lane, s_j[wid], cf, P, M, PJ, MJ);
      mir_store_pm(o, lane, P, M);
      for (int t = 1; t < it.y; t++) {
        vtx_item<false, MASK, false>(it.x + t, rU, zU, wb, N, H, pu, pm, lane, s_j[wid], cf, P, M, PJ, MJ);
        mir_store_pm(o + t * 320, lane, P, M);
      }
      mir_store_pm(o + it.y * 320, lane, PJ, MJ);   // after 32 steps per i-tile lane L holds j = 32 b + L
    }
  }
}

#ifndef LANDAU_VTX_WARPS
#define LANDAU_VTX_WARPS 8
#endif
#ifndef LANDAU_VTX_MINB
#define LANDAU_VTX_MINB 1
#endif
constexpr int kVtxWarps = LANDAU_VTX_WARPS, kVtxMinB = LANDAU_VTX_MINB;   // CTA shape, CTAs per SM

struct VtxItem {   // host-built: tiles (a, b) of the upper half; a == b: the diagonal item
  int a, b;
};

// One (a, b) item reading both tiles from the CTA's staged copy of the vertex (s_i: tile a, s_j: tile b,
// 32 points x 5 double2 each, layout of vtx_stage_j); otherwise exactly vtx_item (same steps, same order).
template <bool DIAG, bool MASK>
__device__ __forceinline__ void vtx_item_staged(const double2 *s_i, const double2 *s_j, int lane, const PairCoef &cf,
                                                Acc5 &P, Acc5 &M, Acc5 &PJ, Acc5 &MJ) {
  const double2 irz = s_i[lane * 5], ip01 = s_i[lane * 5 + 1], ip2m0 = s_i[lane * 5 + 2], im12 = s_i[lane * 5 + 3],
                ir2 = s_i[lane * 5 + 4];
  const double hpi[3] = {ip01.x, ip01.y, ip2m0.x}, hmi[3] = {ip2m0.y, im12.x, im12.y};
  const double r = irz.x, z = irz.y, r2 = ir2.x;
  P = M = PJ = MJ = Acc5{0.0, 0.0, 0.0, 0.0, 0.0};
  const int src = (lane + 1) & 31;
  if constexpr (DIAG) {   // step 0: each point with its own mirror (V forward only; U is the self pair)
    vtx_step<MASK, false, false>(r, z, r2, hpi, hmi, irz.x, irz.y, ir2.x, ip01, ip2m0, im12, cf, 1.0, P, M, PJ, MJ);
  }
  constexpr int k0 = DIAG ? 1 : 0, kmain = DIAG ? 16 : 32;
#pragma unroll kMirUnroll
  for (int k = k0; k < kmain; k++) {
    const int jj = (lane + k) & 31;
    const double2 rz = s_j[jj * 5], p01 = s_j[jj * 5 + 1], p2m0 = s_j[jj * 5 + 2], m12 = s_j[jj * 5 + 3],
                  rr2 = s_j[jj * 5 + 4];
    vtx_step<MASK, true, true>(r, z, r2, hpi, hmi, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, 1.0, P, M, PJ, MJ);
    acc_shfl(PJ, src);
    acc_shfl(MJ, src);
  }
  if constexpr (DIAG) {   // step 16: lanes >= 16 would double-count
    const int jj = (lane + 16) & 31;
    const double2 rz = s_j[jj * 5], p01 = s_j[jj * 5 + 1], p2m0 = s_j[jj * 5 + 2], m12 = s_j[jj * 5 + 3],
                  rr2 = s_j[jj * 5 + 4];
    vtx_step<true, true, true>(r, z, r2, hpi, hmi, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, lane < 16 ? 1.0 : 0.0, P,
                               M, PJ, MJ);
    acc_shfl(PJ, src);
    acc_shfl(MJ, src);
  }
}

// Stream-K decomposition over (vertex, round) work.  The batch's rounds form one flattened sequence
// (vertex-major, rounds in schedule order) with weights wp (a full round of pair items: 2, a round of
// diagonal items: 1 -- their durations); round (v, rd) starting at weight g = v Wv + wp[rd] belongs to
// CTA floor(g S / Wtot) of the S persistent CTAs, so every CTA gets a contiguous, equally heavy range
// for any batch size (no partial last wave: 128 vertices on 148 SMs run 14.7 rounds per SM instead of
// 17).  A vertex whose rounds lie in one CTA is summed in shared memory and written once, as before; a
// vertex cut by a CTA boundary is summed per CTA into a partial slot (the CTA's first segment: slot
// (c, 0), its last: (c, 1)), and the last CTA to finish one of its segments (an atomic counter per
// vertex) adds the partials in CTA order -- a fixed order, so every build is bitwise reproducible.
constexpr int kVtxMaxRounds = 64;   // rounds per vertex the per-vertex kernel supports (host-checked)
struct VtxSched {
  int nbatch, nrounds, S;
  int64_t Wv, Wtot;      // weight per vertex, whole batch
};

// wp: the canonical weight prefix [nrounds + 1], or (PERV) the per-vertex prefixes [nbatch][nrounds + 1]
// of host vtx_tables, where a vertex split between CTAs runs its rounds in an order whose boundaries
// meet the cuts
template <bool PERV = false>
__device__ __forceinline__ int vtx_owner(const VtxSched &sc, const int32_t *wp, int64_t v, int rd) {
  return (int)(((v * sc.Wv + wp[(PERV ? v * (sc.nrounds + 1) : 0) + rd]) * (int64_t)sc.S) / sc.Wtot);
}

// first flattened round index f = v * nrounds + rd owned by CTA >= c (nbatch * nrounds if none):
// owner(v, rd) >= c  <=>  v Wv + wp[rd] >= g_c = ceil(c Wtot / S)
__device__ __forceinline__ int64_t vtx_first_round(const VtxSched &sc, const int32_t *wp, int c) {
  const int64_t g = ((int64_t)c * sc.Wtot + sc.S - 1) / sc.S;
  const int64_t v = g / sc.Wv, rem = g - v * sc.Wv;
  int rd = 0;
  while (rd < sc.nrounds && wp[rd] < rem) rd++;
  return v * sc.nrounds + rd;
}

// write a vertex's sums: G(pu) = Ga, G(pm) = F Gb  (F: negate the rz and K_z components); pu, pm in smem
__device__ __forceinline__ void vtx_write_G(double *Gb, const double *sGa, const double *sGb, int64_t N, int64_t H,
                                            int64_t Hp, const int32_t *s_pu, const int32_t *s_pm) {
  for (int64_t k = threadIdx.x; k < 5 * H; k += blockDim.x) {
    const int64_t c = k / H, u = k - c * H;
    Gb[c * N + s_pu[u]] = sGa[c * Hp + u];
    const double v = sGb[c * Hp + u];
    Gb[c * N + s_pm[u]] = (c == 1 || c == 4) ? -v : v;
  }
}

// Dynamic shared memory of inner_vtx_kernel for H upper-half points (Hp = H rounded up to 32): the sums
// Ga, Gb [5][Hp] each, the staged vertex [Hp][5] double2 (geometry once per CTA, weights per vertex)
// and the mirror maps pu, pm [Hp] int32.
__host__ __device__ constexpr size_t vtx_smem_bytes(int64_t Hp) { return (size_t)Hp * (20 * 8 + 2 * 4); }

template <bool MASK, bool PERV>
__global__ void __launch_bounds__(32 * kVtxWarps, kVtxMinB) inner_vtx_kernel(int64_t N, int64_t H, VtxSched sc,
                                                                      const int32_t *__restrict__ round_ptr,
                                                                      const int32_t *__restrict__ wp,
                                                                      const int16_t *__restrict__ ord,
                                                                      const VtxItem *__restrict__ items,
                                                                      const double *__restrict__ rU,
                                                                      const double *__restrict__ zU,
                                                                      const int32_t *__restrict__ pu,
                                                                      const int32_t *__restrict__ pm,
                                                                      const double *__restrict__ wT,
                                                                      double *__restrict__ G, int64_t G_bstride,
                                                                      double *__restrict__ part,
                                                                      int32_t *__restrict__ counters) {
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  __shared__ int s_last;
  __shared__ int16_t s_ord[kVtxMaxRounds];   // the current vertex's round order
  extern __shared__ double s_G[];   // Ga [5][Hp], Gb [5][Hp] | staged vertex [Hp][5] double2 | pu, pm [Hp]
#ifdef LANDAU_VTX_TRACE   // build variant: per-CTA timeline (globaltimer ns) printed at exit (scripts/vtx_trace.py)
  unsigned long long tr_[64];
  int ntr_ = 0;
#define VTX_MARK(tag)                                                                                   \
  if (threadIdx.x == 0 && ntr_ < 64) {                                                                  \
    unsigned long long t_;                                                                              \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                                              \
    tr_[ntr_++] = (t_ << 4) | (tag);                                                                    \
  }
#else
#define VTX_MARK(tag)
#endif
  VTX_MARK(0);
  const int64_t Hp = (H + 31) / 32 * 32;
  double *sGa = s_G, *sGb = s_G + 5 * Hp;
  double2 *s_V = reinterpret_cast<double2 *>(s_G + 10 * Hp);
  int32_t *s_pu = reinterpret_cast<int32_t *>(s_G + 20 * Hp), *s_pm = s_pu + Hp;
  stage_pair_coef(s_coef, s_ltab);
  // the mesh part of the staged vertex (r, z, r^2) and the mirror maps, once per CTA; padding points
  // sit far away (z = 1e6 + 2 L: distinct from each other and from every mirror) with zero weights
  for (int64_t u = threadIdx.x; u < Hp; u += blockDim.x) {
    const bool v = u < H;
    const double r = v ? rU[u] : 1.0, z = v ? zU[u] : 1.0e6 + 2.0 * (double)(u & 31);
    s_V[u * 5] = make_double2(r, z);
    s_V[u * 5 + 4] = make_double2(r * r, 0.0);
    s_pu[u] = v ? pu[u] : 0;
    s_pm[u] = v ? pm[u] : 0;
  }
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int c = blockIdx.x;
  // this CTA's range [f0, f1): the two cut vertices' weight prefixes are read in parallel into shared
  // memory first (a serial scan through global memory costs a dependent L2 miss per round)
  int64_t f0, f1;
  if constexpr (!PERV) {
    f0 = vtx_first_round(sc, wp, c);
    f1 = vtx_first_round(sc, wp, c + 1);
  } else {
    __shared__ int32_t s_w[2][kVtxMaxRounds + 1];
    int64_t vc[2];
    for (int e = 0; e < 2; e++) {
      const int64_t g = ((int64_t)(c + e) * sc.Wtot + sc.S - 1) / sc.S;
      vc[e] = min(g / sc.Wv, (int64_t)sc.nbatch - 1);
      for (int k = threadIdx.x; k <= sc.nrounds; k += blockDim.x) s_w[e][k] = wp[vc[e] * (sc.nrounds + 1) + k];
    }
    __syncthreads();
    int64_t fr[2];
    for (int e = 0; e < 2; e++) {
      const int64_t g = ((int64_t)(c + e) * sc.Wtot + sc.S - 1) / sc.S;
      const int64_t v = g / sc.Wv, rem = g - v * sc.Wv;
      if (v >= sc.nbatch) {
        fr[e] = (int64_t)sc.nbatch * sc.nrounds;
      } else {
        int rd = 0;
        while (rd < sc.nrounds && s_w[e][rd] < rem) rd++;
        fr[e] = v * sc.nrounds + rd;
      }
    }
    f0 = fr[0];
    f1 = fr[1];
  }
  int64_t f = f0;
  VTX_MARK(1);
  while (f < f1) {
    const int64_t v = f / sc.nrounds;
    const int rd0 = (int)(f - v * sc.nrounds);
    const int rd1 = (int)min((int64_t)sc.nrounds, f1 - v * sc.nrounds);   // this CTA's rounds [rd0, rd1) of v
    f = v * sc.nrounds + rd1;
    // stage the vertex's weights: hp = (A + Bf)/2, hm = (A - Bf)/2 with A = wT(u), Bf = F wT(u')
    const double *wb = wT + v * 3 * N;
    for (int64_t u = threadIdx.x; u < Hp; u += blockDim.x) {
      double A[3] = {0.0, 0.0, 0.0}, B[3] = {0.0, 0.0, 0.0};
      if (u < H) {
        const int64_t p = s_pu[u], q = s_pm[u];
        A[0] = wb[p];
        A[1] = wb[N + p];
        A[2] = wb[2 * N + p];
        B[0] = wb[q];
        B[1] = wb[N + q];
        B[2] = -wb[2 * N + q];
      }
      s_V[u * 5 + 1] = make_double2(0.5 * (A[0] + B[0]), 0.5 * (A[1] + B[1]));
      s_V[u * 5 + 2] = make_double2(0.5 * (A[2] + B[2]), 0.5 * (A[0] - B[0]));
      s_V[u * 5 + 3] = make_double2(0.5 * (A[1] - B[1]), 0.5 * (A[2] - B[2]));
    }
    for (int64_t k = threadIdx.x; k < 10 * Hp; k += blockDim.x) s_G[k] = 0.0;
    if constexpr (PERV)
      for (int k = threadIdx.x; k < sc.nrounds; k += blockDim.x) s_ord[k] = ord[v * sc.nrounds + k];
    __syncthreads();
    VTX_MARK(2);
    for (int rp = rd0; rp < rd1; rp++) {
      const int rd = PERV ? (int)s_ord[rp] : rp;   // this vertex's round at position rp
      for (int q = round_ptr[rd] + wid; q < round_ptr[rd + 1]; q += kVtxWarps) {
        const VtxItem it = items[q];
        Acc5 P, M, PJ, MJ;
        if (it.a == it.b)
          vtx_item_staged<true, MASK>(s_V + it.a * 32 * 5, s_V + it.b * 32 * 5, lane, cf, P, M, PJ, MJ);
        else
          vtx_item_staged<false, MASK>(s_V + it.a * 32 * 5, s_V + it.b * 32 * 5, lane, cf, P, M, PJ, MJ);
        vtx_add_pm(sGa, sGb, Hp, (int64_t)it.a * 32 + lane, P, M);
        if (it.a == it.b) __syncwarp();   // forward and reverse sums of a diagonal item hit the same tile
        vtx_add_pm(sGa, sGb, Hp, (int64_t)it.b * 32 + ((lane + (it.a == it.b ? 17 : 32)) & 31), PJ, MJ);
      }
      __syncthreads();   // the next round's tiles may be this round's
    }
    VTX_MARK(3);
    const int cfirst = vtx_owner<PERV>(sc, wp, v, 0), clast = vtx_owner<PERV>(sc, wp, v, sc.nrounds - 1);
    if (cfirst == clast) {   // the whole vertex ran here
      vtx_write_G(G + v * G_bstride, sGa, sGb, N, H, Hp, s_pu, s_pm);
    } else {                 // one segment of a split vertex: partial slot, then the last one combines
      double *slot = part + ((int64_t)c * 2 + (c == cfirst ? 1 : 0)) * 10 * Hp;
      for (int64_t k = threadIdx.x; k < 10 * Hp; k += blockDim.x) slot[k] = s_G[k];
      __threadfence();
      __syncthreads();
      if (threadIdx.x == 0) s_last = atomicAdd(&counters[v], 1) == clast - cfirst;
      __syncthreads();
      if (s_last) {
        __threadfence();
        const double *p0 = part + ((int64_t)cfirst * 2 + 1) * 10 * Hp;
        constexpr int kU = 8;   // independent loads in flight per thread
        for (int64_t k0 = threadIdx.x; k0 < 10 * Hp; k0 += kU * blockDim.x) {   // partials in CTA order
          double acc[kU];
#pragma unroll
          for (int m = 0; m < kU; m++) {
            const int64_t k = k0 + m * blockDim.x;
            acc[m] = k < 10 * Hp ? __ldcg(p0 + k) : 0.0;
          }
          for (int cc = cfirst + 1; cc <= clast; cc++) {
            const double *pc = part + (int64_t)cc * 2 * 10 * Hp;
#pragma unroll
            for (int m = 0; m < kU; m++) {
              const int64_t k = k0 + m * blockDim.x;
              if (k < 10 * Hp) acc[m] += __ldcg(pc + k);
            }
          }
#pragma unroll
          for (int m = 0; m < kU; m++) {
            const int64_t k = k0 + m * blockDim.x;
            if (k < 10 * Hp) s_G[k] = acc[m];
          }
        }
        __syncthreads();
        vtx_write_G(G + v * G_bstride, sGa, sGb, N, H, Hp, s_pu, s_pm);
        if (threadIdx.x == 0) counters[v] = 0;   // ready for the next build
        VTX_MARK(5);
      }
    }
    __syncthreads();   // the write-out reads s_G (and items read s_V) before the next segment rewrites them
    VTX_MARK(4);
  }
#ifdef LANDAU_VTX_TRACE
  if (threadIdx.x == 0) {
    unsigned smid_;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid_));
    for (int i = 0; i < ntr_; i++) printf("VTX %d %d %llu %llu %u\n", c, i, tr_[i] & 15, tr_[i] >> 4, smid_);
  }
#endif
}

// ------------------------------------------------------------------------------------------------
// N2 (mirror-symmetric, directed): single builds and batches too small for the pair kernels.  A warp
// owns 32 upper-half targets u of one batch item and one split of the upper-half sources j, staged 32
// at a time and read by every lane at once (broadcast); each step evaluates U(u, j) and V(u, j) and
// accumulates forward only, in the sum/difference form of vtx_step -- half the tensor evaluations of
// the directed kernel (H^2 U + V pairs instead of N^2 ordered pairs), no shuffles.  The self pair
// (U(u, u)) and any coincident points are masked.  nsplit == 1: G written directly; otherwise
// partials [batch][nsplit][2][5][Hp] for reduce_mdir_kernel.
// ------------------------------------------------------------------------------------------------
constexpr int kMdirWarps = 4;

__global__ void __launch_bounds__(32 * kMdirWarps) inner_mdir_kernel(int64_t N, int64_t H, int64_t wtiles,
                                                                    int64_t split_len, int nsplit, int64_t nitems,
                                                                    const double *__restrict__ rU,
                                                                    const double *__restrict__ zU,
                                                                    const int32_t *__restrict__ pu,
                                                                    const int32_t *__restrict__ pm,
                                                                    const double *__restrict__ wT,
                                                                    double *__restrict__ G, int64_t G_bstride,
                                                                    double *__restrict__ part) {
  __shared__ double2 s_j[kMdirWarps][32 * 5];
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  stage_pair_coef(s_coef, s_ltab);
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t item = (int64_t)blockIdx.x * kMdirWarps + wid;
  if (item >= nitems) return;   // whole warp: no block-level barrier follows
  const int64_t b = item / (nsplit * wtiles), rem = item % (nsplit * wtiles);
  const int sp = (int)(rem / wtiles);
  const int64_t u = (rem % wtiles) * 32 + lane;
  const double *wb = wT + b * 3 * N;
  const double r = u < H ? rU[u] : 1.0;
  const double z = u < H ? zU[u] : 1.0e6 + lane;   // padding: far away, never stored
  const double r2 = r * r;
  const double nohp[3] = {0.0, 0.0, 0.0};
  Acc5 P{0.0, 0.0, 0.0, 0.0, 0.0}, M{0.0, 0.0, 0.0, 0.0, 0.0}, PJ, MJ;
  const int64_t j0 = (int64_t)sp * split_len, j1 = min(H, j0 + split_len);
  double2 *sj = s_j[wid];
  for (int64_t jt = j0; jt < j1; jt += 32) {
    __syncwarp();
    {   // stage sources jt .. jt + 31 (zero weights past j1)
      const int64_t j = jt + lane;
      double A[3], Bf[3];
      mir_weights(wb, N, j1, pu, pm, j, A, Bf);
      const double rj = j < j1 ? rU[j] : 1.0;
      const double zj = j < j1 ? zU[j] : 2.0e6 + lane;
      double2 *d = sj + lane * 5;
      d[0] = make_double2(rj, zj);
      d[1] = make_double2(0.5 * (A[0] + Bf[0]), 0.5 * (A[1] + Bf[1]));
      d[2] = make_double2(0.5 * (A[2] + Bf[2]), 0.5 * (A[0] - Bf[0]));
      d[3] = make_double2(0.5 * (A[1] - Bf[1]), 0.5 * (A[2] - Bf[2]));
      d[4] = make_double2(rj * rj, 0.0);
    }
    __syncwarp();
    const int n = (int)min((int64_t)32, j1 - jt);
    for (int k = 0; k < n; k++) {
      const double2 rz = sj[k * 5], p01 = sj[k * 5 + 1], p2m0 = sj[k * 5 + 2], m12 = sj[k * 5 + 3],
                    rr2 = sj[k * 5 + 4];
      vtx_step<true, false, true>(r, z, r2, nohp, nohp, rz.x, rz.y, rr2.x, p01, p2m0, m12, cf, 1.0, P, M, PJ, MJ);
    }
  }
  if (u >= H) return;
  const Acc5 ga{P.drr + M.drr, P.drz + M.drz, P.dzz + M.dzz, P.kr + M.kr, P.kz + M.kz};
  const Acc5 gb{P.drr - M.drr, P.drz - M.drz, P.dzz - M.dzz, P.kr - M.kr, P.kz - M.kz};
  if (nsplit == 1) {   // G(pu) = Ga, G(pm) = F Gb
    double *Gb = G + b * G_bstride;
    const int64_t p = pu[u], q = pm[u];
    Gb[p] = ga.drr;
    Gb[N + p] = ga.drz;
    Gb[2 * N + p] = ga.dzz;
    Gb[3 * N + p] = ga.kr;
    Gb[4 * N + p] = ga.kz;
    Gb[q] = gb.drr;
    Gb[N + q] = -gb.drz;
    Gb[2 * N + q] = gb.dzz;
    Gb[3 * N + q] = gb.kr;
    Gb[4 * N + q] = -gb.kz;
  } else {
    const int64_t Hp = wtiles * 32;
    double *o = part + ((b * nsplit + sp) * 10) * Hp + u;
    o[0] = ga.drr;
    o[Hp] = ga.drz;
    o[2 * Hp] = ga.dzz;
    o[3 * Hp] = ga.kr;
    o[4 * Hp] = ga.kz;
    o[5 * Hp] = gb.drr;
    o[6 * Hp] = gb.drz;
    o[7 * Hp] = gb.dzz;
    o[8 * Hp] = gb.kr;
    o[9 * Hp] = gb.kz;
  }
}

// G[b][c][pu(u)] = sum over splits of Ga, G[b][c][pm(u)] = F (sum of Gb).  One block per (b, c,
// 32-target tile): warp w sums the splits q = w, w + 8, ... (independent loads in flight), then warp 0
// adds the 8 warp sums in order -- a fixed summation order, so the result is deterministic.
constexpr int kRedWarps = 8;

__global__ void __launch_bounds__(32 * kRedWarps) reduce_mdir_kernel(int64_t N, int64_t H, int64_t Hp, int nsplit,
                                                                   const int32_t *__restrict__ pu,
                                                                   const int32_t *__restrict__ pm,
                                                                   const double *__restrict__ part,
                                                                   double *__restrict__ G, int64_t G_bstride,
                                                                   int nbatch) {
  __shared__ double2 s_w[kRedWarps][32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t T = Hp / 32, nitems = (int64_t)nbatch * 5 * T;
  for (int64_t it = blockIdx.x; it < nitems; it += gridDim.x) {
    const int64_t b = it / (5 * T), c = (it / T) % 5, u = (it % T) * 32 + lane;
    const double *pb = part + b * nsplit * 10 * Hp + c * Hp + u;
    double sa[2] = {0.0, 0.0}, sb[2] = {0.0, 0.0};
    // lanes past H (the ragged last tile) never read: those slots are not written by the inner kernel
    int q = u < H ? wid : nsplit;
    for (; q + kRedWarps < nsplit; q += 2 * kRedWarps) {
      sa[0] += pb[(int64_t)q * 10 * Hp];
      sb[0] += pb[(int64_t)q * 10 * Hp + 5 * Hp];
      sa[1] += pb[(int64_t)(q + kRedWarps) * 10 * Hp];
      sb[1] += pb[(int64_t)(q + kRedWarps) * 10 * Hp + 5 * Hp];
    }
    if (q < nsplit) {
      sa[0] += pb[(int64_t)q * 10 * Hp];
      sb[0] += pb[(int64_t)q * 10 * Hp + 5 * Hp];
    }
    s_w[wid][lane] = make_double2(sa[0] + sa[1], sb[0] + sb[1]);
    __syncthreads();
    if (wid == 0 && u < H) {
      double ta = 0.0, tb = 0.0;
#pragma unroll
      for (int w = 0; w < kRedWarps; w++) {
        ta += s_w[w][lane].x;
        tb += s_w[w][lane].y;
      }
      G[b * G_bstride + c * N + pu[u]] = ta;
      G[b * G_bstride + c * N + pm[u]] = (c == 1 || c == 4) ? -tb : tb;
    }
    __syncthreads();
  }
}

// G[b][c][pu(u)] = sum of the Ga parts, G[b][c][pm(u)] = F (sum of the Gb parts), over the slots of
// u's tile in the fixed order of tile_slots
__global__ void reduce_mir_kernel(int64_t N, int64_t H, int64_t nslots, const int32_t *__restrict__ tile_ptr,
                                  const int32_t *__restrict__ tile_slots, const int32_t *__restrict__ pu,
                                  const int32_t *__restrict__ pm, const double *__restrict__ part,
                                  double *__restrict__ G, int64_t G_bstride, int nbatch) {
  const int64_t total = (int64_t)nbatch * 5 * H;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / (5 * H), c = (k / H) % 5, u = k % H;
    const int t = (int)(u / 32), lane = (int)(u % 32);
    const double *pbk = part + b * nslots * 320 + c * 32 + lane;
    double sa[4] = {0.0, 0.0, 0.0, 0.0}, sb[4] = {0.0, 0.0, 0.0, 0.0};   // 4 independent chains, fixed order
    const int q0 = tile_ptr[t], q1 = tile_ptr[t + 1];
    int q = q0;
    for (; q + 4 <= q1; q += 4)
#pragma unroll
      for (int m = 0; m < 4; m++) {
        const int64_t sl = tile_slots[q + m];
        sa[m] += pbk[sl * 320];
        sb[m] += pbk[sl * 320 + 160];
      }
    for (; q < q1; q++) {
      sa[0] += pbk[(int64_t)tile_slots[q] * 320];
      sb[0] += pbk[(int64_t)tile_slots[q] * 320 + 160];
    }
    const double ta = (sa[0] + sa[1]) + (sa[2] + sa[3]), tb = (sb[0] + sb[1]) + (sb[2] + sb[3]);
    G[b * G_bstride + c * N + pu[u]] = ta;
    G[b * G_bstride + c * N + pm[u]] = (c == 1 || c == 4) ? -tb : tb;
  }
}

// ------------------------------------------------------------------------------------------------
// Tensor cache fill (NEXT-4): every ordered pair (i, j) once, written column-major for the GEMMs:
//   A1 (3N x N): rows c N + i, c = 0,1,2 -> U^D_rr, U^D_rz, U^D_zz
//   A2 (N x 2N): [U^K_rr | U^D_rz],  A3 (N x 2N): [U^K_zr | U^D_zz]
// Coincident points (the diagonal and any twins) get zeros (Amb-3).
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(128) tensor_fill_kernel(int64_t N, const double *__restrict__ pr,
                                                          const double *__restrict__ pz, double *__restrict__ A1,
                                                          double *__restrict__ A2, double *__restrict__ A3) {
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  stage_pair_coef(s_coef, s_ltab);
  __syncthreads();
  PairCoef cf;
  load_pair_coef(s_coef, s_ltab, cf);
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t j = blockIdx.y;
  if (i >= N) return;
  const double r = pr[i], z = pz[i], rb = pr[j], zb = pz[j];
  bool ok;
  double Udrr, Udrz, Udzz, Ukrr, Ukzr, Vdrr;
  pair_tensors<true>(r, z, r * r, rb, zb, rb * rb, cf, ok, Udrr, Udrz, Udzz, Ukrr, Ukzr, Vdrr);
  if (!ok) Udrr = Udrz = Udzz = Ukrr = Ukzr = 0.0;
  A1[i + j * 3 * N] = Udrr;
  A1[N + i + j * 3 * N] = Udrz;
  A1[2 * N + i + j * 3 * N] = Udzz;
  A2[i + j * N] = Ukrr;
  A2[i + (N + j) * N] = Udrz;
  A3[i + j * N] = Ukzr;
  A3[i + (N + j) * N] = Udzz;
}

// N2r: G[b][c][i] = sum_{s = 0..nsplit-1} part[b][s][c][i] in fixed order (deterministic).
__global__ void reduce_kernel(int64_t nt, int nsplit, const double *__restrict__ part, double *__restrict__ G,
                              int64_t G_bstride, int nbatch) {
  const int64_t total = (int64_t)nbatch * 5 * nt;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / (5 * nt), ci = k % (5 * nt);
    const double *p = part + b * (int64_t)nsplit * 5 * nt + ci;
    double s4[4] = {0.0, 0.0, 0.0, 0.0};   // 4 independent chains, fixed order
    int q = 0;
    for (; q + 4 <= nsplit; q += 4)
#pragma unroll
      for (int m = 0; m < 4; m++) s4[m] += p[(int64_t)(q + m) * 5 * nt];
    for (; q < nsplit; q++) s4[0] += p[(int64_t)q * 5 * nt];
    G[b * G_bstride + ci] = (s4[0] + s4[1]) + (s4[2] + s4[3]);
  }
}


}  // namespace landau
