// kernels_band_mma.cuh -- NEXT-2, round 2: the batched band LU as a BLOCKED
// elimination whose trailing updates run on the FP64 tensor cores (mma.sync m8n8k4 f64, DMMA).
// Same factorisation as band_lu2_kernel (PAPER.md:1@24330-26180, §III-G: RCM order, LU without
// pivoting of A = shift M - J per species block), same step-major factor storage, so
// band_solve_kernel consumes either.  (included once, by landau.cu)
//
// Why: band_lu2_kernel applies one or two rank-1 steps per CTA barrier with 32 FMAs per thread between
// barriers; it is bound by the per-step publish -> barrier -> update chain and by issue overhead (22% of
// the FP64 pipe, profiles/r01_band_ncu.txt), not by the ~0.4 ms of FP64 work of a C4 batch.  Here the
// elimination advances 8 columns per panel (right-looking block LU restricted to the band): the panel is
// factored by a few warps, and the rank-8 trailing update of the whole active window is two DMMA per
// 8 x 8 tile -- 256 FMAs per warp instruction instead of 32 -- between two CTA barriers.
//
// Window: the (8 NT)^2 active square (NT = P/8 + 1 tiles per side, P = B + 1 the padded half-bandwidth
// of BandDesc), held as DMMA accumulator fragments (an 8 x 8 tile: lane l holds row l/4, columns
// 2 (l%4) and 2 (l%4) + 1).  Each warp owns whole tile DIAGONALS d = J - I (bm_plan: longest first, to
// the least-loaded warp), so the panel shift (I, J) -> (I - 1, J - 1) keeps every tile with its warp:
// the shift is a register move along each diagonal, whose first tile retires (published before) and
// whose last slot receives the entering indices; every tile index and shared-memory address is a
// compile-time constant of the warp's instantiation.  Per panel p (columns k = 8p .. 8p + 7):
//   A  the owners publish the column tiles (I, 0) and row tiles (0, J); every thread loads its share of
//      the band entries of the group of 8 indices entering at the end of the next panel;  barrier
//   B  warp 0: corner LU (8 x 8, pivots by shuffles), then warps 1-3 L21 = A21 U11^-1 (a row per lane)
//      and warps 4-6 U12 = L11^-1 A12 (a column per lane), written as DMMA fragments of -L21 and U12;
//      warp 7 clears the next entering buffer;  barrier
//   C  every warp: tile -= L21(I) U12(J) by two DMMA (k = 4 each) for I, J >= 1; warp t writes factor
//      row k + t (coalesced); the diagonals shift and their last tiles take the entering indices; the
//      loaded entries of the next group are scattered densely.
// The first NT panels (p < 0) only fill the window.  Indices >= n are padded with a unit diagonal.
#pragma once
#include <cstdint>
#include <type_traits>
#include <utility>

namespace landau {

__device__ __forceinline__ void dmma_8x8x4(double &d0, double &d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};\n"
               : "+d"(d0), "+d"(d1)
               : "d"(a), "d"(b));
}

constexpr int kBmWarps = 8;
constexpr int kBmE = 2;    // entering entries per thread and group of 8 indices (host-checked)
constexpr int kBmTS = 72;  // panel tile stride: 8 rows of 9 (padded: conflict-free row loads in phase B)

// diagonal -> (warp, first accumulator slot): the main diagonal on warp 0; the others longest first to
// the least-loaded of warps 1-7
template <int NT>
struct BmPlan {
  int warp[2 * NT - 1], off[2 * NT - 1], load[kBmWarps];
};
template <int NT>
constexpr BmPlan<NT> bm_plan() {
  BmPlan<NT> pl{};
  for (int w = 0; w < kBmWarps; w++) pl.load[w] = 0;
  pl.warp[NT - 1] = 0;   // the main diagonal alone on warp 0, which also factors the next corner
  pl.off[NT - 1] = 0;
  pl.load[0] = NT;
  for (int a = 1; a < 2 * NT - 1; a++) {
    const int d = (a + 1) / 2 * (a % 2 ? 1 : -1), len = NT - (d < 0 ? -d : d);
    int best = 1;
    for (int w = 2; w < kBmWarps; w++)
      if (pl.load[w] < pl.load[best]) best = w;
    pl.warp[d + NT - 1] = best;
    pl.off[d + NT - 1] = pl.load[best];
    pl.load[best] += len;
  }
  return pl;
}

// f(d, m0) for every diagonal d owned by warp WID (m0: its first accumulator slot), as compile-time
// constants (std::integral_constant), so every accumulator index is static
template <int NT, int WID, int DI, typename F>
__device__ __forceinline__ void bm_call(F &f) {
  constexpr BmPlan<NT> PL = bm_plan<NT>();
  if constexpr (PL.warp[DI] == WID)
    f(std::integral_constant<int, DI - (NT - 1)>{}, std::integral_constant<int, PL.off[DI]>{});
}
template <int NT, int WID, typename F, int... DI>
__device__ __forceinline__ void bm_diags_impl(F &f, std::integer_sequence<int, DI...>) {
  (bm_call<NT, WID, DI>(f), ...);
}
template <int NT, int WID, typename F>
__device__ __forceinline__ void bm_for_diags(F &&f) {
  bm_diags_impl<NT, WID>(f, std::make_integer_sequence<int, 2 * NT - 1>{});
}

// shared memory (doubles): panels [2 parities][2][NT][72], fragments of -L21 and U12 [2][NT][2][32],
// factored corner (64) + pivot reciprocals (8) [2 parities], entering buffers [2 parities][2][8][8 NT]
__host__ __device__ constexpr int band_mma_smem_doubles(int NT) {
  return 4 * NT * kBmTS + 2 * NT * 64 + 2 * 72 + 4 * 8 * 8 * NT + 64;
}

struct BmArgs {
  const double *ae;   // this matrix's entry values
  double *lu;         // this matrix's factor rows
  const int32_t *ent_ptr;
  const uint16_t *ent_pos;
  int n, Bp, P, W, npan;
  double *pan0, *lfr, *ufr, *cor, *ebuf0;
  double *cin;        // the next corner tile handed from warp 0 to the corner warp (fragment order)
  double *bs;         // FWD: the right-hand side in RCM order (shared memory), eliminated in place
  double *yout;       // FWD: L^-1 b (RCM order) for the backward substitution
};

// LU of the 8 x 8 corner held as a DMMA accumulator fragment (lane: row g, columns c0, c0 + 1), in
// place (U on and above the diagonal, L below), pivots shared by shuffles; writes it row-major to cr[64]
// and the pivot reciprocals to cr[64 + t]
__device__ __forceinline__ void bm_corner_lu(double &v0, double &v1, double *cr, int lane) {
  const int g = lane >> 2, c0 = 2 * (lane & 3);
#pragma unroll
  for (int t = 0; t < 8; t++) {
    const double sel = (t & 1) ? v1 : v0;
    const double piv = __shfl_sync(0xffffffffu, sel, 4 * t + (t >> 1));
    const double at = __shfl_sync(0xffffffffu, sel, 4 * g + (t >> 1));
    const double u0 = __shfl_sync(0xffffffffu, v0, 4 * t + (lane & 3));
    const double u1 = __shfl_sync(0xffffffffu, v1, 4 * t + (lane & 3));
    const double rp = rcp_newton(piv);
    if (lane == 0) cr[64 + t] = rp;
    const double l = at * rp;
    const bool below = g > t;
    v0 = below ? (c0 > t ? fma(-l, u0, v0) : (c0 == t ? l : v0)) : v0;
    v1 = below ? (c0 + 1 > t ? fma(-l, u1, v1) : (c0 + 1 == t ? l : v1)) : v1;
  }
  cr[g * 8 + c0] = v0;
  cr[g * 8 + c0 + 1] = v1;
}

// the warp-specialised pieces (accumulator indices static): publish the first tile of each owned
// diagonal (phase A), the rank-8 DMMA update (phase C), the shift + entering tiles (phase C)
template <int NT, int WID, int TPW>
__device__ __forceinline__ void bm_publish(double (&acc)[TPW][2], double *colp, double *rowp, int g, int c0) {
  bm_for_diags<NT, WID>([&](auto dc, auto mc) {
    constexpr int d = decltype(dc)::value, m0 = decltype(mc)::value;
    if constexpr (d != 0) {   // (the corner was factored ahead, in the previous panel's phase C)
      double *t = d > 0 ? rowp + d * kBmTS : colp + (-d) * kBmTS;
      t[g * 9 + c0] = acc[m0][0];
      t[g * 9 + c0 + 1] = acc[m0][1];
    }
  });
}
template <int NT, int WID, int TPW>
__device__ __forceinline__ void bm_update(double (&acc)[TPW][2], const double *lfr, const double *ufr, int lane,
                                          double *cnext, double *cin) {
  bm_for_diags<NT, WID>([&](auto dc, auto mc) {
    constexpr int d = decltype(dc)::value, m0 = decltype(mc)::value;
    constexpr int len = NT - (d < 0 ? -d : d), I0 = d < 0 ? -d : 0, J0 = d > 0 ? d : 0;
    constexpr int i0 = d == 0 ? 2 : 1;
    if constexpr (d == 0) {   // look-ahead: update tile (1, 1) first and factor it -- the next corner
      dmma_8x8x4(acc[m0 + 1][0], acc[m0 + 1][1], lfr[64 + lane], ufr[64 + lane]);
      dmma_8x8x4(acc[m0 + 1][0], acc[m0 + 1][1], lfr[96 + lane], ufr[96 + lane]);
      if (cnext) {   // hand the updated tile to the corner warp, which factors it (bm_corner_warp)
        cin[2 * lane] = acc[m0 + 1][0];
        cin[2 * lane + 1] = acc[m0 + 1][1];
        __threadfence_block();
        asm volatile("bar.arrive 2, 64;" ::: "memory");
      }
    }
#pragma unroll
    for (int i = i0; i < len; i++) {
      const double *fa = lfr + (I0 + i) * 64, *fb = ufr + (J0 + i) * 64;
      dmma_8x8x4(acc[m0 + i][0], acc[m0 + i][1], fa[lane], fb[lane]);
      dmma_8x8x4(acc[m0 + i][0], acc[m0 + i][1], fa[32 + lane], fb[32 + lane]);
    }
  });
}
template <int NT, int WID, int TPW>
__device__ __forceinline__ void bm_shift(double (&acc)[TPW][2], const double *er, int g, int c0, int k1, int n) {
  constexpr int Q = 8 * NT;
  bm_for_diags<NT, WID>([&](auto dc, auto mc) {
    constexpr int d = decltype(dc)::value, m0 = decltype(mc)::value;
    constexpr int len = NT - (d < 0 ? -d : d);
    constexpr int I1 = (len - 1) + (d < 0 ? -d : 0), J1 = (len - 1) + (d > 0 ? d : 0);
#pragma unroll
    for (int i = 0; i + 1 < len; i++) {
      acc[m0 + i][0] = acc[m0 + i + 1][0];
      acc[m0 + i][1] = acc[m0 + i + 1][1];
    }
    const int row = 8 * I1 + g;
#pragma unroll
    for (int e = 0; e < 2; e++) {
      const int c = c0 + e, col = 8 * J1 + c;
      double v;
      if (I1 == NT - 1 && (J1 < NT - 1 || c <= g)) v = er[g * Q + col];
      else v = er[8 * Q + c * Q + row];
      if (d == 0 && row == col && k1 + row >= n) v = 1.0;   // padding index: unit diagonal
      acc[m0 + len - 1][e] = v;
    }
  });
}
#define BM_SWITCH(CALL)              \
  switch (warp) {                    \
    case 0: CALL(0); break;          \
    case 1: CALL(1); break;          \
    case 2: CALL(2); break;          \
    case 3: CALL(3); break;          \
    case 4: CALL(4); break;          \
    case 5: CALL(5); break;          \
    case 6: CALL(6); break;          \
    default: CALL(7); break;         \
  }

template <int NT, bool FWD>
__device__ __forceinline__ void bm_body(const BmArgs &A) {
  constexpr BmPlan<NT> PL = bm_plan<NT>();
  constexpr int Q = 8 * NT;
  constexpr int TPW = [] {
    int m = 1;
    for (int w = 0; w < kBmWarps; w++) m = PL.load[w] > m ? PL.load[w] : m;
    return m;
  }();
  const int lane = threadIdx.x & 31, tid = threadIdx.x, warp = tid >> 5;
  const int g = lane >> 2, c0 = 2 * (lane & 3);
  const int n = A.n, Bp = A.Bp, P = A.P, W = A.W;
  double acc[TPW][2];
#pragma unroll
  for (int m = 0; m < TPW; m++) acc[m][0] = acc[m][1] = 0.0;
  // the entries of group G held by this thread: entries e0 + tid + 256 m (m < kBmE)
  double ev[kBmE];
  int ep[kBmE];
  auto load_group = [&](int G) {
#pragma unroll
    for (int m = 0; m < kBmE; m++) {
      ep[m] = -1;
      ev[m] = 0.0;
    }
    if (G >= 0 && G < A.npan) {
      const int e0 = A.ent_ptr[8 * G], e1 = A.ent_ptr[min(8 * G + 8, n)];
#pragma unroll
      for (int m = 0; m < kBmE; m++) {
        const int e = e0 + tid + 32 * kBmWarps * m;
        if (e < e1) {
          ep[m] = A.ent_pos[e];
          ev[m] = A.ae[e];
        }
      }
    }
  };
  // ep / (4P) by a multiply: ep < 32 P <= 4096, so the rounding error ep / 2^24 stays below 1 / (4P)
  const unsigned qmul = (1u << 24) / (unsigned)(4 * P) + 1u;
  auto scatter_group = [&](double *er) {   // dense rows er[q][col] (row parts), er[8 Q + q][row] (column parts)
#pragma unroll
    for (int m = 0; m < kBmE; m++)
      if (ep[m] >= 0) {
        const int q = (int)(((unsigned)ep[m] * qmul) >> 24), s = ep[m] - q * 4 * P;   // q = ep / 4P
        if (s < P) er[q * Q + q + 1 + s] = ev[m];                  // A(i, j), j = i - Bp + s: window column q + 1 + s
        else er[8 * Q + q * Q + q + s - 2 * P + 1] = ev[m];        // A(j, i), j = i + s - 3P + 1: window row q + s - 2P + 1
      }
  };
  // prologue: group 0 (entering at panel -NT) into the buffer of parity (-NT) & 1
  {
    double *er = A.ebuf0 + ((-NT) & 1) * 2 * 8 * Q;
    for (int i = tid; i < 2 * 8 * Q; i += 32 * kBmWarps) er[i] = 0.0;
    load_group(0);
    asm volatile("bar.sync 0, %0;" ::"n"(32 * kBmWarps) : "memory");
    scatter_group(er);
    asm volatile("bar.sync 0, %0;" ::"n"(32 * kBmWarps) : "memory");
  }
#ifdef LANDAU_BM_TRACE   // build variant: clock64 per phase, printed by lane 0 of every warp of CTA 0
  long long tph[6] = {0, 0, 0, 0, 0, 0}, t_ = clock64();
#define BM_T(i) { const long long t2_ = clock64(); tph[i] += t2_ - t_; t_ = t2_; }
#else
#define BM_T(i)
#endif
  for (int p = -NT; p < A.npan; p++) {
    const int par = p & 1;
    double *colp = A.pan0 + par * 2 * NT * kBmTS;   // tiles (I, 0): element (r, c) at I*72 + r*9 + c
    double *rowp = colp + NT * kBmTS;               // tiles (0, J)
    double *er = A.ebuf0 + par * 2 * 8 * Q;         // this panel's entering group (p + NT)
    double *er1 = A.ebuf0 + (par ^ 1) * 2 * 8 * Q;  // the next panel's (p + 1 + NT), scattered in phase C
    const int k = 8 * p;
    // ---- A: publish the first tile of every diagonal; load the next entering group's entries
    if (p >= 0) {
#define BM_PUB(w) bm_publish<NT, w, TPW>(acc, colp, rowp, g, c0)
      BM_SWITCH(BM_PUB)
#undef BM_PUB
    }
    load_group(p + 1 + NT);
    BM_T(0)
    asm volatile("bar.sync 0, %0;" ::"n"(32 * kBmWarps) : "memory");
    BM_T(1)
    // ---- B: L21 and U12 from the corner factored ahead (warps 1-6); warps 0 and 7 clear the next
    // entering buffer
    double *cor = A.cor + par * 72;
    if (warp == 0 || warp == 7) {
      for (int i = (warp ? 32 : 0) + lane; i < 2 * 8 * Q; i += 64) er1[i] = 0.0;
      if (FWD && warp == 0 && lane == 0 && p >= 0) {   // forward elimination of the panel's rows: y = L11^-1 b
        double y[8];
#pragma unroll
        for (int t = 0; t < 8; t++) {
          double v = k + t < n ? A.bs[k + t] : 0.0;
#pragma unroll
          for (int s2 = 0; s2 < t; s2++) v = fma(-cor[t * 8 + s2], y[s2], v);
          y[t] = v;
          if (k + t < n) {
            A.bs[k + t] = v;
            A.yout[k + t] = v;
          }
        }
      }
    } else if (p >= 0) {
      {
        if (warp <= 3) {   // L21 = A21 U11^-1: window row r = 8 + (tid - 32)
          const int r = 8 + tid - 32;
          if (r < Q) {
            double *row = colp + (r >> 3) * kBmTS + (r & 7) * 9;
            double x[8];
#pragma unroll
            for (int c = 0; c < 8; c++) x[c] = row[c];
#pragma unroll
            for (int t = 0; t < 8; t++) {
              x[t] *= cor[64 + t];
#pragma unroll
              for (int c = t + 1; c < 8; c++) x[c] = fma(-x[t], cor[t * 8 + c], x[c]);
            }
            double *fa = A.lfr + (r >> 3) * 64 + 4 * (r & 7);
#pragma unroll
            for (int c = 0; c < 8; c++) {
              row[c] = x[c];
              fa[(c >> 2) * 32 + (c & 3)] = -x[c];
            }
          }
        } else {          // U12 = L11^-1 A12: window column cc = 8 + (tid - 128)
          const int cc = 8 + tid - 128;
          if (cc < Q) {
            double *col = rowp + (cc >> 3) * kBmTS + (cc & 7);
            double y[8];
#pragma unroll
            for (int t = 0; t < 8; t++) y[t] = col[t * 9];
#pragma unroll
            for (int t = 0; t < 8; t++)
#pragma unroll
              for (int r = t + 1; r < 8; r++) y[r] = fma(-cor[r * 8 + t], y[t], y[r]);
            double *fb = A.ufr + (cc >> 3) * 64 + 4 * (cc & 7);
#pragma unroll
            for (int t = 0; t < 8; t++) {
              col[t * 9] = y[t];
              fb[(t >> 2) * 32 + (t & 3)] = y[t];
            }
          }
        }
      }
    }
    BM_T(2)
    asm volatile("bar.sync 0, %0;" ::"n"(32 * kBmWarps) : "memory");
    BM_T(3)
    // ---- C: rank-8 trailing update of the tiles with I, J >= 1 (all but the first of each diagonal)
    if (p >= 0) {
    double *cnext = p + 1 < A.npan ? A.cor + (par ^ 1) * 72 : nullptr;
#define BM_UPD(w) bm_update<NT, w, TPW>(acc, A.lfr, A.ufr, lane, cnext, A.cin)
      BM_SWITCH(BM_UPD)
#undef BM_UPD
      if (cnext && warp == kBmWarps - 1) {   // the corner warp (one of the lightest): next panel's corner LU
        asm volatile("bar.sync 2, 64;" ::: "memory");
        double v0 = A.cin[2 * lane], v1 = A.cin[2 * lane + 1];
        bm_corner_lu(v0, v1, cnext, lane);
      }
      if (FWD && warp >= 1 && warp <= 3) {   // b(rows below the panel) -= L21 y
        const int r = 8 + tid - 32;
        if (r < Q && k + r < n) {
          const double *row = colp + (r >> 3) * kBmTS + (r & 7) * 9;
          double v = A.bs[k + r];
#pragma unroll
          for (int c = 0; c < 8; c++) v = fma(-row[c], k + c < n ? A.bs[k + c] : 0.0, v);
          A.bs[k + r] = v;
        }
      }
      // factor row k + warp: (U(t, t), U(t, t+1 .. t+Bp), L(t+1 .. t+Bp, t)) in window coordinates; with
      // FWD the L part is not needed (the forward elimination is done) and not written
      const int t = warp;
      if (k + t < n) {
        double *out = A.lu + (int64_t)(k + t) * W;
        for (int s = lane; s < (FWD ? Bp + 1 : W); s += 32) {
          double v;
          if (s == 0) {
            v = cor[t * 9];
          } else if (s <= Bp) {
            const int c = t + s;
            v = c < 8 ? cor[t * 8 + c] : rowp[(c >> 3) * kBmTS + t * 9 + (c & 7)];
          } else {
            const int r = t + s - Bp;
            v = r < 8 ? cor[r * 8 + t] : colp[(r >> 3) * kBmTS + (r & 7) * 9 + t];
          }
          out[s] = v;
        }
      }
    }
    // shift every diagonal; its last slot takes the entering indices k + 8 NT + q, logical (window of
    // panel p + 1) row / column 8 (NT - 1) + q
    const int k1 = k + 8;
#define BM_SH(w) bm_shift<NT, w, TPW>(acc, er, g, c0, k1, n)
    BM_SWITCH(BM_SH)
#undef BM_SH
    if (p == -1 && warp == 0) bm_corner_lu(acc[0][0], acc[0][1], A.cor, lane);   // the first corner
    BM_T(4)
    scatter_group(er1);
    BM_T(5)
  }
#ifdef LANDAU_BM_TRACE
  if (blockIdx.x == 0 && lane == 0)
    printf("BM warp %d A %lld barA %lld B %lld barB %lld C %lld scatter %lld\n", warp, tph[0], tph[1], tph[2], tph[3], tph[4], tph[5]);
#endif
}

// FWD (the implicit step): also eliminate the right-hand side rhs [batch][ndof] (species blocks at
// vec_off, original order; perm maps RCM -> original) and write y = L^-1 b (RCM order) to yout in the
// same layout; only the U part of the factor rows is written, for band_solve_kernel's backward pass
template <int NT, bool FWD>
__global__ void __launch_bounds__(32 * kBmWarps, NT <= 12 ? 2 : 1) band_lu_mma_kernel(const double *__restrict__ Aent,
                                                                                  int64_t ent_bstride,
                                                                                  double *__restrict__ LU,
                                                                                  int64_t lu_bstride,
                                                                                  const BandDesc *__restrict__ desc,
                                                                                  int nsp, const double *__restrict__ rhs,
                                                                                  double *__restrict__ yout,
                                                                                  const int32_t *__restrict__ perm_all,
                                                                                  const int64_t *__restrict__ perm_off,
                                                                                  const int64_t *__restrict__ vec_off,
                                                                                  int64_t ndof) {
  extern __shared__ double smem[];
  const int bi = blockIdx.x / nsp, sp = blockIdx.x % nsp;
  const BandDesc d = desc[sp];
  BmArgs A;
  A.ae = Aent + (int64_t)bi * ent_bstride + d.aoff;
  A.lu = LU + (int64_t)bi * lu_bstride + d.off;
  A.ent_ptr = d.ent_ptr;
  A.ent_pos = d.ent_pos;
  A.n = d.n;
  A.Bp = d.B;
  A.P = d.B + 1;   // host-checked: P == 8 (NT - 1)
  A.W = 2 * d.B + 1;
  A.npan = (d.n + 7) / 8;
  A.pan0 = smem;
  A.lfr = A.pan0 + 4 * NT * kBmTS;
  A.ufr = A.lfr + NT * 64;
  A.cor = A.ufr + NT * 64;
  A.ebuf0 = A.cor + 2 * 72;
  A.cin = A.ebuf0 + 4 * 8 * 8 * NT;
  A.bs = A.cin + 64;
  A.yout = nullptr;
  if (FWD) {
    const int32_t *perm = perm_all + perm_off[sp];
    const double *bb = rhs + (int64_t)bi * ndof + vec_off[sp];
    for (int i = threadIdx.x; i < d.n; i += blockDim.x) A.bs[i] = bb[perm[i]];
    A.yout = yout + (int64_t)bi * ndof + vec_off[sp];
    // (bm_body's prologue barrier orders these loads before the first use)
  }
  bm_body<NT, FWD>(A);
}

}  // namespace landau
