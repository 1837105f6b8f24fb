// kernels_fe.cuh -- finite-element kernels: point fields (a-1), element matrices (a-4), deterministic gather assembly (a-3 + a-5), mass (a-6)
// (split out of landau.cu; included once, by landau.cu)
#pragma once
#include <cstdint>

#include "kernels.cuh"

namespace landau {


// Per-handle data reaches the kernels as arguments (species table by value, basis tables through
// global memory) -- no per-handle __constant__ state, so several handles can share a device and a
// captured CUDA graph stays valid.

// ------------------------------------------------------------------------------------------------
// Reference tables in shared memory: thread-varying indices into __constant__ memory serialise, so
// kernels that index the tables by thread copy them to shared memory once per block.
// ------------------------------------------------------------------------------------------------
template <int NB>
__device__ __forceinline__ void load_tables(const double *__restrict__ tab, double (*s_phi)[NB], double (*s_dxi)[NB],
                                            double (*s_deta)[NB]) {
  for (int i = threadIdx.x; i < NB * NB; i += blockDim.x) {
    s_phi[i / NB][i % NB] = tab[i];
    s_dxi[i / NB][i % NB] = tab[NB * NB + i];
    s_deta[i / NB][i % NB] = tab[2 * NB * NB + i];
  }
}

// ------------------------------------------------------------------------------------------------
// N1: point fields.  A block handles EPB cells at a time (grid-stride over cells x batch); thread
// (cell, a) first forms the combined element coefficients gD_a = sum_b e_b^2 f_b,a and
// gK_a = sum_b e_b^2/m_b f_b,a through the extraction list (T_D, T_K are linear in f), then thread
// (cell, q) interpolates: w T_D, w T_Kr, w T_Kz at its point.
// ------------------------------------------------------------------------------------------------
template <int NB, int EPB>
__global__ void __launch_bounds__(NB * EPB) field_kernel(int64_t ncell, int nbatch, int64_t ndof_total,
                                                         const double *__restrict__ f,
                                                         const int32_t *__restrict__ ext_ptr,
                                                         const int32_t *__restrict__ ext_dof,
                                                         const double *__restrict__ ext_w,
                                                         const int *__restrict__ cell_grid,
                                                         const double *__restrict__ cell_h, const double *__restrict__ pw,
                                                         const double *__restrict__ tab, const SpeciesConst sp_,
                                                         double *__restrict__ wT, int64_t npts) {
  // tables transposed ([k][q]): in phase 2 consecutive threads are consecutive q (conflict-free)
  __shared__ double s_phi[NB][NB], s_dxi[NB][NB], s_deta[NB][NB];
  __shared__ double gD[EPB][NB], gK[EPB][NB];
  for (int i = threadIdx.x; i < NB * NB; i += blockDim.x) {
    s_phi[i % NB][i / NB] = tab[i];
    s_dxi[i % NB][i / NB] = tab[NB * NB + i];
    s_deta[i % NB][i / NB] = tab[2 * NB * NB + i];
  }
  const SpeciesConst &c_sp = sp_;
  const int el = threadIdx.x / NB, a = threadIdx.x % NB;
  // a block keeps one chunk of EPB cells and walks the batch items b = g, g + G, ... (blockIdx.x =
  // g * nchunks + chunk), so the cell's extraction entries, grid, size and weights are loaded once
  constexpr int kExt = 8;   // extraction entries cached in registers per node (more: read from memory)
  const int64_t nchunks = (ncell + EPB - 1) / EPB;
  const int64_t chunk = blockIdx.x % nchunks, G = gridDim.x / nchunks;
  const int64_t e = chunk * EPB + el;
  const bool live = e < ncell && (int64_t)blockIdx.x < G * nchunks;
  int g = 0, nk = 0;
  int32_t k0 = 0;
  int32_t xd[kExt];
  double xw[kExt], w = 0.0, ws = 0.0;
  if (live) {
    g = cell_grid[e];
    k0 = ext_ptr[e * NB + a];
    nk = ext_ptr[e * NB + a + 1] - k0;
#pragma unroll
    for (int k = 0; k < kExt; k++) {
      xd[k] = k < nk ? ext_dof[k0 + k] : 0;
      xw[k] = k < nk ? ext_w[k0 + k] : 0.0;
    }
    w = pw[e * NB + a];
    ws = w * (2.0 / cell_h[e]);
  }
  for (int64_t b = blockIdx.x / nchunks; b < nbatch; b += G) {
    const double *fb = f + b * ndof_total;
    __syncthreads();
    if (live) {
      double sD = 0.0, sK = 0.0;
      for (int s = 0; s < c_sp.grid_nsp[g]; s++) {
        const int sp = c_sp.grid_sp[g][s];
        const double *fs = fb + c_sp.soff[sp];
        double v = 0.0;
#pragma unroll
        for (int k = 0; k < kExt; k++)
          if (k < nk) v = fma(xw[k], __ldg(fs + xd[k]), v);
        for (int k = kExt; k < nk; k++) v = fma(ext_w[k0 + k], __ldg(fs + ext_dof[k0 + k]), v);
        sD = fma(c_sp.e2[sp], v, sD);
        sK = fma(c_sp.e2m[sp], v, sK);
      }
      gD[el][a] = sD;
      gK[el][a] = sK;
    }
    __syncthreads();
    if (live) {
      const int q = a;   // NQP == NB for (p+1)^2 Gauss points
      const int64_t pt = e * NB + q;
      double td = 0.0, tr = 0.0, tz = 0.0;
#pragma unroll
      for (int k = 0; k < NB; k++) {
        td = fma(s_phi[k][q], gD[el][k], td);
        tr = fma(s_dxi[k][q], gK[el][k], tr);
        tz = fma(s_deta[k][q], gK[el][k], tz);
      }
      double *o = wT + b * 3 * npts;
      o[pt] = w * td;
      o[npts + pt] = ws * tr;
      o[2 * npts + pt] = ws * tz;
    }
  }
}

// ------------------------------------------------------------------------------------------------
// N3: element matrices (species independent).  C^D[k,l] = (2/h)^2 sum_q gk . (w_q G_D(q)) . gl,
// C^K[k,l] = (2/h) sum_q (gk . w_q G_K(q)) phi_l(q), gk the reference gradients.  A thread owns an
// S x S block (S = p + 1) of both matrices of one cell, so each table value it loads from shared
// memory feeds S outputs (the v0 one-entry-per-thread form was shared-memory-bandwidth bound);
// a block handles EPB cells.  Per q:  u_l = A_rr gl_r + A_rz gl_z,  v_l = A_rz gl_r + A_zz gl_z,
// t_k = gk_r K_r + gk_z K_z;  C^D[k,l] += gk_r u_l + gk_z v_l,  C^K[k,l] += t_k phi_l.
// G is read in the chunked layout G[((i / Nc) * nbatch + b) * 5 + c][i % Nc] (Nc = N unless split).
// ------------------------------------------------------------------------------------------------
#ifndef LANDAU_EL_MINB
#define LANDAU_EL_MINB 1
#endif
template <int NB, int S, int EPB>
__global__ void __launch_bounds__(NB * EPB, LANDAU_EL_MINB) element_kernel(int64_t ncell, const double *__restrict__ G, int64_t Nc,
                                                             int nbatch, int b0, int nb, const double *__restrict__ pw,
                                                             const double *__restrict__ cell_h,
                                                             const double *__restrict__ tab, double *__restrict__ Cbuf) {
  static_assert(S * S == NB, "S = p + 1");
  __shared__ double s_phi[NB][NB], s_dxi[NB][NB], s_deta[NB][NB];   // [q][k]
  __shared__ double sA[EPB][5][NB];                                  // w_q G(q) per cell
  load_tables<NB>(tab, s_phi, s_dxi, s_deta);
  const int el = threadIdx.x / NB, t = threadIdx.x % NB;
  const int k0 = (t / S) * S, l0 = (t % S) * S;
  const int64_t nchunks = (ncell + EPB - 1) / EPB;
  for (int64_t it = blockIdx.x; it < nchunks * nb; it += gridDim.x) {   // batch items b0 .. b0 + nb - 1
    const int bc = (int)(it / nchunks), b = b0 + bc;
    const int64_t e = (it % nchunks) * EPB + el;
    __syncthreads();
    if (e < ncell) {
      const int64_t i = e * NB + t;
      const int64_t chunk = i / Nc, off = i % Nc;
      const double *Gb = G + ((chunk * nbatch + b) * 5) * Nc + off;
      const double w = pw[i];
#pragma unroll
      for (int c = 0; c < 5; c++) sA[el][c][t] = w * Gb[c * Nc];
    }
    __syncthreads();
    if (e >= ncell) continue;
    double cd[S][S], ck[S][S];
#pragma unroll
    for (int a = 0; a < S; a++)
#pragma unroll
      for (int c = 0; c < S; c++) cd[a][c] = ck[a][c] = 0.0;
#pragma unroll 2
    for (int q = 0; q < NB; q++) {
      const double Arr = sA[el][0][q], Arz = sA[el][1][q], Azz = sA[el][2][q], Kr = sA[el][3][q], Kz = sA[el][4][q];
      double u[S], v[S], pl[S], gr[S], gz[S], tk[S];
#pragma unroll
      for (int c = 0; c < S; c++) {
        const double glr = s_dxi[q][l0 + c], glz = s_deta[q][l0 + c];
        u[c] = fma(Arr, glr, Arz * glz);
        v[c] = fma(Arz, glr, Azz * glz);
        pl[c] = s_phi[q][l0 + c];
        gr[c] = s_dxi[q][k0 + c];
        gz[c] = s_deta[q][k0 + c];
        tk[c] = fma(gr[c], Kr, gz[c] * Kz);
      }
#pragma unroll
      for (int a = 0; a < S; a++)
#pragma unroll
        for (int c = 0; c < S; c++) {
          cd[a][c] = fma(gr[a], u[c], fma(gz[a], v[c], cd[a][c]));
          ck[a][c] = fma(tk[a], pl[c], ck[a][c]);
        }
    }
    const double sc = 2.0 / cell_h[e];
    double *o = Cbuf + ((int64_t)bc * ncell + e) * 2 * NB * NB;
#pragma unroll
    for (int a = 0; a < S; a++)
#pragma unroll
      for (int c = 0; c < S; c++) {
        reinterpret_cast<double2 *>(o)[(k0 + a) * NB + l0 + c] = make_double2(cd[a][c] * sc * sc, ck[a][c] * sc);
      }
  }
}

// N3 by sum factorisation.  Basis and Gauss points are tensor products (node n = b S + a, point
// q = qz S + qr, a / qr along r), so with 1-D factors L[i][a] = l_a(x_i), D[i][a] = l'_a(x_i) and
// the pair products P_LL[i] = L[i][x] L[i][y], P_LD = L[i][x] D[i][y], P_DL = D[i][x] L[i][y],
// P_DD = D[i][x] D[i][y] of a lane's index pair (x, y):
//   step 1 (z): T_t[(b,d)][qr] = sum_qz P_t(b,d)[qz] A_t(qz, qr) for
//               (t, P, A) = (1, LL, Arr) (2, LD, Arz) (3, DL, Arz) (4, DD, Azz) (5, LL, Kr) (6, DL, Kz)
//   step 2 (r): C^D[(b,a),(d,c)] = sum_qr P_DD(a,c) T1 + P_DL(a,c) T2 + P_LD(a,c) T3 + P_LL(a,c) T4,
//               C^K[(b,a),(d,c)] = sum_qr P_DL(a,c) T5 + P_LL(a,c) T6
// (the rr, rz, zr, zz terms of gk . A . gl and the r, z terms of (gk . K) phi_l), 6 S^4 + 6 S^5
// multiply-adds per cell instead of ~4.5 S^6 for the direct sum.  A warp owns one cell: lane L
// holds the pair (x, y) = (L % S^2) / S, (L % S^2) % S and its 4 S products for both steps (the
// same pair plays (b, d) in step 1 and (a, c) in step 2); the 32 / S^2 lane groups split qr (step 1)
// and (b, d) (step 2).
// ------------------------------------------------------------------------------------------------
#ifndef LANDAU_SF_WARPS
#define LANDAU_SF_WARPS 4
#endif
constexpr int kSfWarps = LANDAU_SF_WARPS;

// per-lane products of the 1-D factors for the lane's index pair (x, y)
template <int S>
__device__ __forceinline__ void sf_tables(const double *tab1, int lane, double PLL[S], double PLD[S], double PDL[S],
                                          double PDD[S]) {
  constexpr int NB = S * S;
  const int xy = lane % NB, x = xy / S, y = xy % S;
#pragma unroll
  for (int i = 0; i < S; i++) {
    const double Lx = tab1[i * S + x], Ly = tab1[i * S + y], Dx = tab1[NB + i * S + x], Dy = tab1[NB + i * S + y];
    PLL[i] = Lx * Ly;
    PLD[i] = Lx * Dy;
    PDL[i] = Dx * Ly;
    PDD[i] = Dx * Dy;
  }
}

// one cell's C^D, C^K (both sum-factorised contractions) from sA = w_q G(q) [5][NB] (filled and
// __syncwarp'ed by the caller); sT: the warp's [6][NB][S] scratch; o: the cell's [NB][NB][2] output
template <int S>
__device__ __forceinline__ void sf_cell(const double (*sA)[S * S], double (*sT)[S * S][S], int lane,
                                        const double PLL[S], const double PLD[S], const double PDL[S],
                                        const double PDD[S], double sc, double *o) {
  constexpr int NB = S * S, NG = 32 / NB;   // lane groups
  static_assert(NG >= 1, "S <= 5");
  const int xy = lane % NB, grp = lane / NB, x = xy / S, y = xy % S;
  const bool act = grp < NG;
  if (act) {   // step 1: contract qz for (b, d) = (x, y)
    for (int qr = grp; qr < S; qr += NG) {
      double t1 = 0.0, t2 = 0.0, t3 = 0.0, t4 = 0.0, t5 = 0.0, t6 = 0.0;
#pragma unroll
      for (int qz = 0; qz < S; qz++) {
        const int q = qz * S + qr;
        const double arr = sA[0][q], arz = sA[1][q], azz = sA[2][q], kr = sA[3][q], kz = sA[4][q];
        t1 = fma(PLL[qz], arr, t1);
        t2 = fma(PLD[qz], arz, t2);
        t3 = fma(PDL[qz], arz, t3);
        t4 = fma(PDD[qz], azz, t4);
        t5 = fma(PLL[qz], kr, t5);
        t6 = fma(PDL[qz], kz, t6);
      }
      sT[0][xy][qr] = t1;
      sT[1][xy][qr] = t2;
      sT[2][xy][qr] = t3;
      sT[3][xy][qr] = t4;
      sT[4][xy][qr] = t5;
      sT[5][xy][qr] = t6;
    }
  }
  __syncwarp();
  if (act) {   // step 2: contract qr for (a, c) = (x, y), every (b, d) of the lane's group
    const double sc2 = sc * sc;
    for (int bd = grp; bd < NB; bd += NG) {
      double cd = 0.0, ck = 0.0;
#pragma unroll
      for (int qr = 0; qr < S; qr++) {
        cd = fma(PDD[qr], sT[0][bd][qr], cd);
        cd = fma(PDL[qr], sT[1][bd][qr], cd);
        cd = fma(PLD[qr], sT[2][bd][qr], cd);
        cd = fma(PLL[qr], sT[3][bd][qr], cd);
        ck = fma(PDL[qr], sT[4][bd][qr], ck);
        ck = fma(PLL[qr], sT[5][bd][qr], ck);
      }
      const int k = (bd / S) * S + x, l = (bd % S) * S + y;
      reinterpret_cast<double2 *>(o)[k * NB + l] = make_double2(cd * sc2, ck * sc);   // (C^D, C^K) interleaved
    }
  }
}

template <int S>
__global__ void __launch_bounds__(32 * kSfWarps) element_sf_kernel(int64_t ncell, const double *__restrict__ G,
                                                                   int64_t Nc, int nbatch, int b0, int nb,
                                                                   const double *__restrict__ pw,
                                                                   const double *__restrict__ cell_h,
                                                                   const double *__restrict__ tab1,
                                                                   double *__restrict__ Cbuf) {
  constexpr int NB = S * S;
  __shared__ double sA[kSfWarps][5][NB];       // w_q G(q)
  __shared__ double sT[kSfWarps][6][NB][S];    // T_t[(b,d)][qr]
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  double PLL[S], PLD[S], PDL[S], PDD[S];
  sf_tables<S>(tab1, lane, PLL, PLD, PDL, PDD);
  const unsigned nc = (unsigned)ncell, nitems = (unsigned)(ncell * nb);   // < 2^32 (checked by the caller)
  for (unsigned it = blockIdx.x * kSfWarps + wid; it < nitems; it += gridDim.x * kSfWarps) {
    const int bc = (int)(it / nc), b = b0 + bc;
    const int64_t e = it % nc;
    __syncwarp();   // the previous cell's readers are done with sA / sT
    if (lane < NB) {
      const int64_t i = e * NB + lane;
      const int64_t chunk = i / Nc, off = i % Nc;
      const double *Gb = G + ((chunk * nbatch + b) * 5) * Nc + off;
      const double w = pw[i];
#pragma unroll
      for (int c = 0; c < 5; c++) sA[wid][c][lane] = w * Gb[c * Nc];
    }
    __syncwarp();
    sf_cell<S>(sA[wid], sT[wid], lane, PLL, PLD, PDL, PDD, 2.0 / cell_h[e], Cbuf + ((int64_t)bc * ncell + e) * 2 * NB * NB);
  }
}

// Mass element matrices (create time): M[k,l] = sum_q w_q phi_k phi_l, stored in the element-buffer
// layout [cell][k][l][2] (interleaved with the advection matrix) so the same gather maps apply.
template <int NB>
__global__ void __launch_bounds__(NB * NB) mass_element_kernel(int64_t ncell, const double *__restrict__ pw,
                                                                 const double *__restrict__ cell_h,
                                                                 const double *__restrict__ tab, double *__restrict__ Mbuf) {
  // [cell][0][k][l] = sum_q w phi_k phi_l (mass, a-6); [cell][1][k][l] = sum_q w phi_k d_z phi_l (the
  // E_z advection term of Eq. 4, @8216-8654, before its species factor e_a E_z / m_a)
  __shared__ double s_phi[NB][NB], s_dxi[NB][NB], s_deta[NB][NB];
  load_tables<NB>(tab, s_phi, s_dxi, s_deta);
  __syncthreads();
  const int64_t e = blockIdx.x;
  const int tid = threadIdx.x, k = tid / NB, l = tid % NB;
  const double sz = 2.0 / cell_h[e];
  double m = 0.0, adv = 0.0;
  for (int q = 0; q < NB; q++) {
    const double wp = pw[e * NB + q] * s_phi[q][k];
    m = fma(wp, s_phi[q][l], m);
    adv = fma(wp, sz * s_deta[q][l], adv);
  }
  Mbuf[e * 2 * NB * NB + 2 * tid] = m;   // [cell][k][l][mass | advection], the element-buffer layout
  Mbuf[e * 2 * NB * NB + 2 * tid + 1] = adv;
}

// ------------------------------------------------------------------------------------------------
// N4: deterministic gather.  For grid slot s (CSR nonzero or COO entry):
//   sD = sum_k w_k C^D[idx_k], sK = sum_k w_k C^K[idx_k]   (fixed (cell, a, b) order)
//   out[b][out_off(a) + s] = fD_a sD + fK_a sK   for every species a on the grid   (a-3 + a-5)
// ------------------------------------------------------------------------------------------------
struct GatherDev {
  const int64_t *ptr;
  const int32_t *idx;
  const double *w;
  int64_t nslots;
  int nsp;                        // species on this grid
  int64_t out_off[kMaxSpecies];   // output offset per species on this grid
  double fD[kMaxSpecies], fK[kMaxSpecies];   // a-3 species factors
};

template <int NB, int BPT>
__global__ void assemble_kernel(const GatherDev gm, const double *__restrict__ Cbuf, int64_t cbuf_bstride,
                                double *__restrict__ out, int64_t out_bstride, int nbatch) {
  // a thread gathers one slot for BPT batch items: the map (ptr, idx, w) is read once and the BPT
  // element-matrix loads per contribution are independent (memory-level parallelism)
  const int b0 = blockIdx.y * BPT;
  const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= gm.nslots) return;
  const int nb = min(BPT, nbatch - b0);
  const double *C = Cbuf + (int64_t)b0 * cbuf_bstride;
  const int64_t k0 = gm.ptr[s], k1 = gm.ptr[s + 1];
  double sD[BPT], sK[BPT];
#pragma unroll
  for (int t = 0; t < BPT; t++) sD[t] = sK[t] = 0.0;
#ifndef LANDAU_ASM_UNROLL
#define LANDAU_ASM_UNROLL 4   // contributions unrolled per slot (1: 181 us, 2: 191, 4: 175, 8: 179 on C4 1024)
#endif
  constexpr int kAsmUnroll = LANDAU_ASM_UNROLL;
#pragma unroll kAsmUnroll
  for (int64_t k = k0; k < k1; k++) {
    const int64_t i = gm.idx[k];
    const double w = gm.w[k];
#pragma unroll
    for (int t = 0; t < BPT; t++)
      if (t < nb) {
        const double2 v = __ldg(reinterpret_cast<const double2 *>(C + t * cbuf_bstride + i));   // (C^D, C^K)
        sD[t] = fma(w, v.x, sD[t]);
        sK[t] = fma(w, v.y, sK[t]);
      }
  }
#pragma unroll
  for (int t = 0; t < BPT; t++)
    if (t < nb) {
      double *o = out + (int64_t)(b0 + t) * out_bstride;
      for (int q = 0; q < gm.nsp; q++) o[gm.out_off[q] + s] = fma(gm.fD[q], sD[t], gm.fK[q] * sK[t]);
    }
}

// ------------------------------------------------------------------------------------------------
// N3 + N4 fused (batches of small meshes, C4): a persistent CTA owns one batch item at a time and
// walks each grid's phases (host_setup.h PhaseMaps: runs of consecutive cells).  Per phase its warps
// compute the phase's element matrices (C^D, C^K) by sum factorisation (sf_cell) into SHARED memory --
// the two-kernel form writes and reads them through HBM (285 MB each way per C4 build) -- then every
// thread gathers output slots of the phase from shared memory, four slots at a time with all their
// map loads independent and coalesced (ELL layout).  A slot straddling phases carries its running
// fma sums from phase to phase in shared memory, so every slot is the same fma chain in the same
// (cell, a, b) order as assemble_kernel: bitwise identical values.
// ------------------------------------------------------------------------------------------------
struct TailDev {
  const int32_t *grid_phase_ptr, *cell_ptr, *slot_ptr;
  const int2 *meta, *optr;
  const int4 *idx4;
  const double2 *w4;   // [2 * slots]: (w0, w1), (w2, w3)
  const int32_t *oidx;
  const double *ow;
  int ngrids, nphases, max_cells, max_cross;
};
constexpr int kTailMaxPhases = 64;

template <int S>
__host__ __device__ constexpr int tail_warps() { return S == 5 ? 8 : 16; }

// dynamic shared memory: element matrices of max_cells cells | sA [warps][5][NB] | sT [warps][6][NB][S]
// | straddling-slot running sums [max_cross] double2
template <int S>
__host__ __device__ constexpr size_t tail_smem_bytes(int max_cells, int max_cross) {
  return sizeof(double) * ((size_t)max_cells * 2 * S * S * S * S + (size_t)tail_warps<S>() * (5 * S * S + 6 * S * S * S) +
                           2 * (size_t)max_cross);
}

template <int S>
__global__ void __launch_bounds__(32 * tail_warps<S>(), 1) tail_kernel(const double *__restrict__ G, int64_t N,
                                                                       int nbatch, const double *__restrict__ pw,
                                                                       const double *__restrict__ cell_h,
                                                                       const double *__restrict__ tab1, const TailDev td,
                                                                       const GatherDev *__restrict__ maps,
                                                                       double *__restrict__ out, int64_t out_bstride) {
  constexpr int NB = S * S, W = tail_warps<S>(), kS = 4;
  extern __shared__ double s_tail[];
  __shared__ int s_gp[kMaxSpecies + 1], s_cp[kTailMaxPhases + 1], s_sp[kTailMaxPhases + 1];
  __shared__ GatherDev s_gm[kMaxSpecies];   // species of each grid (a-3)
  double *sC = s_tail;
  double(*sA)[5][NB] = reinterpret_cast<double(*)[5][NB]>(sC + (size_t)td.max_cells * 2 * NB * NB);
  double(*sT)[6][NB][S] = reinterpret_cast<double(*)[6][NB][S]>(sC + (size_t)td.max_cells * 2 * NB * NB + W * 5 * NB);
  double2 *sX = reinterpret_cast<double2 *>(sC + (size_t)td.max_cells * 2 * NB * NB + W * (5 * NB + 6 * NB * S));
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int k = threadIdx.x; k <= td.nphases; k += blockDim.x) {   // the phase tables, once per CTA
    s_cp[k] = td.cell_ptr[k];
    s_sp[k] = td.slot_ptr[k];
  }
  for (int k = threadIdx.x; k <= td.ngrids; k += blockDim.x) s_gp[k] = td.grid_phase_ptr[k];
  for (int k = threadIdx.x; k < td.ngrids; k += blockDim.x) s_gm[k] = maps[k];
  double PLL[S], PLD[S], PDL[S], PDD[S];
  sf_tables<S>(tab1, lane, PLL, PLD, PDL, PDD);
  __syncthreads();
  for (int b = blockIdx.x; b < nbatch; b += gridDim.x) {
    const double *Gb = G + (int64_t)b * 5 * N;
    double *ob = out + (int64_t)b * out_bstride;
    for (int g = 0; g < td.ngrids; g++) {
      const GatherDev &gm = s_gm[g];
      for (int ph = s_gp[g]; ph < s_gp[g + 1]; ph++) {
        const int64_t c0 = s_cp[ph];
        const int nc = s_cp[ph + 1] - (int)c0;
        for (int lc = wid; lc < nc; lc += W) {   // a-4: one warp per cell
          const int64_t e = c0 + lc;
          __syncwarp();   // the previous cell's readers are done with sA / sT
          if (lane < NB) {
            const int64_t i = e * NB + lane;
            const double w = pw[i];
#pragma unroll
            for (int c = 0; c < 5; c++) sA[wid][c][lane] = w * Gb[c * N + i];
          }
          __syncwarp();
          sf_cell<S>(sA[wid], sT[wid], lane, PLL, PLD, PDL, PDD, 2.0 / cell_h[e], sC + (size_t)lc * 2 * NB * NB);
        }
        __syncthreads();   // the phase's element matrices are complete
        const int s0 = s_sp[ph], s1 = s_sp[ph + 1];
        for (int i0 = s0 + threadIdx.x; i0 < s1; i0 += kS * blockDim.x) {   // a-3 + a-5
          int2 mt[kS], op[kS];
          int4 ix[kS];
          double2 wa[kS], wb[kS];
#pragma unroll
          for (int t = 0; t < kS; t++) {   // every map load of the four slots in flight at once
            const int i = i0 + t * blockDim.x;
            const bool v = i < s1;
            mt[t] = v ? td.meta[i] : make_int2(0, 0);
            ix[t] = v ? td.idx4[i] : make_int4(0, 0, 0, 0);
            wa[t] = v ? td.w4[2 * i] : make_double2(0.0, 0.0);
            wb[t] = v ? td.w4[2 * i + 1] : make_double2(0.0, 0.0);
            op[t] = v ? td.optr[i] : make_int2(0, 0);
          }
#pragma unroll
          for (int t = 0; t < kS; t++) {
            const int i = i0 + t * blockDim.x;
            if (i >= s1) continue;
            const int mode = mt[t].y & 3, nin = (mt[t].y >> 2) & 7, x = mt[t].y >> 5;
            double sD = 0.0, sK = 0.0;
            if (mode >= 2) {   // continue the running sums of the earlier phases
              sD = sX[x].x;
              sK = sX[x].y;
            }
            const int id[4] = {ix[t].x, ix[t].y, ix[t].z, ix[t].w};
            const double wt[4] = {wa[t].x, wa[t].y, wb[t].x, wb[t].y};
#pragma unroll
            for (int u = 0; u < 4; u++)
              if (u < nin) {
                const double2 c = *reinterpret_cast<const double2 *>(sC + id[u]);   // (C^D, C^K)
                sD = fma(wt[u], c.x, sD);
                sK = fma(wt[u], c.y, sK);
              }
            for (int k = op[t].x; k < op[t].y; k++) {   // slots with more than four contributions
              const double2 c = *reinterpret_cast<const double2 *>(sC + td.oidx[k]);
              const double w = td.ow[k];
              sD = fma(w, c.x, sD);
              sK = fma(w, c.y, sK);
            }
            if (mode == 1 || mode == 2) {
              sX[x] = make_double2(sD, sK);
            } else {
              const int64_t s = mt[t].x;
              for (int q = 0; q < gm.nsp; q++) ob[gm.out_off[q] + s] = fma(gm.fD[q], sD, gm.fK[q] * sK);
            }
          }
        }
        __syncthreads();   // the next phase overwrites the element matrices
      }
    }
  }
}

// mass gather (create time): out[s] = sum_k w_k M[idx_k]
// (M points at the mass entries of the element buffer, or at M + 1 for the interleaved advection ones)
__global__ void mass_gather_kernel(const int64_t *__restrict__ ptr, const int32_t *__restrict__ idx,
                                   const double *__restrict__ w, int64_t nslots, const double *__restrict__ M,
                                   double *__restrict__ out) {
  const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nslots) return;
  double v = 0.0;
  for (int64_t k = ptr[s]; k < ptr[s + 1]; k++) v = fma(w[k], M[idx[k]], v);
  out[s] = v;
}

// NEXT-3: y[b][off + i] = scale * sum_q A[q] x[b][off + col[q]] over one species block's CSR rows
// (one warp per row, lanes over its nonzeros, fixed-order shuffle reduction: deterministic)
__global__ void block_spmv_kernel(const int64_t *__restrict__ rowptr, const int32_t *__restrict__ col,
                                 const double *__restrict__ A, int n, int64_t off, int64_t ndof, double scale,
                                 const double *__restrict__ x, double *__restrict__ y, int nbatch) {
  const int lane = threadIdx.x & 31;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (w >= (int64_t)nbatch * n) return;
  const int64_t b = w / n;
  const int i = (int)(w % n);
  const double *xb = x + b * ndof + off;
  double s = 0.0;
  for (int64_t q = rowptr[i] + lane; q < rowptr[i + 1]; q += 32) s = fma(A[q], xb[col[q]], s);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) y[b * ndof + off + i] = scale * s;
}

// NEXT-3: per batch item, out[b] = (sum (x - y)^2, sum x^2) in a fixed-order block reduction
__global__ void __launch_bounds__(256) delta_norm_kernel(const double *__restrict__ x, const double *__restrict__ y,
                                                         int64_t ndof, double *__restrict__ out) {
  __shared__ double s_d[256], s_x[256];
  const int64_t b = blockIdx.x;
  double d = 0.0, xx = 0.0;
  for (int64_t i = threadIdx.x; i < ndof; i += 256) {
    const double xi = x[b * ndof + i], di = xi - y[b * ndof + i];
    d = fma(di, di, d);
    xx = fma(xi, xi, xx);
  }
  s_d[threadIdx.x] = d;
  s_x[threadIdx.x] = xx;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if ((int)threadIdx.x < o) {
      s_d[threadIdx.x] += s_d[threadIdx.x + o];
      s_x[threadIdx.x] += s_x[threadIdx.x + o];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    out[2 * b] = s_d[0];
    out[2 * b + 1] = s_x[0];
  }
}

// NEXT-3: z = a x + y (the implicit step's f_old / dt + sigma)
__global__ void axpby_kernel(int64_t n, double a, const double *__restrict__ x, const double *__restrict__ y,
                             double *__restrict__ z) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    z[i] = fma(a, x[i], y[i]);
}

// N5: out[o0 + i] = shift * M[i]
__global__ void scale_copy_kernel(const double *__restrict__ M, double shift, int64_t n, double *__restrict__ out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = shift * M[i];
}

// every species block in one launch: out[off_a + i] = scale_a * M_a[i], i < n_a (blockIdx.y = a)
struct ScaleCopyDesc {
  const double *M[kMaxSpecies];
  int64_t n[kMaxSpecies], off[kMaxSpecies];
  double scale[kMaxSpecies];
};
__global__ void scale_copy_species_kernel(const ScaleCopyDesc d, double *__restrict__ out) {
  const int a = blockIdx.y;
  const double *M = d.M[a];
  const double sc = d.scale[a];
  double *o = out + d.off[a];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < d.n[a]; i += (int64_t)gridDim.x * blockDim.x)
    o[i] = sc * M[i];
}

// copy chunked G layout -> [b][5][N]
__global__ void unchunk_kernel(const double *__restrict__ G, int64_t N, int64_t Nc, int nbatch, double *__restrict__ out) {
  const int64_t total = (int64_t)nbatch * 5 * N;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = k / (5 * N), c = (k / N) % 5, i = k % N;
    out[k] = G[(((i / Nc) * nbatch + b) * 5 + c) * Nc + (i % Nc)];
  }
}


}  // namespace landau
