// kernels_single.cuh -- one persistent cooperative launch for a whole small build (single C1-C3 grids,
// batches of a few items on a z-mirror mesh): a-1 point fields -> a-2 mirror-directed inner integral
// over source splits -> a-2r split reduction -> a-4 element matrices -> a-3 + a-5 assembly, the phases
// separated by grid-wide barriers instead of kernel boundaries (a C2 build as six graph-replayed
// kernels was 46 us, ~6 us of launch and drain per kernel on B200).  a-1, a-4 and a-5 run exactly the
// arithmetic of field_kernel, element_sf_kernel and assemble_kernel; a-2 evaluates the same tensors as
// inner_mdir_kernel, but a CTA owns a group of 8 source splits of one target tile and adds its warps'
// sums in shared memory before one partial per group is written, so only ~nsplit/8 partials remain for
// a-2r -- the same sums in another grouping (within rounding of the multi-kernel build).
// (included once, by landau.cu, after kernels_fe.cuh and kernels_inner.cuh)
#pragma once
#include <cooperative_groups.h>

#include <cstdint>

#include "kernels.cuh"

namespace landau {

constexpr int kSbWarps = 8;   // 256 threads per CTA, one CTA per SM
#ifndef LANDAU_SB_FOLD_REDUCE
#define LANDAU_SB_FOLD_REDUCE 1
#endif
// a-2r folded into a-4: each element warp sums its points' group partials itself (same order as the
// reduction phase, so bitwise the same G), which saves that phase and one grid barrier
constexpr bool kSbFoldReduce = LANDAU_SB_FOLD_REDUCE != 0;

struct SingleBuildArgs {
  // a-1
  int64_t ncell, ndof_total;
  int nbatch;
  const double *f;
  const int32_t *ext_ptr, *ext_dof;
  const double *ext_w;
  const int *cell_grid;
  const double *cell_h, *pw, *tab, *tab1;
  SpeciesConst sp;
  double *wT;
  int64_t npts;
  // a-2 (mirror directed, nsplit source splits of split_len upper-half points) and a-2r
  int64_t H, T, split_len;
  int nsplit;
  const double *rU, *zU;
  const int32_t *pu, *pm;
  const int32_t *pinv;   // point -> ut (+ H for the mirror point pm[ut])
  double *G, *part;
  // a-4 element buffer, a-5 gather maps (one per grid) and output
  double *Cbuf;
  const GatherDev *maps;
  int ngrids;
  double *out;
  int64_t out_bstride;
};

template <int NB>
__global__ void __launch_bounds__(32 * kSbWarps, 1) single_build_kernel(const SingleBuildArgs a) {
  namespace cg = cooperative_groups;
  constexpr int S = NB == 9 ? 3 : (NB == 16 ? 4 : 5);
  constexpr int EPB = 32 * kSbWarps / NB;   // cells per block in the field phase
  cg::grid_group grid = cg::this_grid();
  __shared__ double s_coef[kNumPairCoef];
  __shared__ double2 s_ltab[kLogTab];
  __shared__ union {
    struct {   // a-1: transposed tables, combined element coefficients
      double phi[NB][NB], dxi[NB][NB], deta[NB][NB], gD[EPB][NB], gK[EPB][NB];
    } fld;
    struct {                         // a-2: the warps' staged source tiles, their sums of one group
      double2 sj[kSbWarps][32 * 5];
      double red[kSbWarps * 32 * 10];
    } in;
    struct {                         // a-4: w G per cell, first-contraction scratch
      double A[kSbWarps][5][NB];
      double T[kSbWarps][6][NB][S];
    } el;
  } u;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#ifdef LANDAU_SB_PROFILE   // build variant: phase timestamps of CTA 0 (globaltimer, ns)
  unsigned long long t_[8];
  int nt_ = 0;
#define SB_STAMP()                                                                  \
  if (blockIdx.x == 0 && threadIdx.x == 0) {                                        \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_[nt_]));                     \
    nt_++;                                                                          \
  }
#else
#define SB_STAMP()
#endif
  SB_STAMP();
  stage_pair_coef(s_coef, s_ltab);

  // ---- a-1 point fields (field_kernel's arithmetic, one cell per NB threads) ----------------------
  for (int i = threadIdx.x; i < NB * NB; i += blockDim.x) {
    u.fld.phi[i % NB][i / NB] = a.tab[i];
    u.fld.dxi[i % NB][i / NB] = a.tab[NB * NB + i];
    u.fld.deta[i % NB][i / NB] = a.tab[2 * NB * NB + i];
  }
#ifndef LANDAU_SB_SKIP
#define LANDAU_SB_SKIP 0
#endif
  if (!(LANDAU_SB_SKIP & 1)) {
    const int el = threadIdx.x / NB, q = threadIdx.x % NB;
    const int64_t nchunks = (a.ncell + EPB - 1) / EPB;
    for (int64_t it = blockIdx.x; it < nchunks * a.nbatch; it += gridDim.x) {
      const int64_t b = it / nchunks, e = (it % nchunks) * EPB + el;
      const bool live = el < EPB && e < a.ncell;
      __syncthreads();   // tables loaded / the previous item's gD, gK consumed
      if (live) {
        const int g = a.cell_grid[e];
        const int32_t k0 = a.ext_ptr[e * NB + q], nk = a.ext_ptr[e * NB + q + 1] - k0;
        const double *fb = a.f + b * a.ndof_total;
        double sD = 0.0, sK = 0.0;
        for (int s = 0; s < a.sp.grid_nsp[g]; s++) {
          const int sp = a.sp.grid_sp[g][s];
          const double *fs = fb + a.sp.soff[sp];
          double v = 0.0;
          for (int k = 0; k < nk; k++) v = fma(a.ext_w[k0 + k], __ldg(fs + a.ext_dof[k0 + k]), v);
          sD = fma(a.sp.e2[sp], v, sD);
          sK = fma(a.sp.e2m[sp], v, sK);
        }
        u.fld.gD[el][q] = sD;
        u.fld.gK[el][q] = sK;
      }
      __syncthreads();
      if (live) {
        const int64_t pt = e * NB + q;
        const double w = a.pw[pt], ws = w * (2.0 / a.cell_h[e]);
        double td = 0.0, tr = 0.0, tz = 0.0;
#pragma unroll
        for (int k = 0; k < NB; k++) {
          td = fma(u.fld.phi[k][q], u.fld.gD[el][k], td);
          tr = fma(u.fld.dxi[k][q], u.fld.gK[el][k], tr);
          tz = fma(u.fld.deta[k][q], u.fld.gK[el][k], tz);
        }
        double *o = a.wT + b * 3 * a.npts;
        o[pt] = w * td;
        o[a.npts + pt] = ws * tr;
        o[2 * a.npts + pt] = ws * tz;
      }
    }
  }
  __threadfence();
  grid.sync();
  SB_STAMP();

  // ---- a-2 inner integral: a CTA item is (b, target tile t, group g of 8 source splits); warp w
  // evaluates split 8 g + w of the sources against the tile (inner_mdir_kernel's per-warp arithmetic),
  // the CTA adds its warps' sums in warp order in shared memory and writes one partial per group ------
  if (!(LANDAU_SB_SKIP & 2)) {
    PairCoef cf;
    load_pair_coef(s_coef, s_ltab, cf);
    const int64_t N = a.npts, Hp = a.T * 32, ngroups = (a.nsplit + kSbWarps - 1) / kSbWarps;
    const int64_t nitems = (int64_t)a.nbatch * a.T * ngroups;
    for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
      const int64_t b = item / (a.T * ngroups), t = (item / ngroups) % a.T, g = item % ngroups;
      const int sp = (int)(g * kSbWarps + wid);
      const int64_t uu = t * 32 + lane;
      const double *wb = a.wT + b * 3 * N;
      const double r = uu < a.H ? a.rU[uu] : 1.0;
      const double z = uu < a.H ? a.zU[uu] : 1.0e6 + lane;
      const double r2 = r * r;
      const double nohp[3] = {0.0, 0.0, 0.0};
      Acc5 P{0.0, 0.0, 0.0, 0.0, 0.0}, M{0.0, 0.0, 0.0, 0.0, 0.0}, PJ, MJ;
      const int64_t j0 = min(a.H, (int64_t)sp * a.split_len), j1 = min(a.H, j0 + a.split_len);
      double2 *sj = u.in.sj[wid];
      for (int64_t jt = j0; jt < j1; jt += 32) {
        __syncwarp();
        {
          const int64_t j = jt + lane;
          double A[3], Bf[3];
          mir_weights(wb, N, j1, a.pu, a.pm, j, A, Bf);
          const double rj = j < j1 ? a.rU[j] : 1.0;
          const double zj = j < j1 ? a.zU[j] : 2.0e6 + lane;
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
      double *rw = u.in.red + ((size_t)wid * 32 + lane) * 10;   // this warp's (Ga, Gb) of the lane's target
      rw[0] = P.drr + M.drr;
      rw[1] = P.drz + M.drz;
      rw[2] = P.dzz + M.dzz;
      rw[3] = P.kr + M.kr;
      rw[4] = P.kz + M.kz;
      rw[5] = P.drr - M.drr;
      rw[6] = P.drz - M.drz;
      rw[7] = P.dzz - M.dzz;
      rw[8] = P.kr - M.kr;
      rw[9] = P.kz - M.kz;
      __syncthreads();
      if (threadIdx.x < 320 && threadIdx.x < 32 * kSbWarps) {   // (lane, component) pairs: the group's sum
        for (int x = threadIdx.x; x < 320; x += 32 * kSbWarps) {
          const int ln = x % 32, c = x / 32;
          double acc = 0.0;
          for (int w = 0; w < kSbWarps; w++) acc += u.in.red[((size_t)w * 32 + ln) * 10 + c];   // warp order
          const int64_t ut = t * 32 + ln;
          if (ut >= a.H) continue;
          if (ngroups == 1) {   // G(pu) = Ga, G(pm) = F Gb
            double *Gb = a.G + b * 5 * N;
            if (c < 5) Gb[c * N + a.pu[ut]] = acc;
            else Gb[(c - 5) * N + a.pm[ut]] = (c == 6 || c == 9) ? -acc : acc;
          } else {
            a.part[((b * ngroups + g) * 10 + c) * Hp + ut] = acc;
          }
        }
      }
      __syncthreads();   // u.in.red is reused by the next item
    }
  }
  __threadfence();
  grid.sync();
  SB_STAMP();

  // ---- a-2r: the groups' partials summed in group order (one thread per (b, component, point)) ----
  {
    const int64_t N = a.npts, Hp = a.T * 32, ngroups = (a.nsplit + kSbWarps - 1) / kSbWarps;
    if (ngroups > 1 && !(LANDAU_SB_SKIP & 4) && !kSbFoldReduce) {
      const int64_t total = (int64_t)a.nbatch * 10 * a.H;
      for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = k / (10 * a.H), c = (k / a.H) % 10, ut = k % a.H;
        double acc = 0.0;
        for (int64_t g = 0; g < ngroups; g++) acc += __ldcg(a.part + ((b * ngroups + g) * 10 + c) * Hp + ut);
        double *Gb = a.G + b * 5 * N;
        if (c < 5) Gb[c * N + a.pu[ut]] = acc;
        else Gb[(c - 5) * N + a.pm[ut]] = (c == 6 || c == 9) ? -acc : acc;
      }
      __threadfence();
      grid.sync();
    }
  }
  SB_STAMP();

  // ---- a-4 element matrices (element_sf_kernel's arithmetic, one warp per cell) -------------------
  if (!(LANDAU_SB_SKIP & 8)) {
    double PLL[S], PLD[S], PDL[S], PDD[S];
    sf_tables<S>(a.tab1, lane, PLL, PLD, PDL, PDD);
    const int64_t N = a.npts, nitems = a.ncell * a.nbatch;
    for (int64_t it = (int64_t)blockIdx.x * kSbWarps + wid; it < nitems; it += (int64_t)gridDim.x * kSbWarps) {
      const int64_t b = it / a.ncell, e = it % a.ncell;
      __syncwarp();
      if (lane < NB) {
        const int64_t i = e * NB + lane;
        const double w = a.pw[i];
        const int64_t Hp = a.T * 32, ngroups = (a.nsplit + kSbWarps - 1) / kSbWarps;
        if (kSbFoldReduce && ngroups > 1) {   // a-2r here: the groups' partials of this point, in group order
          const int32_t pv = a.pinv[i];
          const bool mir = pv >= a.H;
          const int64_t ut = mir ? pv - a.H : pv;
#pragma unroll
          for (int c = 0; c < 5; c++) {
            const int cc = mir ? c + 5 : c;
            double acc = 0.0;
            for (int64_t g = 0; g < ngroups; g++) acc += __ldcg(a.part + ((b * ngroups + g) * 10 + cc) * Hp + ut);
            u.el.A[wid][c][lane] = w * ((mir && (c == 1 || c == 4)) ? -acc : acc);
          }
        } else {
          const double *Gb = a.G + b * 5 * N + i;
#pragma unroll
          for (int c = 0; c < 5; c++) u.el.A[wid][c][lane] = w * Gb[c * N];
        }
      }
      __syncwarp();
      sf_cell<S>(u.el.A[wid], u.el.T[wid], lane, PLL, PLD, PDL, PDD, 2.0 / a.cell_h[e],
                 a.Cbuf + (b * a.ncell + e) * 2 * NB * NB);
    }
  }
  __threadfence();
  grid.sync();
  SB_STAMP();

  // ---- a-3 + a-5 assembly (assemble_kernel's arithmetic: one slot per thread) ----------------------
  for (int g = 0; g < ((LANDAU_SB_SKIP & 16) ? 0 : a.ngrids); g++) {
    const GatherDev &gm = a.maps[g];
    const int64_t total = gm.nslots * a.nbatch;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (int64_t)gridDim.x * blockDim.x) {
      const int64_t b = k / gm.nslots, s = k % gm.nslots;
      const double *C = a.Cbuf + b * a.ncell * 2 * NB * NB;
      double sD = 0.0, sK = 0.0;
      for (int64_t q = gm.ptr[s]; q < gm.ptr[s + 1]; q++) {
        const double w = gm.w[q];
        const double2 v = *reinterpret_cast<const double2 *>(C + gm.idx[q]);
        sD = fma(w, v.x, sD);
        sK = fma(w, v.y, sK);
      }
      double *o = a.out + b * a.out_bstride;
      for (int q = 0; q < gm.nsp; q++) o[gm.out_off[q] + s] = fma(gm.fD[q], sD, gm.fK[q] * sK);
    }
  }
#ifdef LANDAU_SB_PROFILE
  grid.sync();
  SB_STAMP();
  if (blockIdx.x == 0 && threadIdx.x == 0)
    printf("SB grid %d nsplit %d: field %.2f inner %.2f reduce %.2f element %.2f assemble %.2f us\n", gridDim.x,
           a.nsplit, (t_[1] - t_[0]) * 1e-3, (t_[2] - t_[1]) * 1e-3, (t_[3] - t_[2]) * 1e-3, (t_[4] - t_[3]) * 1e-3,
           (t_[5] - t_[4]) * 1e-3);
#endif
}

}  // namespace landau
