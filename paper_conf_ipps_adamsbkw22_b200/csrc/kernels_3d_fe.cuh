// kernels_3d_fe.cuh -- NEXT-4 of SURVEY.md §8(f) completed: the finite-element half of a 3D Cartesian
// Landau Jacobian ("a full 3D model is supported in the library", PAPER.md:1@7997-8072), around the
// 3D inner integral of kernels_3d.cuh, on a uniform grid of ncell^3 Q_p cubes over [-R, R]^3:
//   a-1  field3d_kernel    w T_D = w sum_b e_b^2 f_b,  w T_K = w sum_b e_b^2 (m0/m_b) grad f_b  at
//                          every Gauss point (tensor-product basis from 1-D tables)
//   a-2  inner3d_kernel    (kernels_3d.cuh) G_D [6][N], G_K [3][N]
//   a-4  element3d_kernel  C^D_e[k][l] = sum_q w_q grad phi_k . G_D(q) grad phi_l,
//                          C^K_e[k][l] = sum_q w_q (grad phi_k . G_K(q)) phi_l      (Eqs. 5-6 in 3D)
//   a-3 + a-5              assemble_kernel (kernels_fe.cuh) with the species factors and unit weights
// Layouts: points cube-major (cube (cz ncell + cy) ncell + cx), then q = (a S + b) S + c with a, b, c
// the Gauss indices along z, y, x; local node n = (k S + j) S + i (i along x); element buffer
// [cube][NB][NB] of (C^D, C^K) as double2, like the 2D kernels.  (included once, by landau.cu)
#pragma once
#include <cstdint>

#include "kernels.cuh"

namespace landau {

struct Species3D {   // a-1 factors per species: e^2 and e^2 m0/m
  int S;
  double e2[kMaxSpecies], e2m[kMaxSpecies];
};

// a-1: one thread per Gauss point; f = [S][ndof] species-major
template <int S1>
__global__ void field3d_kernel(int64_t npts, const double *__restrict__ f, int64_t ndof, const int32_t *__restrict__ dofs,
                               const double *__restrict__ L1, const double *__restrict__ D1, double scale,
                               const double *__restrict__ w, const Species3D sp, double *__restrict__ wTD,
                               double *__restrict__ wTK) {
  constexpr int NB = S1 * S1 * S1, NQ = NB;
  __shared__ double sL[S1 * S1], sD[S1 * S1];   // [Gauss point][node]: l_node(x_pt), l'_node(x_pt)
  for (int i = threadIdx.x; i < S1 * S1; i += blockDim.x) {
    sL[i] = L1[i];
    sD[i] = D1[i];
  }
  __syncthreads();
  for (int64_t pt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; pt < npts; pt += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = pt / NQ;
    const int q = (int)(pt - e * NQ), qa = q / (S1 * S1), qb = (q / S1) % S1, qc = q % S1;
    const int32_t *de = dofs + e * NB;
    double TD = 0.0, Tx = 0.0, Ty = 0.0, Tz = 0.0;
    for (int s = 0; s < sp.S; s++) {
      const double *fs = f + s * ndof;
      double v = 0.0, dx = 0.0, dy = 0.0, dz = 0.0;
#pragma unroll
      for (int k = 0; k < S1; k++) {
        const double Lz = sL[qa * S1 + k], Dz = sD[qa * S1 + k];
#pragma unroll
        for (int j = 0; j < S1; j++) {
          const double Ly = sL[qb * S1 + j], Dy = sD[qb * S1 + j];
          const double LyLz = Ly * Lz, DyLz = Dy * Lz, LyDz = Ly * Dz;
#pragma unroll
          for (int i = 0; i < S1; i++) {
            const double fv = __ldg(fs + de[(k * S1 + j) * S1 + i]);
            const double Lx = sL[qc * S1 + i], Dx = sD[qc * S1 + i];
            v = fma(Lx * LyLz, fv, v);
            dx = fma(Dx * LyLz, fv, dx);
            dy = fma(Lx * DyLz, fv, dy);
            dz = fma(Lx * LyDz, fv, dz);
          }
        }
      }
      TD = fma(sp.e2[s], v, TD);
      Tx = fma(sp.e2m[s], dx, Tx);
      Ty = fma(sp.e2m[s], dy, Ty);
      Tz = fma(sp.e2m[s], dz, Tz);
    }
    const double wp = w[pt], ws = wp * scale;   // scale = 2 / h: reference -> physical gradients
    wTD[pt] = wp * TD;
    wTK[pt] = ws * Tx;
    wTK[npts + pt] = ws * Ty;
    wTK[2 * npts + pt] = ws * Tz;
  }
}

// a-4: one CTA per cube.  Per Gauss point q the NB node threads form, for their node n,
// g_n = grad phi_n(q), phi_n(q), t_n = w G_D(q) g_n and s_n = g_n . w G_K(q) in shared memory; then every
// thread adds t_k . g_l and s_k phi_l to its entries (k, l) -- q in order, so the sums are
// deterministic.  G = [9][npts] from landau3d_inner; C = [ncube][NB][NB] double2 (C^D, C^K).
constexpr int k3dElThreads = 256;
template <int S1>
__global__ void __launch_bounds__(k3dElThreads) element3d_kernel(int64_t ncube, const double *__restrict__ G, int64_t npts,
                                                                 const double *__restrict__ w,
                                                                 const double *__restrict__ L1,
                                                                 const double *__restrict__ D1, double scale,
                                                                 double2 *__restrict__ C) {
  constexpr int NB = S1 * S1 * S1, NQ = NB, NE = (NB * NB + k3dElThreads - 1) / k3dElThreads;
  __shared__ double sL[S1 * S1], sD[S1 * S1];
  __shared__ double4 s_g[NB];    // (g_x, g_y, g_z, phi)
  __shared__ double4 s_t[NB];    // (t_x, t_y, t_z, s)
  for (int i = threadIdx.x; i < S1 * S1; i += blockDim.x) {
    sL[i] = L1[i];
    sD[i] = D1[i];
  }
  const int tid = threadIdx.x;
  for (int64_t e = blockIdx.x; e < ncube; e += gridDim.x) {
    double aD[NE], aK[NE];
#pragma unroll
    for (int m = 0; m < NE; m++) aD[m] = aK[m] = 0.0;
    for (int q = 0; q < NQ; q++) {
      __syncthreads();   // the previous point's node data consumed (and the tables loaded)
      if (tid < NB) {
        const int qa = q / (S1 * S1), qb = (q / S1) % S1, qc = q % S1;
        const int k = tid / (S1 * S1), j = (tid / S1) % S1, i = tid % S1;
        const double Lx = sL[qc * S1 + i], Ly = sL[qb * S1 + j], Lz = sL[qa * S1 + k];
        const double gx = scale * sD[qc * S1 + i] * Ly * Lz, gy = scale * Lx * sD[qb * S1 + j] * Lz,
                     gz = scale * Lx * Ly * sD[qa * S1 + k];
        const int64_t pt = e * NQ + q;
        const double wp = w[pt];
        const double Dxx = wp * G[pt], Dxy = wp * G[npts + pt], Dxz = wp * G[2 * npts + pt], Dyy = wp * G[3 * npts + pt],
                     Dyz = wp * G[4 * npts + pt], Dzz = wp * G[5 * npts + pt];
        const double Kx = wp * G[6 * npts + pt], Ky = wp * G[7 * npts + pt], Kz = wp * G[8 * npts + pt];
        s_g[tid] = make_double4(gx, gy, gz, Lx * Ly * Lz);
        s_t[tid] = make_double4(fma(Dxx, gx, fma(Dxy, gy, Dxz * gz)), fma(Dxy, gx, fma(Dyy, gy, Dyz * gz)),
                                fma(Dxz, gx, fma(Dyz, gy, Dzz * gz)), fma(gx, Kx, fma(gy, Ky, gz * Kz)));
      }
      __syncthreads();
#pragma unroll
      for (int m = 0; m < NE; m++) {
        const int ent = tid + m * k3dElThreads;
        if (ent < NB * NB) {
          const double4 t = s_t[ent / NB], g = s_g[ent % NB];
          aD[m] = fma(t.x, g.x, fma(t.y, g.y, fma(t.z, g.z, aD[m])));
          aK[m] = fma(t.w, g.w, aK[m]);
        }
      }
    }
#pragma unroll
    for (int m = 0; m < NE; m++) {
      const int ent = tid + m * k3dElThreads;
      if (ent < NB * NB) C[e * NB * NB + ent] = make_double2(aD[m], aK[m]);
    }
  }
}

}  // namespace landau
