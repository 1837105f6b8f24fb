// kernels_3d.cuh -- NEXT-4 of SURVEY.md §8(f): the inner integral with the 3D Cartesian Landau tensor
// of Eq. 3 (PAPER.md:1@7593), U(u) = (|u|^2 I - u u^T) / |u|^3, u = v_i - v_j -- the "full 3D model"
// of @7997-8072: no azimuthal integration, no elliptic integrals, one rsqrt per ordered pair.
//   G_D(i) = sum_{j: v_j != v_i} wTD_j U(u)      (xx, xy, xz, yy, yz, zz)
//   G_K(i) = sum_j U(u) wTK_j = sum_j rs wTK_j - rs^3 (u . wTK_j) u        (x, y, z)
// with rs = 1/|u|, wTD = w T_D and wTK = w T_K premultiplied by the caller.  Directed pairs: a warp
// owns 32 x TPT targets and one split of the sources, staged 32 at a time in shared memory and read
// by every lane at once (broadcast); coincident points contribute nothing (Amb-3).
// (included once, by landau.cu)
#pragma once
#include <cstdint>

#include "kernels.cuh"

namespace landau {

constexpr int k3dWarps = 4;

template <int TPT>
__global__ void __launch_bounds__(32 * k3dWarps) inner3d_kernel(int64_t n, int64_t split_len, int nsplit, int64_t wtiles,
                                                                int64_t nitems, const double *__restrict__ xyz,
                                                                const double *__restrict__ wTD,
                                                                const double *__restrict__ wTK,
                                                                double *__restrict__ out) {
  __shared__ double2 s_a[k3dWarps][32], s_b[k3dWarps][32], s_c[k3dWarps][32];   // (x, y), (z, wTD), (wTKx, wTKy)
  __shared__ double s_d[k3dWarps][32];                                           // wTKz
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t item = (int64_t)blockIdx.x * k3dWarps + wid;
  if (item >= nitems) return;   // whole warp
  const int sp = (int)(item / wtiles);
  const int64_t wt = item % wtiles;
  double tx[TPT], ty[TPT], tz[TPT];
  double gxx[TPT], gxy[TPT], gxz[TPT], gyy[TPT], gyz[TPT], gzz[TPT], kx[TPT], ky[TPT], kz[TPT];
  int64_t ti[TPT];
#pragma unroll
  for (int t = 0; t < TPT; t++) {
    ti[t] = wt * 32 * TPT + t * 32 + lane;
    const int64_t i = ti[t] < n ? ti[t] : n - 1;
    tx[t] = xyz[i];
    ty[t] = xyz[n + i];
    tz[t] = xyz[2 * n + i];
    gxx[t] = gxy[t] = gxz[t] = gyy[t] = gyz[t] = gzz[t] = kx[t] = ky[t] = kz[t] = 0.0;
  }
  const int64_t j0 = (int64_t)sp * split_len, j1 = min(n, j0 + split_len);
  for (int64_t jt = j0; jt < j1; jt += 32) {
    const int64_t j = jt + lane;
    __syncwarp();
    if (j < j1) {
      s_a[wid][lane] = make_double2(xyz[j], xyz[n + j]);
      s_b[wid][lane] = make_double2(xyz[2 * n + j], wTD[j]);
      s_c[wid][lane] = make_double2(wTK[j], wTK[n + j]);
      s_d[wid][lane] = wTK[2 * n + j];
    }
    __syncwarp();
    const int m = (int)min((int64_t)32, j1 - jt);
#pragma unroll 2
    for (int k = 0; k < m; k++) {
      const double2 a = s_a[wid][k], b = s_b[wid][k], c = s_c[wid][k];
      const double wkz = s_d[wid][k];
#pragma unroll
      for (int t = 0; t < TPT; t++) {
        const double ux = tx[t] - a.x, uy = ty[t] - a.y, uz = tz[t] - b.x;
        const double s2 = fma(ux, ux, fma(uy, uy, uz * uz));
        const bool ok = s2 != 0.0;   // coincident points (the self pair) contribute nothing
        const double rs = ok ? rsqrt_pos(s2) : 0.0;
        const double rs3 = rs * rs * rs;
        const double wa = b.y * rs, wb = b.y * rs3;          // G_D += wa I - wb u u^T
        const double bx = wb * ux, by = wb * uy, bz = wb * uz;
        gxx[t] = fma(-bx, ux, gxx[t] + wa);
        gyy[t] = fma(-by, uy, gyy[t] + wa);
        gzz[t] = fma(-bz, uz, gzz[t] + wa);
        gxy[t] = fma(-bx, uy, gxy[t]);
        gxz[t] = fma(-bx, uz, gxz[t]);
        gyz[t] = fma(-by, uz, gyz[t]);
        const double cd = rs3 * fma(ux, c.x, fma(uy, c.y, uz * wkz));   // G_K += rs wTK - rs^3 (u.wTK) u
        kx[t] = fma(-cd, ux, fma(rs, c.x, kx[t]));
        ky[t] = fma(-cd, uy, fma(rs, c.y, ky[t]));
        kz[t] = fma(-cd, uz, fma(rs, wkz, kz[t]));
      }
    }
  }
  double *o = out + (int64_t)sp * 9 * n;
#pragma unroll
  for (int t = 0; t < TPT; t++) {
    const int64_t i = ti[t];
    if (i >= n) continue;
    o[i] = gxx[t];
    o[n + i] = gxy[t];
    o[2 * n + i] = gxz[t];
    o[3 * n + i] = gyy[t];
    o[4 * n + i] = gyz[t];
    o[5 * n + i] = gzz[t];
    o[6 * n + i] = kx[t];
    o[7 * n + i] = ky[t];
    o[8 * n + i] = kz[t];
  }
}

// G[c][i] = sum over splits of part[s][c][i], splits in order
__global__ void reduce3d_kernel(int64_t n, int nsplit, const double *__restrict__ part, double *__restrict__ G) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < 9 * n; k += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int q = 0; q < nsplit; q++) s += part[(int64_t)q * 9 * n + k];
    G[k] = s;
  }
}

}  // namespace landau
