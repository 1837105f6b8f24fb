/* oracle.c -- plain CPU reference of the Landau Jacobian (see oracle.h for the citation map).
 *
 * TEST INFRASTRUCTURE ONLY (tests/, smoke(), bench.py cpu_baseline / --impl reference).
 * Deliberately simple: long double everywhere, brute-force searches, no blocking or fusion beyond
 * what the definitions state, Neumaier-compensated sums in fixed j order for the inner integral.
 */
#include "oracle.h"

#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef long double ld;
#define PI_L 3.141592653589793238462643383279502884L

/* ------------------------------------------------------------------------------------------ */
/* data                                                                                         */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
  long long ir, iz; /* lattice position in units of (h_min / p) of its grid, z measured from -R */
} pos_t;

typedef struct {
  int n;           /* number of (dof, weight) terms */
  int *dof;
  ld *wt;
} expand_t;

typedef struct {
  int ncell;
  long long cell0;       /* index of the first cell of this grid in the concatenated list */
  double R;
  double *r0, *z0, *h;   /* per cell */
  long long *R0, *Z0, *H; /* integer cell coordinates in units of h_min */
  int ndof;
  double *node_r, *node_z;
  pos_t *node_pos;       /* sorted DOF positions */
  /* per cell: distinct DOFs (sorted) and dense extraction P[Nb][n_e] */
  int *ne;
  int **edofs;
  ld **P;
  /* CSR pattern of one species block on this grid */
  long long *rowptr;
  int *col;
  long long nnz;
  long long npts, pt0;   /* points of this grid and offset of the first one */
} grid_t;

struct oracle_s {
  int ngrids, p, nq, nb, nqp, S;
  double nu;
  double *mass, *charge;
  int *sgrid;
  grid_t *g;
  long long ndof, npts, nnz, ncoo;
  long long *soff;       /* dof offset of species block */
  long long *snnz_off;   /* nnz offset of species block */
  long long *scoo_off;   /* coo offset of species block */
  /* tables at the reference quadrature points: phi[q][a], dxi[q][a], deta[q][a] */
  ld *xq, *wq;           /* 1D Gauss nodes/weights [nq] */
  ld *phi, *dxi, *deta;
  /* points */
  double *pr, *pz, *pw;  /* [npts] */
  int *pgrid;            /* grid of each point */
};

/* ------------------------------------------------------------------------------------------ */
/* 1D building blocks (O1, O2)                                                                 */
/* ------------------------------------------------------------------------------------------ */
/* Gauss-Legendre nodes and weights on [-1, 1] by Newton on P_n (textbook; pinned by P8). */
static void gauss_legendre(int n, ld *x, ld *w) {
  for (int i = 0; i < n; i++) {
    ld t = cosl(PI_L * (i + 0.75L) / (n + 0.5L));
    for (int it = 0; it < 100; it++) {
      ld p0 = 1.0L, p1 = t;
      for (int k = 2; k <= n; k++) {
        ld p2 = ((2 * k - 1) * t * p1 - (k - 1) * p0) / k;
        p0 = p1;
        p1 = p2;
      }
      if (n == 1) { p0 = 1.0L; p1 = t; }
      ld dp = n * (t * p1 - p0) / (t * t - 1.0L);
      ld dt = p1 / dp;
      t -= dt;
      if (fabsl(dt) < 1e-21L) break;
    }
    ld p0 = 1.0L, p1 = t;
    for (int k = 2; k <= n; k++) {
      ld p2 = ((2 * k - 1) * t * p1 - (k - 1) * p0) / k;
      p0 = p1;
      p1 = p2;
    }
    ld dp = n * (t * p1 - p0) / (t * t - 1.0L);
    x[n - 1 - i] = t;
    w[n - 1 - i] = 2.0L / ((1.0L - t * t) * dp * dp);
  }
}

/* Lagrange polynomial a of degree p on equispaced nodes -1 + 2k/p, and its derivative. */
static ld lag(int p, int a, ld x) {
  ld xa = -1.0L + 2.0L * a / p, v = 1.0L;
  for (int k = 0; k <= p; k++)
    if (k != a) v *= (x - (-1.0L + 2.0L * k / p)) / (xa - (-1.0L + 2.0L * k / p));
  return v;
}
static ld dlag(int p, int a, ld x) {
  ld xa = -1.0L + 2.0L * a / p, s = 0.0L;
  for (int m = 0; m <= p; m++) {
    if (m == a) continue;
    ld xm = -1.0L + 2.0L * m / p;
    ld v = 1.0L / (xa - xm);
    for (int k = 0; k <= p; k++)
      if (k != a && k != m) v *= (x - (-1.0L + 2.0L * k / p)) / (xa - (-1.0L + 2.0L * k / p));
    s += v;
  }
  return s;
}

/* ------------------------------------------------------------------------------------------ */
/* O5: the axisymmetric Landau tensors                                                         */
/* ------------------------------------------------------------------------------------------ */
/* K(m), E(m) (parameter convention) by the arithmetic-geometric mean, fed x = 1 - m directly. */
static void ellip_KE(ld m, ld x, ld *K, ld *E) {
  ld a = 1.0L, b = sqrtl(x), c2sum = 0.5L * m, pw = 0.5L; /* sum 2^(n-1) c_n^2, c_0^2 = m */
  for (int it = 0; it < 64; it++) {
    ld c = 0.5L * (a - b);
    ld an = 0.5L * (a + b);
    ld bn = sqrtl(a * b);
    pw *= 2.0L;
    c2sum += pw * c * c;
    a = an;
    b = bn;
    if (fabsl(c) <= 1e-22L * a) break;
  }
  *K = PI_L / (2.0L * a);
  *E = *K * (1.0L - c2sum);
}

/* Phi_n^k(s) = int_0^{2pi} cos^k(phi) (1 - s cos phi)^(-n/2) dphi
 *           = 2 pi sum_{q>=0, k+q even} [(n/2)_q / q!] s^q C(k+q, (k+q)/2) / 2^(k+q)      (s < 1) */
static ld Phi(int n, int k, ld s) {
  ld sum = 0.0L, a = 1.0L, sq = 1.0L;
  for (int q = 0; q < 400; q++) {
    int j = k + q;
    if ((j & 1) == 0) {
      ld b = 1.0L; /* C(j, j/2) / 2^j */
      for (int i = 1; i <= j / 2; i++) b *= (ld)(2 * i - 1) / (ld)(2 * i);
      ld term = a * sq * b;
      sum += term;
      if (q > 4 && fabsl(term) < 1e-24L * fabsl(sum)) break;
    }
    a *= (0.5L * n + q) / (q + 1);
    sq *= s;
  }
  return 2.0L * PI_L * sum;
}

/* int_0^{2pi} sin^2(phi) (1 - s cos phi)^(-3/2) dphi = Phi_3^0 - Phi_3^2, summed term by term:
 * 2 pi sum_{q even} [(3/2)_q / q!] s^q C(q, q/2) 2^-q / (q + 2)  (since C(q+2,.)/2^(q+2) = C(q,.)/2^q (q+1)/(q+2)) */
static ld Phi_sin(ld s) {
  ld sum = 0.0L, a = 1.0L, sq = 1.0L;
  for (int q = 0; q < 400; q++) {
    if ((q & 1) == 0) {
      ld b = 1.0L;
      for (int i = 1; i <= q / 2; i++) b *= (ld)(2 * i - 1) / (ld)(2 * i);
      ld term = a * sq * b / (q + 2);
      sum += term;
      if (q > 4 && fabsl(term) < 1e-24L * fabsl(sum)) break;
    }
    a *= (1.5L + q) / (q + 1);
    sq *= s;
  }
  return 2.0L * PI_L * sum;
}

/* U^D_rr, U^D_rz, U^D_zz, U^K_rr, U^K_zr  (U^K_rz = U^D_rz, U^K_zz = U^D_zz)
 * U^D_ab = int e_a.U(u).e_b dphi,  U^K_ab = int e_a.U(u).ebar_b(phi) dphi, u = v - vbar(phi),
 * U = (|u|^2 I - u u)/|u|^3 (Eq. 3, @7593).  Closed form (s >= 1/4) and series (s < 1/4) as in
 * SURVEY.md §8(c) O5. */
static void tensor_ld(ld r, ld z, ld rb, ld zb, ld U[5]) {
  ld dz = z - zb;
  ld l = r * r + rb * rb + dz * dz;
  ld s = 2.0L * r * rb / l;
  if (s < 0.25L) {
    /* Series branch.  With |u|^2 = l (1 - s cos phi) the integrand numerators of Eq. 3 are
     *   e_r.(|u|^2 I - u u).e_r         = rb^2 sin^2 phi + dz^2
     *   e_r.(|u|^2 I - u u).e_z         = -dz (r - rb cos phi)
     *   e_z.(|u|^2 I - u u).e_z         = r^2 + rb^2 - 2 r rb cos phi
     *   e_r.(|u|^2 I - u u).ebar_r(phi) = dz^2 cos phi + r rb sin^2 phi
     *   e_z.(|u|^2 I - u u).ebar_r(phi) = -dz (r cos phi - rb)
     * so every component is l^(-3/2) times a combination of Phi_3^0, Phi_3^1 and
     * Phi_sin = int sin^2(phi) (1 - s cos phi)^(-3/2) = Phi_3^0 - Phi_3^2 (summed term by term),
     * which keeps near-axis pairs (s -> 0) free of cancellation (Amb-7). */
    ld l32 = 1.0L / (l * sqrtl(l));
    ld P30 = Phi(3, 0, s), P31 = Phi(3, 1, s), Psn = Phi_sin(s);
    U[0] = l32 * (rb * rb * Psn + dz * dz * P30);
    U[1] = -dz * l32 * (r * P30 - rb * P31);
    U[2] = l32 * ((r * r + rb * rb) * P30 - 2.0L * r * rb * P31);
    U[3] = l32 * (dz * dz * P31 + r * rb * Psn);
    U[4] = -dz * l32 * (r * P31 - rb * P30);
    return;
  }
  ld lp = (r + rb) * (r + rb) + dz * dz;  /* lambda_+ */
  ld lm = (r - rb) * (r - rb) + dz * dz;  /* lambda_- */
  ld x = lm / lp, m = 4.0L * r * rb / lp;
  ld K, E;
  ellip_KE(m, x, &K, &E);
  ld sq = sqrtl(lp);
  ld I1 = 4.0L * K / sq;
  ld I3 = 4.0L * E / (lm * sq);
  ld Im = 4.0L * E * sq / (l * l);
  ld A = ((r - rb) * (r + rb) - dz * dz) / (2.0L * r), B = l / (2.0L * r);
  ld Ap = ((r - rb) * (r + rb) + dz * dz) / (2.0L * rb), Bp = l / (2.0L * rb);
  U[0] = I1 - (A * A * I3 + 2.0L * A * B * I1 / l + B * B * Im);
  U[1] = -dz * (A * I3 + B * I1 / l);
  U[2] = I1 - dz * dz * I3;
  U[3] = (I1 - 4.0L * E * sq / l) / s - (A * Ap * I3 + (B * Ap - A * Bp) * I1 / l - B * Bp * Im);
  U[4] = -dz * (Ap * I3 - Bp * I1 / l);
}

void oracle_tensor(double r, double z, double rb, double zb, double out[5]) {
  ld U[5];
  tensor_ld(r, z, rb, zb, U);
  for (int c = 0; c < 5; c++) out[c] = (double)U[c];
}

/* Neumaier-compensated accumulator */
typedef struct { ld s, c; } nsum_t;
static inline void nadd(nsum_t *a, ld x) {
  ld t = a->s + x;
  if (fabsl(a->s) >= fabsl(x)) a->c += (a->s - t) + x;
  else a->c += (x - t) + a->s;
  a->s = t;
}
static inline ld nval(const nsum_t *a) { return a->s + a->c; }

/* O5 for one target: G[5] and |.| sums */
static void inner_one(long long n, const double *r, const double *z, const double *w, const double *TD,
                      const double *TKr, const double *TKz, long long i, ld G[5], ld Ga[5]) {
  nsum_t acc[5], aac[5];
  memset(acc, 0, sizeof acc);
  memset(aac, 0, sizeof aac);
  for (long long j = 0; j < n; j++) {
    if (r[j] == r[i] && z[j] == z[i]) continue; /* Amb-3: coincident points excluded */
    ld U[5];
    tensor_ld(r[i], z[i], r[j], z[j], U);
    ld wd = (ld)w[j] * (ld)TD[j];
    ld wkr = (ld)w[j] * (ld)TKr[j], wkz = (ld)w[j] * (ld)TKz[j];
    nadd(&acc[0], wd * U[0]);
    nadd(&acc[1], wd * U[1]);
    nadd(&acc[2], wd * U[2]);
    nadd(&acc[3], U[3] * wkr + U[1] * wkz);
    nadd(&acc[4], U[4] * wkr + U[2] * wkz);
    ld awd = fabsl(wd), awkr = fabsl(wkr), awkz = fabsl(wkz);
    nadd(&aac[0], awd * fabsl(U[0]));
    nadd(&aac[1], awd * fabsl(U[1]));
    nadd(&aac[2], awd * fabsl(U[2]));
    nadd(&aac[3], fabsl(U[3]) * awkr + fabsl(U[1]) * awkz);
    nadd(&aac[4], fabsl(U[4]) * awkr + fabsl(U[2]) * awkz);
  }
  for (int c = 0; c < 5; c++) {
    G[c] = nval(&acc[c]);
    Ga[c] = nval(&aac[c]);
  }
}

void oracle_inner(long long n, const double *r, const double *z, const double *w, const double *TD,
                  const double *TKr, const double *TKz, long long nt, const long long *targets,
                  double *G, double *Gabs) {
#pragma omp parallel for schedule(dynamic, 4)
  for (long long t = 0; t < nt; t++) {
    ld g[5], ga[5];
    inner_one(n, r, z, w, TD, TKr, TKz, targets ? targets[t] : t, g, ga);
    for (int c = 0; c < 5; c++) {
      if (G) G[c * nt + t] = (double)g[c];
      if (Gabs) Gabs[c * nt + t] = (double)ga[c];
    }
  }
}

/* ------------------------------------------------------------------------------------------ */
/* O12: the inner integral with the 3D Cartesian Landau tensor of Eq. 3    */
/* (@7593), U(u) = (|u|^2 I - u u^T) / |u|^3, u = v_i - v_j, straight from the definition: no     */
/* azimuthal integration, no elliptic integrals.  "A full 3D model is supported in the library"   */
/* (@7997-8072).  Per target i, over sources j with v_j != v_i (Amb-3), in j order (Neumaier):    */
/*   G_D(i) = sum_j wTD_j U(v_i - v_j)       (xx, xy, xz, yy, yz, zz)                          */
/*   G_K(i) = sum_j U(v_i - v_j) wTK_j       (x, y, z)                                         */
/* with wTD = w T_D, wTK = w T_K premultiplied by the caller (Eqs. 7-8 with the 3D tensor).      */
/* ------------------------------------------------------------------------------------------ */
void oracle_tensor3d(double ux, double uy, double uz, double out[6]) {
  const ld u[3] = {ux, uy, uz};
  const ld s2 = u[0] * u[0] + u[1] * u[1] + u[2] * u[2];
  const ld s3 = s2 * sqrtl(s2);
  int k = 0;
  for (int a = 0; a < 3; a++)
    for (int b = a; b < 3; b++) out[k++] = (double)(((a == b ? s2 : 0.0L) - u[a] * u[b]) / s3);
}

void oracle_inner3d(long long n, const double *x, const double *y, const double *z, const double *wTD,
                    const double *wTKx, const double *wTKy, const double *wTKz, double *G, double *Gabs) {
#pragma omp parallel for schedule(dynamic, 16)
  for (long long i = 0; i < n; i++) {
    nsum_t acc[9], aac[9];
    memset(acc, 0, sizeof acc);
    memset(aac, 0, sizeof aac);
    for (long long j = 0; j < n; j++) {
      if (x[j] == x[i] && y[j] == y[i] && z[j] == z[i]) continue;
      const ld u[3] = {(ld)x[i] - x[j], (ld)y[i] - y[j], (ld)z[i] - z[j]};
      const ld s2 = u[0] * u[0] + u[1] * u[1] + u[2] * u[2];
      const ld s3 = s2 * sqrtl(s2);
      ld U[3][3];
      for (int a = 0; a < 3; a++)
        for (int b = 0; b < 3; b++) U[a][b] = ((a == b ? s2 : 0.0L) - u[a] * u[b]) / s3;
      const ld wd = wTD[j], wk[3] = {wTKx[j], wTKy[j], wTKz[j]};
      int k = 0;
      for (int a = 0; a < 3; a++)
        for (int b = a; b < 3; b++, k++) {
          nadd(&acc[k], wd * U[a][b]);
          nadd(&aac[k], fabsl(wd * U[a][b]));
        }
      for (int a = 0; a < 3; a++) {
        nadd(&acc[6 + a], U[a][0] * wk[0] + U[a][1] * wk[1] + U[a][2] * wk[2]);
        nadd(&aac[6 + a], fabsl(U[a][0] * wk[0]) + fabsl(U[a][1] * wk[1]) + fabsl(U[a][2] * wk[2]));
      }
    }
    for (int c = 0; c < 9; c++) {
      if (G) G[c * n + i] = (double)nval(&acc[c]);
      if (Gabs) Gabs[c * n + i] = (double)nval(&aac[c]);
    }
  }
}

/* ------------------------------------------------------------------------------------------ */
/* O1: FE space on the quadtree                                                                */
/* ------------------------------------------------------------------------------------------ */
static int pos_cmp(const void *a, const void *b) {
  const pos_t *x = (const pos_t *)a, *y = (const pos_t *)b;
  if (x->iz != y->iz) return x->iz < y->iz ? -1 : 1;
  if (x->ir != y->ir) return x->ir < y->ir ? -1 : 1;
  return 0;
}

static long long find_pos(const pos_t *arr, long long n, pos_t key) {
  long long lo = 0, hi = n - 1;
  while (lo <= hi) {
    long long mid = (lo + hi) / 2;
    int c = pos_cmp(&arr[mid], &key);
    if (c == 0) return mid;
    if (c < 0) lo = mid + 1;
    else hi = mid - 1;
  }
  return -1;
}

/* is position P on the closed boundary of cell c but not one of c's nodes?  If so return the
 * edge's p+1 node positions and the Lagrange weights of P along it. */
static int hanging_on(const grid_t *g, int c, int p, pos_t P, pos_t *mpos, ld *mw) {
  long long r0 = g->R0[c] * p, z0 = g->Z0[c] * p, H = g->H[c], L = g->H[c] * p;
  if (P.ir < r0 || P.ir > r0 + L || P.iz < z0 || P.iz > z0 + L) return 0;
  int onr = (P.ir == r0 || P.ir == r0 + L), onz = (P.iz == z0 || P.iz == z0 + L);
  if (!onr && !onz) return 0;
  if ((P.ir - r0) % H == 0 && (P.iz - z0) % H == 0) return 0; /* a node of c */
  ld t;
  if (onr) { /* vertical edge r = const, parametrised by z */
    t = (ld)(P.iz - z0) / (ld)L;
    for (int k = 0; k <= p; k++) { mpos[k].ir = P.ir; mpos[k].iz = z0 + k * H; }
  } else {
    t = (ld)(P.ir - r0) / (ld)L;
    for (int k = 0; k <= p; k++) { mpos[k].ir = r0 + k * H; mpos[k].iz = P.iz; }
  }
  for (int k = 0; k <= p; k++) mw[k] = lag(p, k, 2.0L * t - 1.0L);
  return 1;
}

/* resolve a node position into (dof, weight) terms, recursively through constraints */
static void resolve(const grid_t *g, int p, pos_t P, const pos_t *dofpos, int ndof, int depth,
                    ld scale, int *cnt, int *dofs, ld *wts, int cap) {
  long long k = find_pos(dofpos, ndof, P);
  if (k >= 0) {
    for (int i = 0; i < *cnt; i++)
      if (dofs[i] == (int)k) { wts[i] += scale; return; }
    if (*cnt < cap) { dofs[*cnt] = (int)k; wts[*cnt] = scale; (*cnt)++; }
    return;
  }
  if (depth > 8) return;
  pos_t mpos[8];
  ld mw[8];
  for (int c = 0; c < g->ncell; c++) {
    if (hanging_on(g, c, p, P, mpos, mw)) {
      for (int k2 = 0; k2 <= p; k2++)
        if (mw[k2] != 0.0L) resolve(g, p, mpos[k2], dofpos, ndof, depth + 1, scale * mw[k2], cnt, dofs, wts, cap);
      return;
    }
  }
}

static int int_cmp(const void *a, const void *b) {
  int x = *(const int *)a, y = *(const int *)b;
  return (x > y) - (x < y);
}

static int setup_grid(oracle_t *o, grid_t *g, char *err, int errlen) {
  int p = o->p, nb = o->nb;
  double hmin = 1e300;
  for (int c = 0; c < g->ncell; c++) {
    if (!(g->h[c] > 0.0) || g->r0[c] < 0.0) { snprintf(err, errlen, "bad cell %d", c); return -1; }
    if (g->h[c] < hmin) hmin = g->h[c];
  }
  g->R0 = malloc(sizeof(long long) * g->ncell);
  g->Z0 = malloc(sizeof(long long) * g->ncell);
  g->H = malloc(sizeof(long long) * g->ncell);
  for (int c = 0; c < g->ncell; c++) {
    double a = g->r0[c] / hmin, b = (g->z0[c] + g->R) / hmin, h = g->h[c] / hmin;
    g->R0[c] = llround(a);
    g->Z0[c] = llround(b);
    g->H[c] = llround(h);
    if (fabs(a - g->R0[c]) > 1e-6 || fabs(b - g->Z0[c]) > 1e-6 || fabs(h - g->H[c]) > 1e-6) {
      snprintf(err, errlen, "cell %d not on the quadtree lattice", c);
      return -1;
    }
  }
  /* all candidate node positions */
  long long ncand = (long long)g->ncell * nb;
  pos_t *cand = malloc(sizeof(pos_t) * ncand);
  for (int c = 0; c < g->ncell; c++)
    for (int b = 0; b <= p; b++)
      for (int a = 0; a <= p; a++) {
        pos_t P = {g->R0[c] * p + a * g->H[c], g->Z0[c] * p + b * g->H[c]};
        cand[(long long)c * nb + b * (p + 1) + a] = P;
      }
  pos_t *uniq = malloc(sizeof(pos_t) * ncand);
  memcpy(uniq, cand, sizeof(pos_t) * ncand);
  qsort(uniq, ncand, sizeof(pos_t), pos_cmp);
  long long nu = 0;
  for (long long i = 0; i < ncand; i++)
    if (nu == 0 || pos_cmp(&uniq[nu - 1], &uniq[i]) != 0) uniq[nu++] = uniq[i];
  /* a position is a DOF unless it hangs on some cell's edge */
  char *hang = calloc(nu, 1);
#pragma omp parallel for schedule(dynamic, 64)
  for (long long i = 0; i < nu; i++) {
    pos_t mpos[8];
    ld mw[8];
    for (int c = 0; c < g->ncell; c++)
      if (hanging_on(g, c, p, uniq[i], mpos, mw)) { hang[i] = 1; break; }
  }
  g->ndof = 0;
  for (long long i = 0; i < nu; i++)
    if (!hang[i]) g->ndof++;
  g->node_pos = malloc(sizeof(pos_t) * g->ndof);
  g->node_r = malloc(sizeof(double) * g->ndof);
  g->node_z = malloc(sizeof(double) * g->ndof);
  long long k = 0;
  ld unit = (ld)hmin / p;
  for (long long i = 0; i < nu; i++)
    if (!hang[i]) {
      g->node_pos[k] = uniq[i];
      g->node_r[k] = (double)(uniq[i].ir * unit);
      g->node_z[k] = (double)(uniq[i].iz * unit - (ld)g->R);
      k++;
    }
  free(hang);
  free(uniq);
  /* per cell extraction */
  g->ne = malloc(sizeof(int) * g->ncell);
  g->edofs = malloc(sizeof(int *) * g->ncell);
  g->P = malloc(sizeof(ld *) * g->ncell);
  int cap = 64;
  for (int c = 0; c < g->ncell; c++) {
    int *ld_cnt = calloc(nb, sizeof(int));
    int *ld_dof = malloc(sizeof(int) * nb * cap);
    ld *ld_w = malloc(sizeof(ld) * nb * cap);
    int tot = 0;
    for (int a = 0; a < nb; a++) {
      resolve(g, p, cand[(long long)c * nb + a], g->node_pos, g->ndof, 0, 1.0L, &ld_cnt[a],
              ld_dof + a * cap, ld_w + a * cap, cap);
      if (ld_cnt[a] == 0) { snprintf(err, errlen, "unresolvable node in cell %d", c); return -1; }
      tot += ld_cnt[a];
    }
    int *all = malloc(sizeof(int) * tot);
    int t = 0;
    for (int a = 0; a < nb; a++)
      for (int i = 0; i < ld_cnt[a]; i++) all[t++] = ld_dof[a * cap + i];
    qsort(all, tot, sizeof(int), int_cmp);
    int n = 0;
    for (int i = 0; i < tot; i++)
      if (n == 0 || all[n - 1] != all[i]) all[n++] = all[i];
    g->ne[c] = n;
    g->edofs[c] = all;
    g->P[c] = calloc((size_t)nb * n, sizeof(ld));
    for (int a = 0; a < nb; a++)
      for (int i = 0; i < ld_cnt[a]; i++) {
        int d = ld_dof[a * cap + i];
        int col = -1;
        for (int j = 0; j < n; j++)
          if (all[j] == d) { col = j; break; }
        g->P[c][a * n + col] += ld_w[a * cap + i];
      }
    free(ld_cnt);
    free(ld_dof);
    free(ld_w);
  }
  free(cand);
  /* CSR pattern: union over cells of edofs x edofs */
  int *rcnt = calloc(g->ndof, sizeof(int));
  for (int c = 0; c < g->ncell; c++)
    for (int i = 0; i < g->ne[c]; i++) rcnt[g->edofs[c][i]] += g->ne[c];
  long long *off = malloc(sizeof(long long) * (g->ndof + 1));
  off[0] = 0;
  for (int i = 0; i < g->ndof; i++) off[i + 1] = off[i] + rcnt[i];
  int *tmp = malloc(sizeof(int) * (off[g->ndof] ? off[g->ndof] : 1));
  memset(rcnt, 0, sizeof(int) * g->ndof);
  for (int c = 0; c < g->ncell; c++)
    for (int i = 0; i < g->ne[c]; i++) {
      int row = g->edofs[c][i];
      for (int j = 0; j < g->ne[c]; j++) tmp[off[row] + rcnt[row]++] = g->edofs[c][j];
    }
  g->rowptr = malloc(sizeof(long long) * (g->ndof + 1));
  g->rowptr[0] = 0;
  for (int i = 0; i < g->ndof; i++) {
    int *seg = tmp + off[i];
    int n = rcnt[i];
    qsort(seg, n, sizeof(int), int_cmp);
    int u = 0;
    for (int j = 0; j < n; j++)
      if (u == 0 || seg[u - 1] != seg[j]) seg[u++] = seg[j];
    g->rowptr[i + 1] = g->rowptr[i] + u;
  }
  g->nnz = g->rowptr[g->ndof];
  g->col = malloc(sizeof(int) * (g->nnz ? g->nnz : 1));
  for (int i = 0; i < g->ndof; i++) {
    long long u = g->rowptr[i + 1] - g->rowptr[i];
    memcpy(g->col + g->rowptr[i], tmp + off[i], sizeof(int) * u);
  }
  free(tmp);
  free(off);
  free(rcnt);
  return 0;
}

/* 2:1 balance across edges (Amb-10): neighbours sharing an edge segment differ by <= one level */
static int check_balance(const grid_t *g) {
  for (int a = 0; a < g->ncell; a++)
    for (int b = 0; b < g->ncell; b++) {
      if (a == b) continue;
      long long ar0 = g->R0[a], ar1 = ar0 + g->H[a], az0 = g->Z0[a], az1 = az0 + g->H[a];
      long long br0 = g->R0[b], br1 = br0 + g->H[b], bz0 = g->Z0[b], bz1 = bz0 + g->H[b];
      /* overlap of interiors */
      if (ar0 < br1 && br0 < ar1 && az0 < bz1 && bz0 < az1) return -1;
      int share = 0;
      if ((ar1 == br0 || br1 == ar0) && az0 < bz1 && bz0 < az1) share = 1;
      if ((az1 == bz0 || bz1 == az0) && ar0 < br1 && br0 < ar1) share = 1;
      if (share && (g->H[a] > 2 * g->H[b] || g->H[b] > 2 * g->H[a])) return -2;
    }
  return 0;
}

oracle_t *oracle_create(int ngrids, const long long *ncells, const double *cells, const double *radius,
                        int order, int nq1d, int nspecies, const double *mass, const double *charge,
                        const int *grid, double nu, char *err, int errlen) {
  if (order < 1 || order > 6 || ngrids < 1 || nspecies < 1) {
    snprintf(err, errlen, "bad order/ngrids/nspecies");
    return NULL;
  }
  oracle_t *o = calloc(1, sizeof(oracle_t));
  o->ngrids = ngrids;
  o->p = order;
  o->nq = nq1d > 0 ? nq1d : order + 1;
  o->nb = (order + 1) * (order + 1);
  o->nqp = o->nq * o->nq;
  o->S = nspecies;
  o->nu = nu;
  o->mass = malloc(sizeof(double) * nspecies);
  o->charge = malloc(sizeof(double) * nspecies);
  o->sgrid = malloc(sizeof(int) * nspecies);
  for (int a = 0; a < nspecies; a++) {
    if (!(mass[a] > 0.0) || grid[a] < 0 || grid[a] >= ngrids) {
      snprintf(err, errlen, "bad species %d", a);
      return NULL;
    }
    o->mass[a] = mass[a];
    o->charge[a] = charge[a];
    o->sgrid[a] = grid[a];
  }
  /* reference tables (O1, O2) */
  int p = o->p, nq = o->nq, nb = o->nb, nqp = o->nqp;
  o->xq = malloc(sizeof(ld) * nq);
  o->wq = malloc(sizeof(ld) * nq);
  gauss_legendre(nq, o->xq, o->wq);
  o->phi = malloc(sizeof(ld) * nqp * nb);
  o->dxi = malloc(sizeof(ld) * nqp * nb);
  o->deta = malloc(sizeof(ld) * nqp * nb);
  for (int qb = 0; qb < nq; qb++)
    for (int qa = 0; qa < nq; qa++)
      for (int b = 0; b <= p; b++)
        for (int a = 0; a <= p; a++) {
          int q = qb * nq + qa, n = b * (p + 1) + a;
          o->phi[q * nb + n] = lag(p, a, o->xq[qa]) * lag(p, b, o->xq[qb]);
          o->dxi[q * nb + n] = dlag(p, a, o->xq[qa]) * lag(p, b, o->xq[qb]);
          o->deta[q * nb + n] = lag(p, a, o->xq[qa]) * dlag(p, b, o->xq[qb]);
        }
  o->g = calloc(ngrids, sizeof(grid_t));
  long long c0 = 0, pt0 = 0;
  for (int gi = 0; gi < ngrids; gi++) {
    grid_t *g = &o->g[gi];
    g->ncell = (int)ncells[gi];
    g->cell0 = c0;
    g->R = radius[gi];
    g->r0 = malloc(sizeof(double) * g->ncell);
    g->z0 = malloc(sizeof(double) * g->ncell);
    g->h = malloc(sizeof(double) * g->ncell);
    for (int c = 0; c < g->ncell; c++) {
      g->r0[c] = cells[3 * (c0 + c) + 0];
      g->z0[c] = cells[3 * (c0 + c) + 1];
      g->h[c] = cells[3 * (c0 + c) + 2];
    }
    if (setup_grid(o, g, err, errlen)) return NULL;
    int bal = check_balance(g);
    if (bal) {
      snprintf(err, errlen, bal == -1 ? "overlapping cells" : "quadtree not 2:1 balanced");
      return NULL;
    }
    g->npts = (long long)g->ncell * nqp;
    g->pt0 = pt0;
    pt0 += g->npts;
    c0 += g->ncell;
  }
  o->npts = pt0;
  o->pr = malloc(sizeof(double) * o->npts);
  o->pz = malloc(sizeof(double) * o->npts);
  o->pw = malloc(sizeof(double) * o->npts);
  o->pgrid = malloc(sizeof(int) * o->npts);
  for (int gi = 0; gi < ngrids; gi++) {
    grid_t *g = &o->g[gi];
    for (int c = 0; c < g->ncell; c++) {
      ld hh = g->h[c];
      for (int qb = 0; qb < nq; qb++)
        for (int qa = 0; qa < nq; qa++) {
          long long k = g->pt0 + (long long)c * nqp + qb * nq + qa;
          ld r = g->r0[c] + hh * (o->xq[qa] + 1.0L) / 2.0L;
          ld z = g->z0[c] + hh * (o->xq[qb] + 1.0L) / 2.0L;
          o->pr[k] = (double)r;
          o->pz[k] = (double)z;
          o->pw[k] = (double)(o->wq[qa] * o->wq[qb] * (hh / 2.0L) * (hh / 2.0L) * r);
          o->pgrid[k] = gi;
        }
    }
  }
  o->soff = malloc(sizeof(long long) * (nspecies + 1));
  o->snnz_off = malloc(sizeof(long long) * (nspecies + 1));
  o->scoo_off = malloc(sizeof(long long) * (nspecies + 1));
  o->soff[0] = o->snnz_off[0] = o->scoo_off[0] = 0;
  for (int a = 0; a < nspecies; a++) {
    grid_t *g = &o->g[o->sgrid[a]];
    long long nc = 0;
    for (int c = 0; c < g->ncell; c++) nc += (long long)g->ne[c] * g->ne[c];
    o->soff[a + 1] = o->soff[a] + g->ndof;
    o->snnz_off[a + 1] = o->snnz_off[a] + g->nnz;
    o->scoo_off[a + 1] = o->scoo_off[a] + nc;
  }
  o->ndof = o->soff[nspecies];
  o->nnz = o->snnz_off[nspecies];
  o->ncoo = o->scoo_off[nspecies];
  return o;
}

void oracle_destroy(oracle_t *o) {
  if (!o) return;
  for (int gi = 0; gi < o->ngrids; gi++) {
    grid_t *g = &o->g[gi];
    for (int c = 0; c < g->ncell; c++) {
      free(g->edofs ? g->edofs[c] : NULL);
      free(g->P ? g->P[c] : NULL);
    }
    free(g->edofs); free(g->P); free(g->ne);
    free(g->r0); free(g->z0); free(g->h); free(g->R0); free(g->Z0); free(g->H);
    free(g->node_pos); free(g->node_r); free(g->node_z); free(g->rowptr); free(g->col);
  }
  free(o->g); free(o->mass); free(o->charge); free(o->sgrid);
  free(o->soff); free(o->snnz_off); free(o->scoo_off);
  free(o->xq); free(o->wq); free(o->phi); free(o->dxi); free(o->deta);
  free(o->pr); free(o->pz); free(o->pw); free(o->pgrid);
  free(o);
}

void oracle_sizes(const oracle_t *o, long long *ndof, long long *npoints, long long *nnz, long long *ncoo) {
  if (ndof) *ndof = o->ndof;
  if (npoints) *npoints = o->npts;
  if (nnz) *nnz = o->nnz;
  if (ncoo) *ncoo = o->ncoo;
}
long long oracle_grid_ndof(const oracle_t *o, int g) { return o->g[g].ndof; }
long long oracle_grid_npoints(const oracle_t *o, int g) { return o->g[g].npts; }
void oracle_grid_nodes(const oracle_t *o, int g, double *r, double *z) {
  memcpy(r, o->g[g].node_r, sizeof(double) * o->g[g].ndof);
  memcpy(z, o->g[g].node_z, sizeof(double) * o->g[g].ndof);
}
void oracle_points(const oracle_t *o, double *r, double *z, double *w) {
  memcpy(r, o->pr, sizeof(double) * o->npts);
  memcpy(z, o->pz, sizeof(double) * o->npts);
  memcpy(w, o->pw, sizeof(double) * o->npts);
}
void oracle_pattern(const oracle_t *o, long long *rowptr, int *col) {
  long long r = 0;
  rowptr[0] = 0;
  for (int a = 0; a < o->S; a++) {
    const grid_t *g = &o->g[o->sgrid[a]];
    for (int i = 0; i < g->ndof; i++, r++) {
      rowptr[r + 1] = rowptr[r] + (g->rowptr[i + 1] - g->rowptr[i]);
      for (long long k = g->rowptr[i]; k < g->rowptr[i + 1]; k++)
        col[rowptr[r] + (k - g->rowptr[i])] = (int)(o->soff[a] + g->col[k]);
    }
  }
}
void oracle_coo_pattern(const oracle_t *o, int *row, int *col) {
  long long k = 0;
  for (int a = 0; a < o->S; a++) {
    const grid_t *g = &o->g[o->sgrid[a]];
    for (int c = 0; c < g->ncell; c++)
      for (int i = 0; i < g->ne[c]; i++)
        for (int j = 0; j < g->ne[c]; j++, k++) {
          row[k] = (int)(o->soff[a] + g->edofs[c][i]);
          col[k] = (int)(o->soff[a] + g->edofs[c][j]);
        }
  }
}

/* ------------------------------------------------------------------------------------------ */
/* O3, O4: point fields                                                                        */
/* ------------------------------------------------------------------------------------------ */
/* T_D, T_K (and their absolute-value counterparts) at every point */
static void point_fields_ld(const oracle_t *o, const double *f, ld *TD, ld *TKr, ld *TKz, ld *TDa,
                            ld *TKra, ld *TKza) {
  int nb = o->nb, nqp = o->nqp;
  for (int gi = 0; gi < o->ngrids; gi++) {
    const grid_t *g = &o->g[gi];
#pragma omp parallel for schedule(static)
    for (int c = 0; c < g->ncell; c++) {
      int n = g->ne[c];
      ld fe[64], fea[64];
      for (int q = 0; q < nqp; q++) {
        long long k = g->pt0 + (long long)c * nqp + q;
        TD[k] = TKr[k] = TKz[k] = TDa[k] = TKra[k] = TKza[k] = 0.0L;
      }
      for (int a = 0; a < o->S; a++) {
        if (o->sgrid[a] != gi) continue;
        ld e2 = (ld)o->charge[a] * (ld)o->charge[a];
        ld im = 1.0L / (ld)o->mass[a]; /* m0 / m_a, m0 = m_e */
        /* element coefficients (extraction P_e) */
        for (int b = 0; b < nb; b++) {
          fe[b] = fea[b] = 0.0L;
          for (int j = 0; j < n; j++) {
            ld pv = g->P[c][b * n + j];
            ld fv = f[o->soff[a] + g->edofs[c][j]];
            fe[b] += pv * fv;
            fea[b] += fabsl(pv) * fabsl(fv);
          }
        }
        ld s = 2.0L / (ld)g->h[c];
        for (int q = 0; q < nqp; q++) {
          ld fv = 0, dr = 0, dz = 0, fa = 0, dra = 0, dza = 0;
          for (int b = 0; b < nb; b++) {
            fv += o->phi[q * nb + b] * fe[b];
            dr += s * o->dxi[q * nb + b] * fe[b];
            dz += s * o->deta[q * nb + b] * fe[b];
            fa += fabsl(o->phi[q * nb + b]) * fea[b];
            dra += s * fabsl(o->dxi[q * nb + b]) * fea[b];
            dza += s * fabsl(o->deta[q * nb + b]) * fea[b];
          }
          long long k = g->pt0 + (long long)c * nqp + q;
          TD[k] += e2 * fv;
          TKr[k] += e2 * im * dr;
          TKz[k] += e2 * im * dz;
          TDa[k] += e2 * fa;
          TKra[k] += e2 * im * dra;
          TKza[k] += e2 * im * dza;
        }
      }
    }
  }
}

void oracle_point_fields(const oracle_t *o, const double *f, double *TD, double *TKr, double *TKz) {
  long long N = o->npts;
  ld *b = malloc(sizeof(ld) * N * 6);
  point_fields_ld(o, f, b, b + N, b + 2 * N, b + 3 * N, b + 4 * N, b + 5 * N);
  for (long long k = 0; k < N; k++) {
    TD[k] = (double)b[k];
    TKr[k] = (double)b[N + k];
    TKz[k] = (double)b[2 * N + k];
  }
  free(b);
}

/* O5 at targets, including the |.| version driven by |T| */
static void coeffs_ld(const oracle_t *o, const double *f, long long nt, const long long *targets, ld *G,
                      ld *Ga) {
  long long N = o->npts;
  ld *b = malloc(sizeof(ld) * N * 6);
  point_fields_ld(o, f, b, b + N, b + 2 * N, b + 3 * N, b + 4 * N, b + 5 * N);
  double *TD = malloc(sizeof(double) * N * 6);
  double *TKr = TD + N, *TKz = TD + 2 * N, *TDa = TD + 3 * N, *TKra = TD + 4 * N, *TKza = TD + 5 * N;
  for (long long k = 0; k < 6 * N; k++) TD[k] = (double)b[k];
  free(b);
#pragma omp parallel for schedule(dynamic, 4)
  for (long long t = 0; t < nt; t++) {
    long long i = targets ? targets[t] : t;
    ld g[5], ga[5], g2[5], ga2[5];
    inner_one(N, o->pr, o->pz, o->pw, TD, TKr, TKz, i, g, ga);
    inner_one(N, o->pr, o->pz, o->pw, TDa, TKra, TKza, i, g2, ga2);
    (void)g2;
    for (int c = 0; c < 5; c++) {
      G[c * nt + t] = g[c];
      Ga[c * nt + t] = ga2[c]; /* sum |w| |T|^abs |U| */
    }
  }
  free(TD);
}

void oracle_point_coeffs(const oracle_t *o, const double *f, long long nt, const long long *targets,
                         double *G, double *Gabs) {
  ld *g = malloc(sizeof(ld) * 10 * nt);
  coeffs_ld(o, f, nt, targets, g, g + 5 * nt);
  for (long long k = 0; k < 5 * nt; k++) {
    if (G) G[k] = (double)g[k];
    if (Gabs) Gabs[k] = (double)g[5 * nt + k];
  }
  free(g);
}

/* ------------------------------------------------------------------------------------------ */
/* O6-O8                                                                                       */
/* ------------------------------------------------------------------------------------------ */
/* element matrix of species a on cell c of grid g from the point coefficients of that cell.
 * Gc[5][nqp], Gac[5][nqp]; C[nb][nb] (k = test row, l = trial column), Ca = |.| version. */
static void element_matrix(const oracle_t *o, int a, const grid_t *g, int c, const ld *Gc, const ld *Gac,
                           ld *C, ld *Ca) {
  int nb = o->nb, nqp = o->nqp;
  ld e2 = (ld)o->charge[a] * (ld)o->charge[a], im = 1.0L / (ld)o->mass[a], nu = o->nu;
  ld fD = -nu * e2 * im * im; /* D~ = -nu e^2 (m0/m)^2 G_D */
  ld fK = nu * e2 * im;       /* K~ =  nu e^2 (m0/m) G_K   */
  ld s = 2.0L / (ld)g->h[c];
  for (int k = 0; k < nb * nb; k++) C[k] = Ca[k] = 0.0L;
  for (int q = 0; q < nqp; q++) {
    long long pk = g->pt0 + (long long)c * nqp + q;
    ld w = o->pw[pk];
    ld Drr = fD * Gc[0 * nqp + q], Drz = fD * Gc[1 * nqp + q], Dzz = fD * Gc[2 * nqp + q];
    ld Kr = fK * Gc[3 * nqp + q], Kz = fK * Gc[4 * nqp + q];
    ld aD = fabsl(fD), aK = fabsl(fK);
    ld Arr = aD * Gac[0 * nqp + q], Arz = aD * Gac[1 * nqp + q], Azz = aD * Gac[2 * nqp + q];
    ld AKr = aK * Gac[3 * nqp + q], AKz = aK * Gac[4 * nqp + q];
    for (int k = 0; k < nb; k++) {
      ld gkr = s * o->dxi[q * nb + k], gkz = s * o->deta[q * nb + k];
      for (int l = 0; l < nb; l++) {
        ld glr = s * o->dxi[q * nb + l], glz = s * o->deta[q * nb + l], pl = o->phi[q * nb + l];
        ld v = gkr * (Drr * glr + Drz * glz) + gkz * (Drz * glr + Dzz * glz) + (gkr * Kr + gkz * Kz) * pl;
        ld va = fabsl(gkr) * (Arr * fabsl(glr) + Arz * fabsl(glz)) + fabsl(gkz) * (Arz * fabsl(glr) + Azz * fabsl(glz)) +
                (fabsl(gkr) * AKr + fabsl(gkz) * AKz) * fabsl(pl);
        C[k * nb + l] += w * v;
        Ca[k * nb + l] += fabsl(w) * va;
      }
    }
  }
}

/* P_e^T C P_e (n_e x n_e) */
static void expand(const oracle_t *o, const grid_t *g, int c, const ld *C, const ld *Ca, ld *X, ld *Xa) {
  int nb = o->nb, n = g->ne[c];
  const ld *P = g->P[c];
  for (int i = 0; i < n * n; i++) X[i] = Xa[i] = 0.0L;
  for (int k = 0; k < nb; k++)
    for (int l = 0; l < nb; l++) {
      ld v = C[k * nb + l], va = Ca[k * nb + l];
      if (v == 0.0L && va == 0.0L) continue;
      for (int i = 0; i < n; i++) {
        ld pk = P[k * n + i];
        if (pk == 0.0L) continue;
        for (int j = 0; j < n; j++) {
          ld pl = P[l * n + j];
          if (pl == 0.0L) continue;
          X[i * n + j] += pk * v * pl;
          Xa[i * n + j] += fabsl(pk) * va * fabsl(pl);
        }
      }
    }
}

static long long csr_find(const grid_t *g, int row, int col) {
  long long lo = g->rowptr[row], hi = g->rowptr[row + 1] - 1;
  while (lo <= hi) {
    long long mid = (lo + hi) / 2;
    if (g->col[mid] == col) return mid;
    if (g->col[mid] < col) lo = mid + 1;
    else hi = mid - 1;
  }
  return -1;
}

/* shared driver: computes G at the points of the selected cells, then element matrices, then
 * either CSR assembly or COO output */
static void jacobian_driver(const oracle_t *o, const double *f, const unsigned char *mask, double *vals,
                            double *absvals, int coo) {
  int nqp = o->nqp, nb = o->nb;
  /* targets = points of selected cells */
  long long nt = 0;
  long long *tg = malloc(sizeof(long long) * o->npts);
  for (int gi = 0; gi < o->ngrids; gi++) {
    const grid_t *g = &o->g[gi];
    for (int c = 0; c < g->ncell; c++)
      if (!mask || mask[g->cell0 + c])
        for (int q = 0; q < nqp; q++) tg[nt++] = g->pt0 + (long long)c * nqp + q;
  }
  ld *G = malloc(sizeof(ld) * 10 * (nt ? nt : 1));
  coeffs_ld(o, f, nt, tg, G, G + 5 * nt);
  long long *where = malloc(sizeof(long long) * o->npts);
  for (long long k = 0; k < o->npts; k++) where[k] = -1;
  for (long long t = 0; t < nt; t++) where[tg[t]] = t;
  if (!coo) {
    for (long long k = 0; k < o->nnz; k++) vals[k] = absvals[k] = 0.0;
  }
  for (int a = 0; a < o->S; a++) {
    const grid_t *g = &o->g[o->sgrid[a]];
    ld *acc = NULL, *acca = NULL;
    if (!coo) {
      acc = calloc(g->nnz ? g->nnz : 1, sizeof(ld));
      acca = calloc(g->nnz ? g->nnz : 1, sizeof(ld));
    }
    long long coff = o->scoo_off[a];
    for (int c = 0; c < g->ncell; c++) {
      int n = g->ne[c];
      if (mask && !mask[g->cell0 + c]) { coff += (long long)n * n; continue; }
      ld Gc[5 * 64], Gac[5 * 64];
      for (int q = 0; q < nqp; q++) {
        long long t = where[g->pt0 + (long long)c * nqp + q];
        for (int cc = 0; cc < 5; cc++) {
          Gc[cc * nqp + q] = G[cc * nt + t];
          Gac[cc * nqp + q] = G[5 * nt + cc * nt + t];
        }
      }
      ld *C = malloc(sizeof(ld) * nb * nb * 2);
      ld *X = malloc(sizeof(ld) * n * n * 2);
      element_matrix(o, a, g, c, Gc, Gac, C, C + nb * nb);
      expand(o, g, c, C, C + nb * nb, X, X + n * n);
      for (int i = 0; i < n; i++)
        for (int j = 0; j < n; j++) {
          if (coo) {
            vals[coff + i * n + j] = (double)X[i * n + j];
            absvals[coff + i * n + j] = (double)X[n * n + i * n + j];
          } else {
            long long k = csr_find(g, g->edofs[c][i], g->edofs[c][j]);
            acc[k] += X[i * n + j];
            acca[k] += X[n * n + i * n + j];
          }
        }
      coff += (long long)n * n;
      free(C);
      free(X);
    }
    if (!coo) {
      for (long long k = 0; k < g->nnz; k++) {
        vals[o->snnz_off[a] + k] = (double)acc[k];
        absvals[o->snnz_off[a] + k] = (double)acca[k];
      }
      free(acc);
      free(acca);
    }
  }
  free(where);
  free(G);
  free(tg);
}

void oracle_jacobian(const oracle_t *o, const double *f, double *vals, double *absvals) {
  jacobian_driver(o, f, NULL, vals, absvals, 0);
}
void oracle_jacobian_coo(const oracle_t *o, const double *f, const unsigned char *mask, double *vals,
                         double *absvals) {
  jacobian_driver(o, f, mask, vals, absvals, 1);
}

/* O9: mass, sum_q w phi_k phi_l (kind 0); O11: E_z advection, sum_q w phi_k d_z phi_l (kind 1) --
 * the element matrix of Eq. 4's (0, e E_z / m) . grad f term tested with psi = phi_k, before the
 * species factor e_a E_z / m_a (@8216-8654; same w = w_hat detJ r as the mass, Amb-2) */
static void mass_driver(const oracle_t *o, double shift, double *vals, int coo, int kind) {
  int nqp = o->nqp, nb = o->nb;
  if (!coo)
    for (long long k = 0; k < o->nnz; k++) vals[k] = 0.0;
  for (int a = 0; a < o->S; a++) {
    const grid_t *g = &o->g[o->sgrid[a]];
    ld *acc = coo ? NULL : calloc(g->nnz ? g->nnz : 1, sizeof(ld));
    long long coff = o->scoo_off[a];
    for (int c = 0; c < g->ncell; c++) {
      int n = g->ne[c];
      ld s = 2.0L / (ld)g->h[c];
      ld *M = calloc((size_t)nb * nb, sizeof(ld));
      for (int q = 0; q < nqp; q++) {
        ld w = o->pw[g->pt0 + (long long)c * nqp + q];
        for (int k = 0; k < nb; k++)
          for (int l = 0; l < nb; l++)
            M[k * nb + l] += w * o->phi[q * nb + k] * (kind == 0 ? o->phi[q * nb + l] : s * o->deta[q * nb + l]);
      }
      ld *X = calloc((size_t)n * n * 2, sizeof(ld));
      expand(o, g, c, M, M, X, X + n * n);
      for (int i = 0; i < n; i++)
        for (int j = 0; j < n; j++) {
          ld v = (ld)shift * X[i * n + j];
          if (coo) vals[coff + i * n + j] = (double)v;
          else acc[csr_find(g, g->edofs[c][i], g->edofs[c][j])] += v;
        }
      coff += (long long)n * n;
      free(M);
      free(X);
    }
    if (!coo) {
      for (long long k = 0; k < g->nnz; k++) vals[o->snnz_off[a] + k] = (double)acc[k];
      free(acc);
    }
  }
}
void oracle_mass(const oracle_t *o, double shift, double *vals) { mass_driver(o, shift, vals, 0, 0); }
void oracle_mass_coo(const oracle_t *o, double shift, double *vals) { mass_driver(o, shift, vals, 1, 0); }
void oracle_advection(const oracle_t *o, double *vals) { mass_driver(o, 1.0, vals, 0, 1); }
void oracle_advection_coo(const oracle_t *o, double *vals) { mass_driver(o, 1.0, vals, 1, 1); }

void oracle_set_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}
int oracle_get_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* ------------------------------------------------------------------------------------------ */
/* O13 (SURVEY §8(f) NEXT-4 completed: "a full 3D model is supported in the library"           */
/* @7997-8072): the Landau Jacobian in 3D Cartesian velocity space -- O1-O8 and O10 with the    */
/* tensor of O12, on a uniform grid of ncell^3 Q_p cubes over [-R, R]^3 (no hanging nodes, no   */
/* r weight: the Cartesian weak form of Eq. 4 @8216-8560 is int psi ... dv over R^3):           */
/*   DOFs   the lattice of M = ncell p + 1 equispaced nodes per direction,                      */
/*          dof(ix, iy, iz) = (iz M + iy) M + ix at (-R + ix h/p, -R + iy h/p, -R + iz h/p)      */
/*   points (p+1)^3 Gauss-Legendre points per cube, w = w_a w_b w_c (h/2)^3                     */
/*   O3/O4  T_D = sum_b e_b^2 f_b, T_K = sum_b e_b^2 (m0/m_b) grad f_b at every point            */
/*   O12    G_D(i) = sum_{j: v_j != v_i} w_j T_D(j) U(v_i - v_j), G_K(i) = sum_j U w_j T_K(j)      */
/*   O6/O7  C_e[k][l] = sum_q w_q (grad phi_k . D~ grad phi_l + (grad phi_k . K~) phi_l),       */
/*          D~ = -nu e_a^2 (m0/m_a)^2 G_D, K~ = nu e_a^2 (m0/m_a) G_K (the forms of Eqs. 5-6)    */
/*   O8     J_a = sum_e C_e added at (dof_k, dof_l), species-block-diagonal, CSR rows sorted      */
/*   O10    the same with every product in absolute value (fields from |phi| |f|)               */
/* ------------------------------------------------------------------------------------------ */
/* 1D: the lattice indices sharing a cube with lattice index i: [lo, hi] */
static void o3_range(int ncell, int p, long long i, long long *lo, long long *hi) {
  long long c0 = i / p, c1 = c0;
  if (i % p == 0 && c0 > 0) c0--;  /* a cube boundary node belongs to the cubes on both sides */
  if (c1 >= ncell) c1 = ncell - 1;
  *lo = c0 * p;
  *hi = (c1 + 1) * p;
}

void oracle3d_sizes(int ncell, int order, long long *ndof, long long *npoints, long long *nnz) {
  long long M = (long long)ncell * order + 1, s = 0;
  for (long long i = 0; i < M; i++) {
    long long lo, hi;
    o3_range(ncell, order, i, &lo, &hi);
    s += hi - lo + 1;
  }
  if (ndof) *ndof = M * M * M;
  if (npoints) *npoints = (long long)ncell * ncell * ncell * (order + 1) * (order + 1) * (order + 1);
  if (nnz) *nnz = s * s * s; /* the pattern is the tensor product of the 1D ones */
}

void oracle3d_pattern(int ncell, int order, long long *rowptr, int *col) {
  long long M = (long long)ncell * order + 1, k = 0;
  rowptr[0] = 0;
  for (long long iz = 0; iz < M; iz++)
    for (long long iy = 0; iy < M; iy++)
      for (long long ix = 0; ix < M; ix++) {
        long long lx, hx, ly, hy, lz, hz;
        o3_range(ncell, order, ix, &lx, &hx);
        o3_range(ncell, order, iy, &ly, &hy);
        o3_range(ncell, order, iz, &lz, &hz);
        for (long long jz = lz; jz <= hz; jz++)
          for (long long jy = ly; jy <= hy; jy++)
            for (long long jx = lx; jx <= hx; jx++) col[k++] = (int)((jz * M + jy) * M + jx);
        rowptr[(iz * M + iy) * M + ix + 1] = k;
      }
}

void oracle3d_nodes(int ncell, int order, double R, double *xyz) {
  long long M = (long long)ncell * order + 1, nd = M * M * M;
  ld d = 2.0L * (ld)R / ((ld)ncell * order);
  for (long long iz = 0; iz < M; iz++)
    for (long long iy = 0; iy < M; iy++)
      for (long long ix = 0; ix < M; ix++) {
        long long k = (iz * M + iy) * M + ix;
        xyz[k] = (double)(-(ld)R + ix * d);
        xyz[nd + k] = (double)(-(ld)R + iy * d);
        xyz[2 * nd + k] = (double)(-(ld)R + iz * d);
      }
}

static long long o3_find(const long long *rowptr, const int *col, long long row, int c) {
  long long lo = rowptr[row], hi = rowptr[row + 1] - 1;
  while (lo <= hi) {
    long long mid = (lo + hi) / 2;
    if (col[mid] == c) return mid;
    if (col[mid] < c) lo = mid + 1;
    else hi = mid - 1;
  }
  return -1;
}

/* the grid: points (coordinates, weights), reference basis at the Gauss points, cube DOFs */
typedef struct {
  int p, s1, nb, nq, ncell;
  long long M, nc3, ndof, N, nnz;
  ld h, s; /* cube side, 2 / h */
  double *x, *y, *z;
  ld *w;
  ld *bas;        /* [q][n][phi, d/dx, d/dy, d/dz] (physical gradients) */
  long long *dofs; /* [cube][nb] */
} o3grid_t;

static void o3_grid(int ncell, int order, double R, o3grid_t *g) {
  const int p = order, s1 = p + 1, nb = s1 * s1 * s1;
  g->p = p;
  g->s1 = s1;
  g->nb = nb;
  g->nq = nb;
  g->ncell = ncell;
  g->M = (long long)ncell * p + 1;
  g->nc3 = (long long)ncell * ncell * ncell;
  oracle3d_sizes(ncell, order, &g->ndof, &g->N, &g->nnz);
  g->h = 2.0L * (ld)R / ncell;
  g->s = 2.0L / g->h;
  ld xg[8], wg[8];
  gauss_legendre(s1, xg, wg);
  g->x = malloc(sizeof(double) * 3 * g->N);
  g->y = g->x + g->N;
  g->z = g->x + 2 * g->N;
  g->w = malloc(sizeof(ld) * g->N);
  g->bas = malloc(sizeof(ld) * 4 * (size_t)nb * nb);
  g->dofs = malloc(sizeof(long long) * g->nc3 * nb);
  for (int qa = 0; qa < s1; qa++) /* Gauss index along z, y, x */
    for (int qb = 0; qb < s1; qb++)
      for (int qc = 0; qc < s1; qc++) {
        int q = (qa * s1 + qb) * s1 + qc;
        for (int k = 0; k < s1; k++)
          for (int j = 0; j < s1; j++)
            for (int i = 0; i < s1; i++) {
              int n = (k * s1 + j) * s1 + i;
              ld Lx = lag(p, i, xg[qc]), Ly = lag(p, j, xg[qb]), Lz = lag(p, k, xg[qa]);
              ld *b = g->bas + 4 * ((size_t)q * nb + n);
              b[0] = Lx * Ly * Lz;
              b[1] = g->s * dlag(p, i, xg[qc]) * Ly * Lz;
              b[2] = g->s * Lx * dlag(p, j, xg[qb]) * Lz;
              b[3] = g->s * Lx * Ly * dlag(p, k, xg[qa]);
            }
      }
  for (long long cz = 0; cz < ncell; cz++)
    for (long long cy = 0; cy < ncell; cy++)
      for (long long cx = 0; cx < ncell; cx++) {
        long long c = (cz * ncell + cy) * ncell + cx;
        for (int k = 0; k < s1; k++)
          for (int j = 0; j < s1; j++)
            for (int i = 0; i < s1; i++)
              g->dofs[c * nb + (k * s1 + j) * s1 + i] = ((cz * p + k) * g->M + (cy * p + j)) * g->M + (cx * p + i);
        for (int qa = 0; qa < s1; qa++)
          for (int qb = 0; qb < s1; qb++)
            for (int qc = 0; qc < s1; qc++) {
              long long pt = c * g->nq + (qa * s1 + qb) * s1 + qc;
              g->x[pt] = (double)(-(ld)R + g->h * cx + 0.5L * g->h * (xg[qc] + 1.0L));
              g->y[pt] = (double)(-(ld)R + g->h * cy + 0.5L * g->h * (xg[qb] + 1.0L));
              g->z[pt] = (double)(-(ld)R + g->h * cz + 0.5L * g->h * (xg[qa] + 1.0L));
              g->w[pt] = wg[qa] * wg[qb] * wg[qc] * (0.5L * g->h) * (0.5L * g->h) * (0.5L * g->h);
            }
      }
}

static void o3_free(o3grid_t *g) {
  free(g->x);
  free(g->w);
  free(g->bas);
  free(g->dofs);
}

/* O3, O4 at every point: T[8][N] = T_D, T_Kx, T_Ky, T_Kz (not multiplied by w), then the |.| versions */
static void o3_fields(const o3grid_t *g, int S, const double *mass, const double *charge, const double *f, ld *T) {
  const long long N = g->N;
  for (long long k = 0; k < 8 * N; k++) T[k] = 0.0L;
#pragma omp parallel for schedule(static)
  for (long long pt = 0; pt < N; pt++) {
    long long c = pt / g->nq;
    int q = (int)(pt % g->nq);
    for (int a = 0; a < S; a++) {
      ld e2 = (ld)charge[a] * (ld)charge[a], im = 1.0L / (ld)mass[a];
      ld v[4] = {0, 0, 0, 0}, va[4] = {0, 0, 0, 0};
      for (int n = 0; n < g->nb; n++) {
        ld fv = f[(long long)a * g->ndof + g->dofs[c * g->nb + n]];
        const ld *b = g->bas + 4 * ((size_t)q * g->nb + n);
        for (int t = 0; t < 4; t++) {
          v[t] += b[t] * fv;
          va[t] += fabsl(b[t]) * fabsl(fv);
        }
      }
      T[pt] += e2 * v[0];
      T[4 * N + pt] += e2 * va[0];
      for (int t = 1; t < 4; t++) {
        T[t * N + pt] += e2 * im * v[t];
        T[(4 + t) * N + pt] += e2 * im * va[t];
      }
    }
  }
}

/* O12 at every point: G[18][N] = signed sums from w T, then |.| sums from w |T|^abs */
static void o3_inner(const o3grid_t *g, const ld *T, ld *G) {
  const long long N = g->N;
  const double *x = g->x, *y = g->y, *z = g->z;
#pragma omp parallel for schedule(dynamic, 8)
  for (long long i = 0; i < N; i++) {
    nsum_t acc[9], aac[9];
    memset(acc, 0, sizeof acc);
    memset(aac, 0, sizeof aac);
    for (long long j = 0; j < N; j++) {
      if (x[j] == x[i] && y[j] == y[i] && z[j] == z[i]) continue; /* Amb-3 */
      const ld u[3] = {(ld)x[i] - x[j], (ld)y[i] - y[j], (ld)z[i] - z[j]};
      const ld s2 = u[0] * u[0] + u[1] * u[1] + u[2] * u[2], s3 = s2 * sqrtl(s2);
      ld U[3][3];
      for (int a = 0; a < 3; a++)
        for (int b = 0; b < 3; b++) U[a][b] = ((a == b ? s2 : 0.0L) - u[a] * u[b]) / s3;
      const ld wj = g->w[j];
      int k = 0;
      for (int a = 0; a < 3; a++)
        for (int b = a; b < 3; b++, k++) {
          nadd(&acc[k], wj * T[j] * U[a][b]);
          nadd(&aac[k], wj * T[4 * N + j] * fabsl(U[a][b]));
        }
      for (int a = 0; a < 3; a++) {
        nadd(&acc[6 + a], wj * (U[a][0] * T[N + j] + U[a][1] * T[2 * N + j] + U[a][2] * T[3 * N + j]));
        nadd(&aac[6 + a], wj * (fabsl(U[a][0]) * T[5 * N + j] + fabsl(U[a][1]) * T[6 * N + j] + fabsl(U[a][2]) * T[7 * N + j]));
      }
    }
    for (int c = 0; c < 9; c++) {
      G[c * N + i] = nval(&acc[c]);
      G[(9 + c) * N + i] = nval(&aac[c]);
    }
  }
}

/* O6-O8 (+O10 when Ga != NULL): per species the element matrices from G at the cube's points, added
 * at (dof_k, dof_l) of the CSR pattern; vals [S][nnz] */
static void o3_assemble(const o3grid_t *g, int S, const double *mass, const double *charge, double nu, const ld *G,
                        const ld *Ga, double *vals, double *absvals) {
  const long long N = g->N, nnz = g->nnz;
  const int nb = g->nb, nq = g->nq;
  long long *rowptr = malloc(sizeof(long long) * (g->ndof + 1));
  int *col = malloc(sizeof(int) * nnz);
  oracle3d_pattern(g->ncell, g->p, rowptr, col);
  ld *acc = calloc((size_t)2 * S * nnz, sizeof(ld));
  const int sym[3][3] = {{0, 1, 2}, {1, 3, 4}, {2, 4, 5}};
#pragma omp parallel for schedule(static)
  for (int a = 0; a < S; a++) {
    ld e2 = (ld)charge[a] * (ld)charge[a], im = 1.0L / (ld)mass[a];
    ld fD = -(ld)nu * e2 * im * im, fK = (ld)nu * e2 * im; /* O6 */
    ld *C = malloc(sizeof(ld) * 2 * nb * nb);
    for (long long c = 0; c < g->nc3; c++) {
      for (int k = 0; k < 2 * nb * nb; k++) C[k] = 0.0L;
      for (int q = 0; q < nq; q++) { /* O7 */
        long long pt = c * nq + q;
        ld D[3][3], K[3], Da[3][3], Ka[3];
        for (int r = 0; r < 3; r++) {
          for (int t = 0; t < 3; t++) {
            D[r][t] = fD * G[sym[r][t] * N + pt];
            Da[r][t] = Ga ? fabsl(fD) * Ga[sym[r][t] * N + pt] : 0.0L;
          }
          K[r] = fK * G[(6 + r) * N + pt];
          Ka[r] = Ga ? fabsl(fK) * Ga[(6 + r) * N + pt] : 0.0L;
        }
        for (int k = 0; k < nb; k++) {
          const ld *bk = g->bas + 4 * ((size_t)q * nb + k);
          for (int l = 0; l < nb; l++) {
            const ld *bl = g->bas + 4 * ((size_t)q * nb + l);
            ld v = 0.0L, va = 0.0L;
            for (int r = 0; r < 3; r++) {
              for (int t = 0; t < 3; t++) {
                v += bk[1 + r] * D[r][t] * bl[1 + t];
                va += fabsl(bk[1 + r]) * Da[r][t] * fabsl(bl[1 + t]);
              }
              v += bk[1 + r] * K[r] * bl[0];
              va += fabsl(bk[1 + r]) * Ka[r] * fabsl(bl[0]);
            }
            C[k * nb + l] += g->w[pt] * v;
            C[nb * nb + k * nb + l] += fabsl(g->w[pt]) * va;
          }
        }
      }
      for (int k = 0; k < nb; k++) /* O8 */
        for (int l = 0; l < nb; l++) {
          long long at = o3_find(rowptr, col, g->dofs[c * nb + k], (int)g->dofs[c * nb + l]);
          acc[(long long)a * nnz + at] += C[k * nb + l];
          acc[(long long)(S + a) * nnz + at] += C[nb * nb + k * nb + l];
        }
    }
    free(C);
  }
  for (long long k = 0; k < (long long)S * nnz; k++) {
    vals[k] = (double)acc[k];
    if (absvals) absvals[k] = (double)acc[(long long)S * nnz + k];
  }
  free(acc);
  free(col);
  free(rowptr);
}

void oracle3d_points(int ncell, int order, double R, double *xyz, double *w) {
  o3grid_t g;
  o3_grid(ncell, order, R, &g);
  for (long long k = 0; k < g.N; k++) {
    xyz[k] = g.x[k];
    xyz[g.N + k] = g.y[k];
    xyz[2 * g.N + k] = g.z[k];
    w[k] = (double)g.w[k];
  }
  o3_free(&g);
}

void oracle3d_fields(int ncell, int order, double R, int S, const double *mass, const double *charge, const double *f,
                     double *T) {
  o3grid_t g;
  o3_grid(ncell, order, R, &g);
  ld *t = malloc(sizeof(ld) * 8 * g.N);
  o3_fields(&g, S, mass, charge, f, t);
  for (long long k = 0; k < 4 * g.N; k++) T[k] = (double)t[k];
  free(t);
  o3_free(&g);
}

void oracle3d_assemble(int ncell, int order, double R, int S, const double *mass, const double *charge, double nu,
                       const double *G, double *vals) {
  o3grid_t g;
  o3_grid(ncell, order, R, &g);
  ld *Gl = malloc(sizeof(ld) * 9 * g.N);
  for (long long k = 0; k < 9 * g.N; k++) Gl[k] = G[k];
  o3_assemble(&g, S, mass, charge, nu, Gl, NULL, vals, NULL);
  free(Gl);
  o3_free(&g);
}

void oracle3d_jacobian(int ncell, int order, double R, int S, const double *mass, const double *charge, double nu,
                       const double *f, double *vals, double *absvals) {
  o3grid_t g;
  o3_grid(ncell, order, R, &g);
  ld *T = malloc(sizeof(ld) * 8 * g.N), *G = malloc(sizeof(ld) * 18 * g.N);
  o3_fields(&g, S, mass, charge, f, T);
  o3_inner(&g, T, G);
  o3_assemble(&g, S, mass, charge, nu, G, G + 9 * g.N, vals, absvals);
  free(G);
  free(T);
  o3_free(&g);
}
