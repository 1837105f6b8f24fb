/* oracle.h -- plain, slow, CPU reference for the Landau Jacobian hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load liboracle.so.  It shares no code, header, table or constant
 * generator with the CUDA path (paper_conf_ipps_adamsbkw22_b200/csrc); neither side includes or
 * links the other.
 *
 * What it computes (PAPER.md = Adams, Brennan, Knepley, Wang, IPDPS 2022; "@N" = character offset
 * N in the single-line /root/reference/PAPER.md; "O<k>" = step k of SURVEY.md §8(c)):
 *   O1  Q_p Lagrange space (equispaced nodes) on a 2:1-balanced quadtree, hanging-node constraints
 *       interpolated from the coarse edge (@14112, @42262; readings Amb-8, Amb-10, Amb-12)
 *   O2  (p+1)^2 Gauss-Legendre points per cell, w = w_a w_b (h/2)^2 r, no 2 pi (Amb-2, Amb-9)
 *   O3  f, grad f at the points;  O4  T_D, T_K sums over the source point's species (Alg. 1
 *       lines 5-8 @15260-15570; Eqs. 10-11 @12313-13111)
 *   O5  inner integral G_D(i) = sum_{j != i} w_j T_D(j) U^D(i,j),  G_K(i) = sum_j w_j U^K(i,j).T_K(j)
 *       (Eqs. 7-8 @9251-9509, Alg. 1 lines 3-11 @14935-15669), U^D/U^K = exact azimuthal
 *       integrals of Eq. 3 (@7593) written with complete elliptic integrals K, E (long-double AGM)
 *       for s >= 1/4, and the binomial series in s below (Amb-1, Amb-6, Amb-7); Neumaier sums.
 *   O6  species factors (Alg. 1 lines 13-16 @15729-16012);  O7 element matrices (Eqs. 5-6
 *       @8833-9206);  O8 assembly J_a = sum_e P_e^T C_e P_e, species-block-diagonal (@11277)
 *   O9  mass matrix shift * sum_e P_e^T (sum_q w phi phi) P_e (@39757-39999)
 *   O10 condition scale: the same assembly with every product replaced by its absolute value.
 *   O11 E_z advection matrix sum_e P_e^T (sum_q w phi_k d_z phi_l) P_e (Eq. 4, @8216-8654)
 *   O12 the inner integral with the 3D Cartesian tensor of Eq. 3 (@7997-8072)
 *   O13 the whole 3D Cartesian Jacobian (O3-O8, O10 on a uniform grid of Q_p cubes, tensor of O12)
 * Pins: see tests/test_oracle_*.py (P1-P9 of SURVEY.md §8(c); P13 for O12).
 */
#ifndef LANDAU_ORACLE_H
#define LANDAU_ORACLE_H
#ifdef __cplusplus
extern "C" {
#endif

typedef struct oracle_s oracle_t;

/* cells: concatenated [sum ncells][3] = {r0, z0, h} (lower-left corner, square side h) per grid;
 * grid g covers [0, radius[g]] x [-radius[g], radius[g]].  nq1d = 0 -> order + 1.
 * Returns NULL on invalid input and writes a message to err. */
oracle_t *oracle_create(int ngrids, const long long *ncells, const double *cells, const double *radius,
                        int order, int nq1d, int nspecies, const double *mass, const double *charge,
                        const int *grid, double nu, char *err, int errlen);
void oracle_destroy(oracle_t *o);

/* ndof = sum over species of ndof(grid(species)); nnz = CSR nonzeros of the block-diagonal J;
 * ncoo = sum over species of sum over cells of its grid of n_e^2 (n_e = distinct DOFs of cell e). */
void oracle_sizes(const oracle_t *o, long long *ndof, long long *npoints, long long *nnz, long long *ncoo);
long long oracle_grid_ndof(const oracle_t *o, int g);
long long oracle_grid_npoints(const oracle_t *o, int g);
/* DOF node coordinates of grid g, in the oracle's own numbering (z ascending, then r ascending). */
void oracle_grid_nodes(const oracle_t *o, int g, double *r, double *z);
/* quadrature points, grid-major, cell order as given, q = qz*(nq1d) + qr inside a cell */
void oracle_points(const oracle_t *o, double *r, double *z, double *w);
/* CSR pattern of the species-block-diagonal matrix (rows/cols sorted) */
void oracle_pattern(const oracle_t *o, long long *rowptr, int *col);
/* COO pattern: per species, per cell, the cell's sorted distinct DOFs x same, row-major */
void oracle_coo_pattern(const oracle_t *o, int *row, int *col);

/* O12: U(u) of Eq. 3 in 3D Cartesian velocity space, (xx, xy, xz, yy, yz, zz). */
void oracle_tensor3d(double ux, double uy, double uz, double out[6]);
/* O12: G = [9][n] = (G_D xx, xy, xz, yy, yz, zz, G_K x, y, z) at every point (wTD = w T_D and
 * wTK = w T_K premultiplied), coincident points excluded; Gabs: the sums of absolute values. */
void oracle_inner3d(long long n, const double *x, const double *y, const double *z, const double *wTD,
                    const double *wTKx, const double *wTKy, const double *wTKz, double *G, double *Gabs);

/* O13: the 3D Cartesian Landau Jacobian (NEXT-4 completed, @7997-8072) on a uniform grid of
 * ncell^3 Q_p cubes over [-R, R]^3: DOF dof(ix, iy, iz) = (iz M + iy) M + ix of the lattice of
 * M = ncell p + 1 nodes per direction; (p+1)^3 Gauss points per cube; O3/O4 fields, O12 inner
 * integral, O6/O7 element matrices grad phi_k . D~ grad phi_l + (grad phi_k . K~) phi_l, O8 assembly
 * (no constraints), O10 |.| scale.  f = [S][ndof] (species-major), vals / absvals = [S][nnz] CSR values
 * in the pattern of oracle3d_pattern (rows and columns ascending; absvals may be NULL). */
void oracle3d_sizes(int ncell, int order, long long *ndof, long long *npoints, long long *nnz);
void oracle3d_pattern(int ncell, int order, long long *rowptr, int *col);
void oracle3d_nodes(int ncell, int order, double R, double *xyz);  /* [3][ndof] */
/* the Gauss points [3][npoints] and weights [npoints] (cube-major; q = (a S + b) S + c along z, y, x) */
void oracle3d_points(int ncell, int order, double R, double *xyz, double *w);
/* O3/O4 alone: T [4][npoints] = T_D, T_Kx, T_Ky, T_Kz (not multiplied by w) */
void oracle3d_fields(int ncell, int order, double R, int S, const double *mass, const double *charge, const double *f,
                     double *T);
/* O6-O8 alone, from a given G [9][npoints] (G_D xx, xy, xz, yy, yz, zz, G_K x, y, z): vals [S][nnz] */
void oracle3d_assemble(int ncell, int order, double R, int S, const double *mass, const double *charge, double nu,
                       const double *G, double *vals);
void oracle3d_jacobian(int ncell, int order, double R, int S, const double *mass, const double *charge, double nu,
                       const double *f, double *vals, double *absvals);

/* U^D_rr, U^D_rz, U^D_zz, U^K_rr, U^K_zr at target (r, z), source (rb, zb). */
void oracle_tensor(double r, double z, double rb, double zb, double out[5]);

/* O5 on arbitrary points: for each target t (index into the n points), G[c*nt + t], c = 0..4 =
 * (G_D rr, rz, zz, G_K r, z); Gabs: same sums of absolute values.  Pairs with identical
 * coordinates are skipped (Amb-3).  Either Gabs may be NULL. */
void oracle_inner(long long n, const double *r, const double *z, const double *w, const double *TD,
                  const double *TKr, const double *TKz, long long nt, const long long *targets,
                  double *G, double *Gabs);

/* O3+O4: per point T_D, T_K (not multiplied by w). f = species-major coefficients [ndof]. */
void oracle_point_fields(const oracle_t *o, const double *f, double *TD, double *TKr, double *TKz);
/* O3-O5 for a subset of points (targets = NULL, nt = npoints -> all): G[5][nt], Gabs[5][nt] */
void oracle_point_coeffs(const oracle_t *o, const double *f, long long nt, const long long *targets,
                         double *G, double *Gabs);
/* O3-O8(+O10): CSR values [nnz] and |.| scale [nnz] */
void oracle_jacobian(const oracle_t *o, const double *f, double *vals, double *absvals);
/* O3-O7(+O10) in COO layout [ncoo]; elem_mask (global cell index, may be NULL = all) selects the
 * cells computed (others untouched) - the inner integral is then evaluated only at their points. */
void oracle_jacobian_coo(const oracle_t *o, const double *f, const unsigned char *elem_mask,
                         double *vals, double *absvals);
/* O9: CSR values [nnz] of shift * M for every species block */
void oracle_mass(const oracle_t *o, double shift, double *vals);
void oracle_mass_coo(const oracle_t *o, double shift, double *vals);
/* O11: CSR / COO values of the unscaled E_z advection matrix sum_e P_e^T (sum_q w phi_k d_z phi_l) P_e
 * for every species block (the caller applies e_a E_z / m_a; Eq. 4 @8216-8654) */
void oracle_advection(const oracle_t *o, double *vals);
void oracle_advection_coo(const oracle_t *o, double *vals);

void oracle_set_threads(int n);
int oracle_get_threads(void);

#ifdef __cplusplus
}
#endif
#endif
