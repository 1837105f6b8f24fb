/* landau.h -- C ABI of liblandau.so: the FP64 conservative finite-element Landau Jacobian on B200.
 *
 * Reference: M. F. Adams, D. P. Brennan, M. G. Knepley, P. Wang, "Landau collision operator in the
 * CUDA programming model applied to thermal quench plasmas", IPDPS 2022.  Citations "@N" are
 * character offsets into the single-line paper text PAPER.md; "Amb-k" are the
 * readings of ambiguous passages listed in DESIGN.md.
 *
 * What a build computes; all arithmetic is FP64 on the device:
 *   a-1  f, grad f of every species at the quadrature points from the FE coefficients (Alg. 1
 *        lines 5-8 @15260-15570; Eqs. 10-11 @12313-13111), summed into
 *        T_D(j) = sum_b e_b^2 f_b(j),  T_K(j) = sum_b e_b^2 (m0/m_b) grad f_b(j)  (b on j's grid);
 *   a-2  the inner integral (Eqs. 7-8 @9251-9509; Alg. 1 lines 3-11 @14935-15669)
 *        G_D(i) = sum_{j: (r_j,z_j) != (r_i,z_i)} w_j T_D(j) U^D(i,j),
 *        G_K(i) = sum_j w_j U^K(i,j) . T_K(j), with U^D, U^K the azimuthal integrals of Eq. 3
 *        (@7593) written with complete elliptic integrals (Amb-1, Amb-6);
 *   a-3  species factors  D~_a = -nu e_a^2 (m0/m_a)^2 G_D,  K~_a = nu e_a^2 (m0/m_a) G_K
 *        (Alg. 1 lines 13-16 @15729-16012);
 *   a-4  element matrices C_a[k,l] = sum_q w_q [grad phi_k . D~_a . grad phi_l + (grad phi_k . K~_a) phi_l]
 *        (Eqs. 5-6 @8833-9206; rows = test functions);
 *   a-5  assembly J_a = sum_e P_e^T C_a,e P_e with hanging-node interpolation P_e (@14112, @42262),
 *        species-block-diagonal (@11094-11357), deterministic (no atomics; Amb-15);
 *   a-6  mass  shift * sum_e P_e^T (sum_q w_q phi_k phi_l) P_e (@39757-39999).
 * J is the Picard ("approximate linearization", @10657-10914) matrix with C(f) ~= J f (Amb-4); the
 * caller forms shift*M - J.
 *
 * Units: App. A (@58269): velocities in v0 = (8 k T_e / (pi m_e))^(1/2), masses in m_e (m0 = m_e),
 * charges in e, nu_ab = nu e_a^2 e_b^2 with nu = 1 for lnLambda = 10 (Amb-13).
 *
 * Discretisation conventions (fixed by this ABI):
 *   - grid g is a 2:1-balanced quadtree of square leaf cells {r0, z0, h} (lower-left corner, side h)
 *     tiling [0, R_g] x [-R_g, R_g]; cells are given leaves-only, in any order;
 *   - Q_p Lagrange elements, p in {2,3,4}, equispaced nodes (Amb-8); a node on the interior of a
 *     coarser neighbour's edge is constrained to that edge's degree-p interpolant (Amb-10);
 *   - (p+1)^2 Gauss-Legendre points per cell, weight w = w_a w_b (h/2)^2 r, no 2 pi (Amb-2, Amb-9);
 *   - points are numbered grid-major, cells in input order, q = qz*(p+1) + qr inside a cell;
 *   - DOFs of a grid: the non-constrained node positions, ordered by z ascending then r ascending
 *     (Amb-12); the state vector is species-major: [f_0 on grid(0)][f_1 on grid(1)]...;
 *   - CSR: block a holds rows/columns offset by sum_{b<a} ndof(grid(b)); columns sorted;
 *   - COO: per species a, per cell e of grid(a) (input order), the n_e x n_e block P_e^T C P_e over
 *     the cell's sorted distinct DOFs, row-major; duplicates across cells are to be summed.
 *
 * Conventions of the calls:
 *   - every call returns 0 (LANDAU_OK) or a negative code; nothing throws or aborts;
 *   - device pointers (suffix _dev) are owned by the caller; the library owns its workspace;
 *   - all device work is enqueued on the stream given to landau_create; outputs are valid once that
 *     stream has synchronised; set_state copies its input (the caller may reuse it immediately);
 *   - one handle per host thread; a handle is tied to one device.
 */
#ifndef LANDAU_H
#define LANDAU_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct landau_s *landau_t;

enum {
  LANDAU_OK = 0,
  LANDAU_EINVAL = -1,       /* invalid argument (bad mesh, order, species, format, size)        */
  LANDAU_ENOMEM = -2,       /* host or device allocation failed                                  */
  LANDAU_ECUDA = -3,        /* a CUDA runtime call or kernel launch failed                       */
  LANDAU_ENCCL = -4,        /* NCCL could not be loaded or a collective failed                   */
  LANDAU_ESTATE = -5,       /* jacobian/point_coeffs before set_state (or batch size mismatch)   */
  LANDAU_EUNSUPPORTED = -6  /* valid request this build does not implement                       */
};
enum { LANDAU_CSR = 0, LANDAU_COO = 1 };
enum { LANDAU_DIST_REPLICATE = 0, LANDAU_DIST_BATCH = 1, LANDAU_DIST_ELEMENTS = 2 };

typedef struct {
  int32_t ngrids;
  const int64_t *ncells;   /* [ngrids] leaf cells per grid                                       */
  const double *cells;     /* [sum ncells][3] = {r0, z0, h}, grids concatenated                  */
  const double *radius;    /* [ngrids] R_g                                                       */
} landau_mesh_t;

typedef struct {
  int32_t order;           /* p in {2, 3, 4}                                                     */
  int32_t nq1d;            /* Gauss points per direction; 0 -> p + 1 (the only supported value)   */
  int32_t nspecies;        /* S in [1, 16]                                                       */
  const double *mass;      /* [S] m_a / m_e > 0                                                  */
  const double *charge;    /* [S] e_a / e (only e_a^2 enters)                                    */
  const int32_t *grid;     /* [S] grid index of each species                                     */
  double nu;               /* nu_ab = nu e_a^2 e_b^2                                             */
} landau_params_t;

typedef struct {
  int32_t rank, world;         /* this process and the number of processes (one GPU each)        */
  const void *nccl_unique_id;  /* 128 bytes from landau_nccl_unique_id on rank 0, broadcast by the
                                  caller (torch.distributed); only read for LANDAU_DIST_ELEMENTS   */
  int32_t mode;                /* LANDAU_DIST_*: REPLICATE and BATCH need no communicator (the
                                  caller splits batches); ELEMENTS distributes one mesh's inner
                                  integral over the ranks: on a z-mirror mesh (every configuration
                                  of SURVEY §8(d)) the upper-half tile pairs are split into world
                                  contiguous equal-work ranges (landau_pair_partition) and the
                                  partial G summed by one NCCL all-reduce; otherwise the target
                                  cells are split into world contiguous equal ranges
                                  (landau_partition) and G all-gathered over NCCL.  Every rank then
                                  forms the element matrices and the full CSR/COO itself.          */
} landau_dist_t;

/* cuda_device = LANDAU_HOST_ONLY builds only the host-side plan (sizes, nodes, points, patterns can
 * be queried without a GPU); every device call on such a handle returns LANDAU_EUNSUPPORTED. */
#define LANDAU_HOST_ONLY (-1)

/* Create a handle: validates the mesh (EINVAL if cells overlap, do not tile [0,R]x[-R,R], are not
 * on a quadtree lattice, r0 < 0, h <= 0, or violate 2:1 edge balance), builds the FE space, the
 * CSR/COO patterns and the assembly gather map on the host, uploads them and computes the mass
 * matrix on the device.  cuda_stream is a cudaStream_t (NULL = legacy default stream).
 * dist may be NULL (single process). */
int landau_create(landau_t *out, const landau_mesh_t *mesh, const landau_params_t *prm, int32_t cuda_device,
                  void *cuda_stream, const landau_dist_t *dist);
void landau_destroy(landau_t h);

/* Sizes: ndof = sum over species of ndof(grid(a)); npoints = N; nnz_csr and ncoo of the whole
 * block-diagonal matrix.  Any output pointer may be NULL. */
int landau_get_sizes(landau_t h, int64_t *ndof, int64_t *npoints, int64_t *nnz_csr, int64_t *ncoo);
int landau_get_grid_ndof(landau_t h, int32_t grid, int64_t *ndof);
/* host, caller-allocated [ndof(grid)]: coordinates of the DOF nodes of one grid, in DOF order */
int landau_get_nodes(landau_t h, int32_t grid, double *r, double *z);
/* host, caller-allocated [npoints]: quadrature points and weights */
int landau_get_points(landau_t h, double *r, double *z, double *w);
/* host, caller-allocated; any pointer may be NULL: csr_rowptr [ndof+1], csr_col [nnz_csr],
 * coo_row/coo_col [ncoo] */
int landau_get_pattern(landau_t h, int64_t *csr_rowptr, int32_t *csr_col, int32_t *coo_row, int32_t *coo_col);

/* State: f_dev = [ndof] species-major FE coefficients (device).  Batched: [nbatch][ndof]; the
 * batch shares the mesh (independent spatial vertices). */
int landau_set_state(landau_t h, const double *f_dev);
int landau_set_state_batched(landau_t h, int64_t nbatch, const double *f_dev);

/* Jacobian of the current state: values_dev = [nnz_csr] (LANDAU_CSR) or [ncoo] (LANDAU_COO);
 * batched: [nbatch][nnz] with nbatch equal to the last set_state_batched. */
int landau_jacobian(landau_t h, double *values_dev, int32_t format);
int landau_jacobian_batched(landau_t h, int64_t nbatch, double *values_dev, int32_t format);

/* Convenience for host data (end-to-end path): copies f_host [nbatch][ndof] to the device, builds,
 * copies the values back to values_host [nbatch][nnz] and synchronises.  Large batches are cut into
 * up to 8 chunks whose uploads, builds and downloads overlap on two internal copy streams (pinned
 * host memory required for the overlap).  Does not change the handle's set_state state. */
int landau_jacobian_host(landau_t h, int64_t nbatch, const double *f_host, double *values_host, int32_t format);

/* Mass matrix values shift * M for every species block: [nnz_csr] or [ncoo]. */
int landau_mass(landau_t h, double shift, double *values_dev, int32_t format);

/* Debug/parity hook for step a-2: G_dev = [5][npoints] (G_D rr, rz, zz, G_K r, z) of the current
 * state (batched: [nbatch][5][npoints]). */
int landau_point_coeffs(landau_t h, double *G_dev);
int landau_point_coeffs_batched(landau_t h, int64_t nbatch, double *G_dev);

/* Element split (LANDAU_DIST_ELEMENTS): contiguous cell range [e0, e1) owned by a rank for a mesh
 * of nelem cells; pure host arithmetic, usable without a GPU. */
int landau_partition(int64_t nelem, int32_t world, int32_t rank, int64_t *e0, int64_t *e1);
/* Pair split (LANDAU_DIST_ELEMENTS on a z-mirror mesh): the mirror kernel's items -- tile pairs
 * (a, b), a <= b, in the order b = 0.., a = 0..b, ntiles (T) upper-half tiles of 32 points,
 * T (T + 1) / 2 items -- weighted 2 per pair and 1 per diagonal item (half its steps); rank takes
 * the contiguous item range [q0, q1) whose weight prefix covers [rank T^2 / world,
 * (rank + 1) T^2 / world).  Pure host arithmetic.  EINVAL: ntiles < 0, world < 1, rank outside
 * [0, world), NULL outputs. */
int landau_pair_partition(int64_t ntiles, int32_t world, int32_t rank, int64_t *q0, int64_t *q1);
/* 128-byte NCCL unique id (rank 0 only; loads libnccl.so.2 on demand). */
int landau_nccl_unique_id(void *out128);

/* Per-stage device timers (CUDA events on the handle's stream): stage = 0 field, 1 inner,
 * 2 reduce, 3 element, 4 assemble, 5 mass, 6 allgather, 7 band factor, 8 band solve.  enable resets
 * the accumulators. */
enum { LANDAU_T_FIELD = 0, LANDAU_T_INNER, LANDAU_T_REDUCE, LANDAU_T_ELEMENT, LANDAU_T_ASSEMBLE,
       LANDAU_T_MASS, LANDAU_T_ALLGATHER, LANDAU_T_FACTOR, LANDAU_T_SOLVE, LANDAU_NTIMERS };
int landau_set_timing(landau_t h, int32_t enable);
/* ms[LANDAU_NTIMERS] total milliseconds, launches[LANDAU_NTIMERS] kernel launches (synchronises) */
int landau_get_timing(landau_t h, double *ms, int64_t *launches);
/* kernels launched by this handle since creation (all stages) */
int landau_get_launch_count(landau_t h, int64_t *count);

/* Tensor cache (SURVEY §8(f) NEXT-4, U-caching variant): the axisymmetric tensors depend only on the
 * mesh, so for a handle whose builds share it (batched vertices, repeated Newton iterations) the
 * library can evaluate the five N x N tensor matrices U^D_rr, U^D_rz, U^D_zz, U^K_rr, U^K_zr once
 * (7 N^2 doubles, stacked for GEMM) and then form the inner integral of a batch as three FP64 GEMMs
 * (cuBLAS DGEMM on the FP64 tensor cores, libcublas.so.12 loaded on demand):
 *   [G_Drr; G_Drz; G_Dzz] = [U^D_rr; U^D_rz; U^D_zz] (3N x N) . W_D (N x batch)
 *   G_Kr = [U^K_rr  U^D_rz] (N x 2N) . [W_Kr; W_Kz],   G_Kz = [U^K_zr  U^D_zz] . [W_Kr; W_Kz].
 * The same sums as the pairwise kernels up to summation order.  EUNSUPPORTED for element-split
 * handles or when 7 N^2 doubles exceed 16 GiB; enable = 0 frees the cache.  enable = 2 keeps the
 * GEMM formulation but re-evaluates the tensors (every ordered pair) at every build: the cost of a
 * build that shares nothing with the previous one. */
int landau_set_tensor_cache(landau_t h, int32_t enable);

/* NEXT-2 (PAPER.md:1@24330-26180, §III-G): the paper's direct solver for the implicit
 * step.  Each species block of A = shift * M - J is put in reverse Cuthill-McKee order and band
 * storage (half-bandwidth B = UBW = LBW of the grid's pattern) and factored by the outer-product
 * band LU without pivoting (Golub-Van Loan Alg. 4.3.1), one CTA per (batch item, species block);
 * the solve is a forward/backward substitution, one warp per block.  Without pivoting the
 * factorisation needs A to be safely non-singular on its leading minors, as it is for the shift of
 * an implicit step (shift * M dominant); a zero pivot yields inf/nan in x, nothing aborts.
 *   landau_band_info:      B and the RCM permutation perm[new] = old of one grid (host, may be NULL)
 *   landau_band_factor_batched: J_csr_dev = [nbatch][nnz_csr] (e.g. from landau_jacobian_batched)
 *   landau_band_solve_batched:  b_dev, x_dev = [nbatch][ndof] species-major (may alias); uses the
 *                          last factorisation (ESTATE before any, when nbatch differs, or after an
 *                          implicit step, whose fused factorisation keeps only U -- factor again) */
int landau_band_info(landau_t h, int32_t grid, int32_t *bandwidth, int32_t *perm);
int landau_band_factor_batched(landau_t h, int64_t nbatch, double shift, const double *J_csr_dev);
int landau_band_solve_batched(landau_t h, int64_t nbatch, const double *b_dev, double *x_dev);
/* The same factorisation of A = shift * M + E_z (e_a / m_a) A_E - J per species block a, with A_E the
 * advection matrix below (the electric-field term of Eq. 4).  Ez = 0 is landau_band_factor_batched. */
int landau_band_factor_field_batched(landau_t h, int64_t nbatch, double shift, double Ez, const double *J_csr_dev);

/* E_z advection matrix of Eq. 4 (PAPER.md:1@8216-8654): the weak form of (0, e_a E_z / m_a) . grad f_a
 * tested with psi = phi_k, i.e. per species block E_z (e_a / m_a) sum_e P_e^T (sum_q w phi_k d_z phi_l) P_e
 * with the mass matrix's w (no 2 pi, Amb-2); charges in e, masses in m0, E_z in the same App.-A units
 * as time.  values_dev: [nnz_csr] or [ncoo] device buffer (caller-owned); cached at create. */
int landau_advection(landau_t h, double Ez, double *values_dev, int32_t format);

/* NEXT-3: one backward-Euler step of Eq. 4 without source,
 *   M (f^{n+1} - f^n) / dt + E_z (e/m) A_E f^{n+1} = C(f^{n+1}),   C(f) = J(f) f (Amb-4),
 * solved by the paper's quasi-Newton iteration with the Jacobian fully recomputed about each iterate
 * (PAPER.md:1@10500-10978): (M/dt + E_z (e/m) A_E - J(f^k)) f^{k+1} = M f^n / dt, every item of the
 * batch independently, entirely on the device (set_state, Jacobian build, band LU, solve per
 * iteration).  f_old_dev, f_new_dev: [nbatch][ndof] device buffers, distinct (f_new is overwritten;
 * the iteration starts from f_old).  Stops after max_iter iterations, or earlier once every item's
 * ||f^{k+1} - f^k|| / ||f^{k+1}|| <= rtol (rtol > 0 reads the norms back once per iteration; rtol <= 0
 * runs exactly max_iter iterations with one read-back at the end).  iters (host, may be NULL): the
 * iterations run; dnorm (host, may be NULL): the largest relative change of the last iteration.
 * The handle's state afterwards is the last iterate f^{k} the final Jacobian was built about.
 * Where the blocked (DMMA) band kernel applies, each iteration's factorisation also eliminates the
 * right-hand side forward and stores only U (the solve then runs the backward pass alone); env
 * LANDAU_BAND_FUSED=0 selects factor + full solve.  Either way the band factor held afterwards is the
 * last iteration's. */
int landau_implicit_step_batched(landau_t h, int64_t nbatch, double dt, double Ez, const double *f_old_dev,
                                 double *f_new_dev, int32_t max_iter, double rtol, int32_t *iters, double *dnorm);
/* The same step with the source term S_a(t) of Eq. 1 / Eq. 4 (PAPER.md:1@6337, @8216; the thermal-quench
 * "pulse of cold ions ... injected with the source term in (4)", @34560): src_dev [nbatch][ndof]
 * (device, species-major, may be NULL = no source) holds the FE coefficients sigma of S_a at t^{n+1};
 * (psi_k, S_a) = (M sigma)_k with the mass matrix's weighted L2 product (Amb-2), so each iterate solves
 *   (M/dt + E_z (e_a/m_a) A_E - J(f^k)) f^{k+1} = M (f^n / dt + sigma)
 * and every iterate satisfies the per-species density balance
 *   1^T [M (f^{k+1} - f^n)/dt + E_z (e_a/m_a) A_E f^{k+1}] = 1^T M sigma   (1^T J = 0).
 * The time profile and shape of the source are the caller's (R-7).  Errors as above. */
int landau_implicit_step_source_batched(landau_t h, int64_t nbatch, double dt, double Ez, const double *f_old_dev,
                                        const double *src_dev, double *f_new_dev, int32_t max_iter, double rtol,
                                        int32_t *iters, double *dnorm);

/* Mirror symmetry (v_par -> -v_par, i.e. z -> -z): when every grid's quadrature points come in pairs
 * (r, z), (r, -z) BIT-EXACTLY (no point on z = 0; the dyadic meshes of every configuration of SURVEY
 * §8(d) qualify, the cell-centre point formula keeps mirrored points exact negatives) the batched
 * (symmetric) inner integral evaluates each tensor once for four ordered interactions: reflection keeps
 * lambda+-, x, m and every azimuthal integral and negates the rz / zr components,
 * U(i', j') = F U(i, j) F with F = diag(1, -1), on top of the i <-> j symmetry (N^2/4 tensor
 * evaluations per build instead of N^2/2).  A mesh symmetric only up to rounding is not detected (the
 * general kernels run at the caller's exact points).  On by default when available.
 * enable: 0 = plain symmetric kernel; 1 = mirror, automatic (batches with at least 8 round weights per
 * SM -- C2: 32 vertices -- run the per-vertex kernel: one CTA per SM, a stream-K split of the batch's
 * (vertex, round) work, sums in shared memory, a split vertex's two or more partials added in CTA order;
 * smaller batches the slot kernel or, below that, the mirror-directed kernel); 2 = mirror slot kernel
 * only; 3 = per-vertex kernel for every batch size (one CTA per vertex when the batch is below one
 * vertex per SM: no vertex split).  enable != 0 on a non-symmetric mesh, or 3 when a
 * vertex's sums and staged inputs (168 B per upper-half point) exceed 200 KB of shared memory, is EUNSUPPORTED;
 * enable outside 0..3 is EINVAL. */
int landau_set_mirror(landau_t h, int32_t enable);
/* Whether the mesh is exactly z-mirror-symmetric (host logic, also on LANDAU_HOST_ONLY handles) and
 * whether the mirror kernels are in use on this handle.  Either pointer may be NULL.  EINVAL: h NULL. */
int landau_get_mirror(landau_t h, int32_t *mirror_symmetric, int32_t *mirror_active);
/* The per-vertex kernel's stream-K schedule, for diagnostics and tests: nrounds (host,
 * may be NULL) rounds per vertex; weight_prefix (host, [nrounds + 1], may be NULL) the cumulative round
 * weights (a round of pair items weighs 2, of diagonal items 1); ctas (may be NULL) the CTAs of an
 * automatic-mode launch.  Round rd of batch item v runs on CTA floor((v W + wp[rd]) ctas / (nbatch W)),
 * W = wp[nrounds]; a vertex whose rounds share one CTA is summed in one fixed order, whatever the batch.
 * EUNSUPPORTED when the per-vertex kernel is not available on this handle. */
int landau_get_vtx_schedule(landau_t h, int32_t *nrounds, int32_t *weight_prefix, int32_t *ctas);
/* The automatic-mode CTAs of the first and the last round of every vertex of an nbatch build (host,
 * caller-allocated [nbatch] each; first != last: the vertex is split between CTAs and summed through
 * partial slots).  A split vertex runs its rounds in its own order, chosen on the host so that every
 * stream-K cut falls on a round boundary (exact balance); the others keep the canonical order of
 * weight_prefix above.  EUNSUPPORTED as above. */
int landau_get_vtx_split(landau_t h, int64_t nbatch, int32_t *first_cta, int32_t *last_cta);

/* NEXT-4: the inner integral with the 3D Cartesian Landau tensor of Eq. 3
 * (PAPER.md:1@7593, "a full 3D model is supported in the library" @7997-8072), without azimuthal
 * reduction or elliptic integrals: for every point i of a 3D velocity-space point set,
 *   G_D(i) = sum_{j: v_j != v_i} wTD_j U(v_i - v_j),   G_K(i) = sum_j U(v_i - v_j) wTK_j,
 *   U(u) = (|u|^2 I - u u^T) / |u|^3.
 * xyz_dev: [3][n] point coordinates (x, y, z rows); wTD_dev: [n] w T_D; wTK_dev: [3][n] w T_K
 * (quadrature weights premultiplied, as in step a-1); G_dev: [9][n] output (G_D xx, xy, xz, yy, yz,
 * zz, G_K x, y, z).  All device pointers owned by the caller, on the current CUDA device; enqueued on
 * cuda_stream (temporary split-j partials come from the stream-ordered allocator).  Coincident
 * points contribute nothing.  EINVAL: n < 0 or a NULL pointer with n > 0; ENOMEM: partials;
 * ECUDA: launch failure.  Element matrices and assembly of a 3D model are not part of this call. */
int landau3d_inner(int64_t n, const double *xyz_dev, const double *wTD_dev, const double *wTK_dev, double *G_dev,
                   void *cuda_stream);

/* NEXT-4 completed ("a full 3D model is supported in the library", PAPER.md:1@7997-8072): the whole
 * Landau Jacobian in 3D Cartesian velocity space -- a-1 point fields, the inner integral of
 * landau3d_inner, a-4 element matrices (Eqs. 5-6 without the r weight: C^D_e[k][l] = sum_q w_q
 * grad phi_k . G_D grad phi_l, C^K_e[k][l] = sum_q w_q (grad phi_k . G_K) phi_l), a-3 species factors
 * and a-5 assembly -- on a uniform grid of ncell^3 Q_p cubes (order 2 or 3) over [-R, R]^3.
 *   DOFs: the lattice of M = ncell p + 1 equispaced nodes per direction, dof = (iz M + iy) M + ix at
 *   (-R + ix h/p, ...), h = 2R / ncell (landau3d_get_nodes: host [3][ndof]); (p+1)^3 Gauss points per
 *   cube.  The CSR pattern (landau3d_get_pattern: host rowptr [ndof+1], col [nnz]) has rows and
 *   columns ascending and is the same for every species block.
 *   landau3d_create: species masses (m0 units, > 0) and charges [nspecies <= 16], nu; the handle is
 *     tied to cuda_device and enqueues on cuda_stream.  EINVAL: bad sizes or parameters; ENOMEM.
 *   landau3d_jacobian: f_dev [nspecies][ndof] (device, species-major) -> J_dev [nspecies][nnz] CSR
 *     values of the species-block-diagonal Jacobian (device).  Enqueued; ECUDA on launch failure.
 *   landau3d_set_timing / _get_timing: per-stage CUDA-event times of the last build (field, inner,
 *     element, assemble; milliseconds; synchronises the stream when enabled). */
typedef struct landau3d_s *landau3d_t;
int landau3d_create(landau3d_t *out, int32_t ncell, int32_t order, double R, int32_t nspecies, const double *mass,
                    const double *charge, double nu, int32_t cuda_device, void *cuda_stream);
int landau3d_get_sizes(landau3d_t h, int64_t *ndof, int64_t *npoints, int64_t *nnz);
int landau3d_get_pattern(landau3d_t h, int64_t *rowptr, int32_t *col);
int landau3d_get_nodes(landau3d_t h, double *xyz);
int landau3d_jacobian(landau3d_t h, const double *f_dev, double *J_dev);
int landau3d_set_timing(landau3d_t h, int32_t enable);
int landau3d_get_timing(landau3d_t h, float *ms4);
void landau3d_destroy(landau3d_t h);

/* How the last build ran (for FLOP accounting and diagnostics). */
typedef struct {
  int32_t inner_path;        /* 0: directed pair kernel (every ordered pair, split-j when small);
                                1: symmetric pair kernel (every unordered pair once, both targets);
                                2: tensor cache + FP64 GEMM (landau_set_tensor_cache);
                                3: mirror-symmetric pair kernel, partial-sum slots (landau_set_mirror;
                                   with the pair split: this rank's share of the items)
                                4: mirror-symmetric per-vertex kernel (+ slot kernel for a remainder)
                                5: mirror-symmetric directed kernel (single builds, small batches) */
  int64_t nbatch;            /* batch items of the last build                                      */
  int64_t targets;           /* target points per batch item (all N unless element-split)          */
  int64_t sources;           /* source points per batch item (N)                                   */
  int64_t pair_evaluations;  /* pair-body evaluations issued, per batch item, including padded and
                                masked lanes: directed ~ targets x sources, symmetric ~ N^2 / 2    */
  int64_t nsplit;            /* source splits (directed path)                                      */
} landau_stats_t;
int landau_get_stats(landau_t h, landau_stats_t *stats);

const char *landau_strerror(int code);
/* last detailed error message of a handle (or of the last failed create when h == NULL) */
const char *landau_last_error(landau_t h);
const char *landau_version(void);

#ifdef __cplusplus
}
#endif
#endif
