// host_setup.h -- step a-0 of SURVEY.md §8(a): everything the device kernels need that depends only
// on the mesh, the order and the species (built once per handle, on the host, in C++17).
//
//   * quadtree validation (lattice alignment, no overlap, full tiling, 2:1 edge balance; Amb-10)
//   * Gauss-Legendre points/weights and Q_p tables at the reference points (Amb-8, Amb-9)
//   * DOF numbering: non-hanging node positions ordered by (z, r) (Amb-12)
//   * hanging-node extraction P_e: a node inside a coarser neighbour's edge takes that edge's
//     degree-p Lagrange interpolant ("interpolate ... to four DOFs" for Q3, PAPER.md:1@42262)
//   * CSR pattern (species-block-diagonal, @11277), COO layout, and the deterministic gather maps
//     that replace the paper's atomic MatSetValues (@23291-24297, Amb-15).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace landau {

struct GridPlan {
  double R = 0;
  int64_t cell0 = 0;        // first global cell index
  int64_t ncell = 0;
  int64_t pt0 = 0;          // first global point index
  int ndof = 0;
  std::vector<double> node_r, node_z;   // [ndof]
  // per cell: sorted distinct DOFs and dense extraction P[Nb][n_e]
  std::vector<int> ne;                   // [ncell]
  std::vector<int64_t> edof_off;         // [ncell+1]
  std::vector<int> edof;                 // distinct DOFs
  std::vector<int64_t> P_off;            // [ncell+1]
  std::vector<double> P;                 // Nb * n_e per cell
  // CSR pattern of one species block
  std::vector<int64_t> rowptr;           // [ndof+1]
  std::vector<int> col;
  int64_t ncoo = 0;                      // sum_e n_e^2
  // NEXT-2 band solver (PAPER.md:1@25294): reverse Cuthill-McKee ordering of this grid's DOF graph
  std::vector<int> rcm_perm;             // [ndof] new -> old
  std::vector<int> rcm_iperm;            // [ndof] old -> new
  int band = 0;                          // half-bandwidth B = max |iperm(i) - iperm(j)| over the pattern
  // Entries in the order the register-window factorisation consumes them, relative to the padded
  // half-bandwidth Bp = (B + 1 rounded up to 8) - 1: RCM row i "enters" with its lower row part
  // A(i, j), j <= i (pos = j - i + Bp in 0..Bp) and its upper column part A(j, i), j < i
  // (pos = Bp + 1 + j - i + Bp in Bp+1..2Bp).  ent_slot = CSR slot of the entry; ent_pos stores
  // (i mod 8) (2 Bp + 1) + pos, the entry's place in the dense buffer of its group of 8 rows.
  int band_p = 0;
  std::vector<int32_t> ent_ptr;          // [ndof+1]
  std::vector<int32_t> ent_slot;         // [nnz]
  std::vector<uint16_t> ent_pos;         // [nnz]
  int ent_max = 0;                       // max entries of one entering row
};

// A gather map: output slot s = sum over its contributions (idx, w) of w * Celem[idx], in a fixed
// order (cell, a, b).  idx = e * 2 Nb^2 + 2 (a * Nb + b) indexes the [cell][Nb][Nb][2] element buffer
// (C^D and C^K of an entry side by side: one 16-byte load per contribution).
struct GatherMap {
  std::vector<int64_t> ptr;   // [nslots+1]
  std::vector<int32_t> idx;
  std::vector<double> w;
};

struct Plan {
  int p = 0, nq = 0, nb = 0, nqp = 0;
  int ngrids = 0, nspecies = 0;
  int64_t ncell = 0, npts = 0;
  std::vector<GridPlan> grids;
  // global per cell
  std::vector<double> cell_h;            // [ncell]
  std::vector<int> cell_grid;            // [ncell]
  // global per point
  std::vector<double> pr, pz, pw;        // [npts]
  // reference tables at the Gauss points: [nqp][nb]
  std::vector<double> tab_phi, tab_dxi, tab_deta;
  // their 1-D factors (q = qz * nq + qr, node n = b * (p+1) + a): l_a(x_i), l'_a(x_i) as [i][a]
  std::vector<double> tab1_L, tab1_D;
  // field extraction per cell-local node: ext_ptr[ncell*nb+1] -> (dof in its grid, weight)
  std::vector<int32_t> ext_ptr, ext_dof;
  std::vector<double> ext_w;
  // gather maps per grid (CSR slots, COO slots)
  std::vector<GatherMap> csr_map, coo_map;
};

// Phased gather maps of the fused element + assembly kernel (tail_kernel, kernels_fe.cuh): each grid's
// cells are cut into phases of at most `cap` consecutive cells (input order, so every slot's
// contributions -- listed in (cell, a, b) order by the gather map -- arrive phase after phase and a
// slot straddling phases continues one fma chain: the result equals assemble_kernel's bit for bit).  A
// phase's element matrices live in shared memory, cell c of the phase at offset c * 2 Nb^2.  Per phase,
// the output slots it touches (sorted) with their contributions in the phase: the first four inline
// (ELL layout: one 16-byte index quad and two 16-byte weight pairs per slot, independent coalesced
// loads), the rest in an overflow list.  meta = (slot, mode | n_inline << 2 | cross id << 5), mode 0: every
// contribution in this phase (write), 1: first phase of a straddling slot (keep the running sum in
// shared memory under the cross id), 2: middle (continue it), 3: last (continue it and write).
struct PhaseMaps {
  std::vector<int32_t> grid_phase_ptr;   // [ngrids + 1] phases of each grid
  std::vector<int32_t> cell_ptr;         // [nphases + 1] first cell (global index) of each phase, + end
  std::vector<int32_t> slot_ptr;         // [nphases + 1] into the per-slot arrays
  std::vector<int32_t> meta;             // [2 * total phase slots] (slot, mode | n_inline << 2 | x << 5)
  std::vector<int32_t> idx4;             // [4 * total] the four inline element-matrix indices (doubles)
  std::vector<double> w4;                // [4 * total] their weights
  std::vector<int32_t> optr;             // [2 * total] overflow range [begin, end) into oidx / ow
  std::vector<int32_t> oidx;
  std::vector<double> ow;
  int max_cells = 0, max_cross = 0;
};
// cap >= 1 cells per phase; returns "" or an error (more than INT32_MAX entries).
std::string build_phase_maps(const Plan &plan, const std::vector<GatherMap> &maps, int cap, PhaseMaps &out);

// NEXT-4 completed: the 3D Cartesian model on a uniform grid of ncell^3 Q_p cubes over [-R, R]^3
// (kernels_3d_fe.cuh).  DOFs: the lattice of M = ncell p + 1 nodes per direction,
// dof(ix, iy, iz) = (iz M + iy) M + ix; points cube-major, q = (a S + b) S + c (Gauss indices along
// z, y, x), w = w_a w_b w_c (h/2)^3; local node n = (k S + j) S + i.  The CSR pattern: rows and
// columns ascending (the tensor product of the 1-D patterns); the gather map lists, per CSR slot, the
// element-buffer entries e 2 NB^2 + 2 (k NB + l) of every cube holding both DOFs, in cube order,
// weight 1 (no constraints on a uniform grid).
struct Plan3D {
  int ncell = 0, p = 0, s1 = 0, nb = 0;
  double R = 0.0, h = 0.0;
  int64_t ndof = 0, npts = 0, nnz = 0;
  std::vector<double> L1, D1;            // [S][S]: l_a(x_i), l'_a(x_i) at [i * S + a]
  std::vector<double> xyz, w;            // [3][npts], [npts]
  std::vector<int32_t> dofs;             // [ncube][nb]
  std::vector<int64_t> rowptr;           // [ndof + 1]
  std::vector<int32_t> col;              // [nnz]
  GatherMap map;                         // [nnz] slots
};
std::string build_plan3d(int ncell, int order, double R, Plan3D &plan);

// Build the plan.  Returns "" on success or an error message (the mesh is invalid).
std::string build_plan(int ngrids, const int64_t *ncells, const double *cells, const double *radius, int order,
                       Plan &plan);

}  // namespace landau
