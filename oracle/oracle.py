"""ctypes wrapper of liboracle.so -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may import
this module.  It shares nothing with the CUDA path except the seeded input generators
(paper_conf_ipps_adamsbkw22_b200/inputs.py, which hold no method arithmetic).
See oracle.h for what each call computes and which passage of the paper it follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

_d = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_i64 = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
_i32 = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
_u8 = np.ctypeslib.ndpointer(dtype=np.uint8, flags="C_CONTIGUOUS")


def build():
    subprocess.run(["make", "-s", "-C", _HERE], check=True)


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            build()
        L = C.CDLL(path)
        vp = C.c_void_p
        L.oracle_create.restype = vp
        L.oracle_create.argtypes = [C.c_int, _i64, _d, _d, C.c_int, C.c_int, C.c_int, _d, _d, _i32,
                                    C.c_double, C.c_char_p, C.c_int]
        L.oracle_destroy.argtypes = [vp]
        P64 = C.POINTER(C.c_longlong)
        L.oracle_sizes.argtypes = [vp, P64, P64, P64, P64]
        L.oracle_grid_ndof.restype = C.c_longlong
        L.oracle_grid_ndof.argtypes = [vp, C.c_int]
        L.oracle_grid_npoints.restype = C.c_longlong
        L.oracle_grid_npoints.argtypes = [vp, C.c_int]
        L.oracle_grid_nodes.argtypes = [vp, C.c_int, _d, _d]
        L.oracle_points.argtypes = [vp, _d, _d, _d]
        L.oracle_pattern.argtypes = [vp, _i64, _i32]
        L.oracle_coo_pattern.argtypes = [vp, _i32, _i32]
        L.oracle_tensor.argtypes = [C.c_double, C.c_double, C.c_double, C.c_double, _d]
        L.oracle_inner.argtypes = [C.c_longlong, _d, _d, _d, _d, _d, _d, C.c_longlong, vp, vp, vp]
        L.oracle_point_fields.argtypes = [vp, _d, _d, _d, _d]
        L.oracle_point_coeffs.argtypes = [vp, _d, C.c_longlong, vp, vp, vp]
        L.oracle_jacobian.argtypes = [vp, _d, _d, _d]
        L.oracle_jacobian_coo.argtypes = [vp, _d, vp, _d, _d]
        L.oracle_mass.argtypes = [vp, C.c_double, _d]
        L.oracle_mass_coo.argtypes = [vp, C.c_double, _d]
        L.oracle_advection.argtypes = [vp, _d]
        L.oracle_advection_coo.argtypes = [vp, _d]
        L.oracle_tensor3d.argtypes = [C.c_double, C.c_double, C.c_double, _d]
        L.oracle_inner3d.argtypes = [C.c_longlong, _d, _d, _d, _d, _d, _d, _d, _d, _d]
        L.oracle3d_sizes.argtypes = [C.c_int, C.c_int, P64, P64, P64]
        L.oracle3d_pattern.argtypes = [C.c_int, C.c_int, _i64, _i32]
        L.oracle3d_nodes.argtypes = [C.c_int, C.c_int, C.c_double, _d]
        L.oracle3d_jacobian.argtypes = [C.c_int, C.c_int, C.c_double, C.c_int, _d, _d, C.c_double, _d, _d, _d]
        L.oracle3d_points.argtypes = [C.c_int, C.c_int, C.c_double, _d, _d]
        L.oracle3d_fields.argtypes = [C.c_int, C.c_int, C.c_double, C.c_int, _d, _d, _d, _d]
        L.oracle3d_assemble.argtypes = [C.c_int, C.c_int, C.c_double, C.c_int, _d, _d, C.c_double, _d, _d]
        L.oracle_set_threads.argtypes = [C.c_int]
        L.oracle_get_threads.restype = C.c_int
        _LIB = L
    return _LIB


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def tensor(r, z, rb, zb):
    out = np.zeros(5)
    lib().oracle_tensor(float(r), float(z), float(rb), float(zb), out)
    return out


def tensor3d(u):
    """O12: the 3D Cartesian Landau tensor U(u) of Eq. 3 as (xx, xy, xz, yy, yz, zz)."""
    out = np.zeros(6)
    lib().oracle_tensor3d(float(u[0]), float(u[1]), float(u[2]), out)
    return out


def inner3d(x, y, z, wTD, wTK):
    """O12: (G [9][n], Gabs [9][n]) of the 3D Cartesian inner integral (wTK: [3][n])."""
    x, y, z, wTD = (np.ascontiguousarray(a, dtype=np.float64) for a in (x, y, z, wTD))
    wTK = np.ascontiguousarray(wTK, dtype=np.float64)
    n = x.size
    G = np.zeros(9 * n)
    Ga = np.zeros(9 * n)
    lib().oracle_inner3d(n, x, y, z, wTD, wTK[0].copy(), wTK[1].copy(), wTK[2].copy(), G, Ga)
    return G.reshape(9, n), Ga.reshape(9, n)


def inner(r, z, w, TD, TKr, TKz, targets=None, with_abs=False):
    r, z, w, TD, TKr, TKz = (np.ascontiguousarray(a, dtype=np.float64) for a in (r, z, w, TD, TKr, TKz))
    n = r.size
    tg = None if targets is None else np.ascontiguousarray(targets, dtype=np.int64)
    nt = n if tg is None else tg.size
    G = np.zeros((5, nt))
    Ga = np.zeros((5, nt)) if with_abs else None
    lib().oracle_inner(n, r, z, w, TD, TKr, TKz, nt, _ptr(tg), _ptr(G), _ptr(Ga))
    return (G, Ga) if with_abs else G


def set_threads(n):
    lib().oracle_set_threads(int(n))


def get_threads():
    return int(lib().oracle_get_threads())


class Oracle:
    """The whole O0-O10 pipeline for one Problem (paper_conf_ipps_adamsbkw22_b200.inputs.Problem)."""

    def __init__(self, prob, nq1d: int = 0):
        L = lib()
        err = C.create_string_buffer(256)
        self.prob = prob
        self._h = L.oracle_create(len(prob.grids), prob.ncells, prob.cells, prob.radius, prob.order, nq1d,
                                  len(prob.species), prob.mass, prob.charge, prob.grid_of, prob.nu, err, 256)
        if not self._h:
            raise ValueError("oracle_create: " + err.value.decode())
        a, b, c, d = (C.c_longlong() for _ in range(4))
        L.oracle_sizes(self._h, C.byref(a), C.byref(b), C.byref(c), C.byref(d))
        self.ndof, self.npoints, self.nnz, self.ncoo = a.value, b.value, c.value, d.value

    def __del__(self):
        if getattr(self, "_h", None) and _LIB is not None:
            _LIB.oracle_destroy(self._h)
            self._h = None

    def grid_ndof(self, g):
        return int(lib().oracle_grid_ndof(self._h, g))

    def nodes(self, g):
        n = self.grid_ndof(g)
        r, z = np.zeros(n), np.zeros(n)
        lib().oracle_grid_nodes(self._h, g, r, z)
        return r, z

    def all_nodes(self):
        return [self.nodes(g) for g in range(len(self.prob.grids))]

    def points(self):
        r, z, w = (np.zeros(self.npoints) for _ in range(3))
        lib().oracle_points(self._h, r, z, w)
        return r, z, w

    def pattern(self):
        rp = np.zeros(self.ndof + 1, dtype=np.int64)
        col = np.zeros(max(self.nnz, 1), dtype=np.int32)
        lib().oracle_pattern(self._h, rp, col)
        return rp, col[: self.nnz]

    def coo_pattern(self):
        row = np.zeros(max(self.ncoo, 1), dtype=np.int32)
        col = np.zeros(max(self.ncoo, 1), dtype=np.int32)
        lib().oracle_coo_pattern(self._h, row, col)
        return row[: self.ncoo], col[: self.ncoo]

    def point_fields(self, f):
        f = np.ascontiguousarray(f, dtype=np.float64)
        TD, TKr, TKz = (np.zeros(self.npoints) for _ in range(3))
        lib().oracle_point_fields(self._h, f, TD, TKr, TKz)
        return TD, TKr, TKz

    def point_coeffs(self, f, targets=None):
        f = np.ascontiguousarray(f, dtype=np.float64)
        tg = None if targets is None else np.ascontiguousarray(targets, dtype=np.int64)
        nt = self.npoints if tg is None else tg.size
        G, Ga = np.zeros((5, nt)), np.zeros((5, nt))
        lib().oracle_point_coeffs(self._h, f, nt, _ptr(tg), _ptr(G), _ptr(Ga))
        return G, Ga

    def jacobian(self, f):
        f = np.ascontiguousarray(f, dtype=np.float64)
        v, va = np.zeros(max(self.nnz, 1)), np.zeros(max(self.nnz, 1))
        lib().oracle_jacobian(self._h, f, v, va)
        return v[: self.nnz], va[: self.nnz]

    def jacobian_coo(self, f, elem_mask=None):
        f = np.ascontiguousarray(f, dtype=np.float64)
        m = None if elem_mask is None else np.ascontiguousarray(elem_mask, dtype=np.uint8)
        v, va = np.full(max(self.ncoo, 1), np.nan), np.full(max(self.ncoo, 1), np.nan)
        lib().oracle_jacobian_coo(self._h, f, _ptr(m), v, va)
        return v[: self.ncoo], va[: self.ncoo]

    def mass(self, shift=1.0):
        v = np.zeros(max(self.nnz, 1))
        lib().oracle_mass(self._h, float(shift), v)
        return v[: self.nnz]

    def mass_coo(self, shift=1.0):
        v = np.zeros(max(self.ncoo, 1))
        lib().oracle_mass_coo(self._h, float(shift), v)
        return v[: self.ncoo]

    def advection(self):
        """O11: unscaled E_z advection matrix (CSR values, every species block)."""
        v = np.zeros(max(self.nnz, 1))
        lib().oracle_advection(self._h, v)
        return v[: self.nnz]

    def advection_coo(self):
        v = np.zeros(max(self.ncoo, 1))
        lib().oracle_advection_coo(self._h, v)
        return v[: self.ncoo]

    def species_rows(self):
        """species index of every row of the block-diagonal system (species-major blocks, @11277)"""
        return np.concatenate([np.full(self.grid_ndof(int(g)), a, dtype=np.int64)
                               for a, g in enumerate(self.prob.grid_of)])

    def implicit_step(self, f_old, dt, Ez=0.0, iters=4, src=None):
        """Backward-Euler step of Eq. 4 by the paper's quasi-Newton iteration (@10500-10978): with the
        Jacobian J(f^k) recomputed about the current iterate,
            (M/dt + E_z (e_a/m_a) A_E - J(f^k)) f^{k+1} = M f^old / dt + M sigma,
        i.e. Newton on F(f) = M (f - f^old)/dt + E_z (e/m) A_E f - C(f) - (psi, S) with the approximate
        Jacobian M/dt + E_z (e/m) A_E - J(f^k) (C(f^k) = J(f^k) f^k, Amb-4).  sigma: the FE coefficients
        of the source S_a(t^{n+1}) of Eq. 1 / Eq. 4 (None: no source); (psi_k, S_a) = (M sigma)_k, the
        weighted L2 product of the mass matrix (Amb-2, R-7).  A sparse direct solve (a library
        primitive) stands in for the paper's band LU.  Returns the iterates f^1..f^iters."""
        import scipy.sparse as sps
        import scipy.sparse.linalg as spla
        rp, col = self.pattern()
        n = self.ndof
        M, Ae = self.mass(1.0), self.advection()
        rows = np.repeat(np.arange(n), np.diff(rp))
        eta = Ez * (np.asarray(self.prob.charge, float) / np.asarray(self.prob.mass, float))[self.species_rows()]
        Mm = sps.csr_matrix((M, col, rp), shape=(n, n))
        b = Mm @ np.asarray(f_old, float) / dt
        if src is not None:
            b = b + Mm @ np.asarray(src, float)
        f = np.array(f_old, dtype=np.float64)
        out = []
        for _ in range(iters):
            J, _ = self.jacobian(f)
            A = sps.csr_matrix((M / dt + eta[rows] * Ae - J, col, rp), shape=(n, n))
            f = spla.spsolve(A.tocsc(), b)
            out.append(f.copy())
        return out

    def coefficients(self, with_noise=True):
        from paper_conf_ipps_adamsbkw22_b200 import inputs
        return inputs.coefficients(self.prob, self.all_nodes(), with_noise)


class Oracle3D:
    """O13: the 3D Cartesian Landau Jacobian on a uniform grid of ncell^3 Q_p cubes over [-R, R]^3
    (oracle.h).  species: sequence of (mass, charge)."""

    def __init__(self, ncell, order, R, species, nu=1.0):
        self.ncell, self.order, self.R, self.nu = int(ncell), int(order), float(R), float(nu)
        self.mass = np.array([m for m, _ in species], dtype=np.float64)
        self.charge = np.array([e for _, e in species], dtype=np.float64)
        a, b, c = (C.c_longlong() for _ in range(3))
        lib().oracle3d_sizes(self.ncell, self.order, C.byref(a), C.byref(b), C.byref(c))
        self.ndof, self.npoints, self.nnz = a.value, b.value, c.value

    def pattern(self):
        rp = np.zeros(self.ndof + 1, dtype=np.int64)
        col = np.zeros(self.nnz, dtype=np.int32)
        lib().oracle3d_pattern(self.ncell, self.order, rp, col)
        return rp, col

    def nodes(self):
        xyz = np.zeros((3, self.ndof))
        lib().oracle3d_nodes(self.ncell, self.order, self.R, xyz)
        return xyz

    def points(self):
        xyz, w = np.zeros((3, self.npoints)), np.zeros(self.npoints)
        lib().oracle3d_points(self.ncell, self.order, self.R, xyz, w)
        return xyz, w

    def fields(self, f):
        """O3/O4: [4][npoints] = T_D, T_K (x, y, z), not multiplied by w"""
        S = self.mass.size
        f = np.ascontiguousarray(f, dtype=np.float64).reshape(S, self.ndof)
        T = np.zeros((4, self.npoints))
        lib().oracle3d_fields(self.ncell, self.order, self.R, S, self.mass, self.charge, f, T)
        return T

    def assemble(self, G):
        """O6-O8 from a given G [9][npoints] -> [S][nnz]"""
        S = self.mass.size
        v = np.zeros((S, self.nnz))
        lib().oracle3d_assemble(self.ncell, self.order, self.R, S, self.mass, self.charge, self.nu,
                                np.ascontiguousarray(G, dtype=np.float64), v)
        return v

    def jacobian(self, f):
        """f [S][ndof] -> (J, J^abs), each [S][nnz]"""
        S = self.mass.size
        f = np.ascontiguousarray(f, dtype=np.float64).reshape(S, self.ndof)
        v, va = np.zeros((S, self.nnz)), np.zeros((S, self.nnz))
        lib().oracle3d_jacobian(self.ncell, self.order, self.R, S, self.mass, self.charge, self.nu, f, v, va)
        return v, va
