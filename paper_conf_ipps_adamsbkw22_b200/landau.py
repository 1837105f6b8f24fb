"""Thin ctypes binding of liblandau.so (include/landau.h).  Argument marshalling only: every step
of a Jacobian build runs in the library's CUDA kernels.  PyTorch supplies device memory, the stream
and (for the element split) the process group that broadcasts the NCCL id.

There is no CPU fallback: if liblandau.so is missing or a call fails, this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LANDAU_LIB") or os.path.join(_HERE, "liblandau.so")

LANDAU_OK, LANDAU_EINVAL, LANDAU_ENOMEM, LANDAU_ECUDA, LANDAU_ENCCL, LANDAU_ESTATE, LANDAU_EUNSUPPORTED = \
    0, -1, -2, -3, -4, -5, -6
LANDAU_CSR, LANDAU_COO = 0, 1
LANDAU_DIST_REPLICATE, LANDAU_DIST_BATCH, LANDAU_DIST_ELEMENTS = 0, 1, 2
LANDAU_HOST_ONLY = -1
TIMERS = ("field", "inner", "reduce", "element", "assemble", "mass", "allgather", "factor", "solve")

_lib = None


class LandauError(RuntimeError):
    def __init__(self, code, where, detail=""):
        self.code = code
        super().__init__(f"{where}: {landau_strerror(code)} ({code}) {detail}".strip())


class _Mesh(C.Structure):
    _fields_ = [("ngrids", C.c_int32), ("ncells", C.POINTER(C.c_int64)), ("cells", C.POINTER(C.c_double)),
                ("radius", C.POINTER(C.c_double))]


class _Params(C.Structure):
    _fields_ = [("order", C.c_int32), ("nq1d", C.c_int32), ("nspecies", C.c_int32),
                ("mass", C.POINTER(C.c_double)), ("charge", C.POINTER(C.c_double)),
                ("grid", C.POINTER(C.c_int32)), ("nu", C.c_double)]


class _Stats(C.Structure):
    _fields_ = [("inner_path", C.c_int32), ("nbatch", C.c_int64), ("targets", C.c_int64), ("sources", C.c_int64),
                ("pair_evaluations", C.c_int64), ("nsplit", C.c_int64)]


class _Dist(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("nccl_unique_id", C.c_void_p), ("mode", C.c_int32)]


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                              "(no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        vp, i32, i64, d = C.c_void_p, C.c_int32, C.c_int64, C.c_double
        P64, Pd, P32 = C.POINTER(C.c_int64), C.POINTER(C.c_double), C.POINTER(C.c_int32)
        sig = {
            "landau_create": (C.c_int, [C.POINTER(vp), C.POINTER(_Mesh), C.POINTER(_Params), i32, vp, C.POINTER(_Dist)]),
            "landau_destroy": (None, [vp]),
            "landau_get_sizes": (C.c_int, [vp, P64, P64, P64, P64]),
            "landau_get_grid_ndof": (C.c_int, [vp, i32, P64]),
            "landau_get_nodes": (C.c_int, [vp, i32, Pd, Pd]),
            "landau_get_points": (C.c_int, [vp, Pd, Pd, Pd]),
            "landau_get_pattern": (C.c_int, [vp, P64, P32, P32, P32]),
            "landau_set_state": (C.c_int, [vp, vp]),
            "landau_set_state_batched": (C.c_int, [vp, i64, vp]),
            "landau_jacobian": (C.c_int, [vp, vp, i32]),
            "landau_jacobian_batched": (C.c_int, [vp, i64, vp, i32]),
            "landau_jacobian_host": (C.c_int, [vp, i64, vp, vp, i32]),
            "landau_mass": (C.c_int, [vp, d, vp, i32]),
            "landau_point_coeffs": (C.c_int, [vp, vp]),
            "landau_point_coeffs_batched": (C.c_int, [vp, i64, vp]),
            "landau_partition": (C.c_int, [i64, i32, i32, P64, P64]),
            "landau_pair_partition": (C.c_int, [i64, i32, i32, P64, P64]),
            "landau3d_inner": (C.c_int, [i64, vp, vp, vp, vp, vp]),
            "landau3d_create": (C.c_int, [C.POINTER(vp), i32, i32, d, i32, Pd, Pd, d, i32, vp]),
            "landau3d_get_sizes": (C.c_int, [vp, P64, P64, P64]),
            "landau3d_get_pattern": (C.c_int, [vp, P64, P32]),
            "landau3d_get_nodes": (C.c_int, [vp, Pd]),
            "landau3d_jacobian": (C.c_int, [vp, vp, vp]),
            "landau3d_set_timing": (C.c_int, [vp, i32]),
            "landau3d_get_timing": (C.c_int, [vp, C.POINTER(C.c_float)]),
            "landau3d_destroy": (None, [vp]),
            "landau_nccl_unique_id": (C.c_int, [vp]),
            "landau_set_timing": (C.c_int, [vp, i32]),
            "landau_get_timing": (C.c_int, [vp, Pd, P64]),
            "landau_get_launch_count": (C.c_int, [vp, P64]),
            "landau_get_stats": (C.c_int, [vp, C.POINTER(_Stats)]),
            "landau_set_tensor_cache": (C.c_int, [vp, i32]),
            "landau_set_mirror": (C.c_int, [vp, i32]),
            "landau_get_mirror": (C.c_int, [vp, P32, P32]),
            "landau_get_vtx_schedule": (C.c_int, [vp, P32, P32, P32]),
            "landau_get_vtx_split": (C.c_int, [vp, i64, P32, P32]),
            "landau_band_info": (C.c_int, [vp, i32, P32, P32]),
            "landau_band_factor_batched": (C.c_int, [vp, i64, d, vp]),
            "landau_band_solve_batched": (C.c_int, [vp, i64, vp, vp]),
            "landau_band_factor_field_batched": (C.c_int, [vp, i64, d, d, vp]),
            "landau_advection": (C.c_int, [vp, d, vp, i32]),
            "landau_implicit_step_batched": (C.c_int, [vp, i64, d, d, vp, vp, i32, d, P32, Pd]),
            "landau_implicit_step_source_batched": (C.c_int, [vp, i64, d, d, vp, vp, vp, i32, d, P32, Pd]),
            "landau_strerror": (C.c_char_p, [C.c_int]),
            "landau_last_error": (C.c_char_p, [vp]),
            "landau_version": (C.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def landau_strerror(code):
    return lib().landau_strerror(int(code)).decode()


def landau_version():
    return lib().landau_version().decode()


def landau_partition(nelem, world, rank):
    e0, e1 = C.c_int64(), C.c_int64()
    rc = lib().landau_partition(int(nelem), int(world), int(rank), C.byref(e0), C.byref(e1))
    if rc:
        raise LandauError(rc, "landau_partition")
    return e0.value, e1.value


def landau_pair_partition(ntiles, world, rank):
    """Item range [q0, q1) of the pair split (LANDAU_DIST_ELEMENTS on a z-mirror mesh)."""
    q0, q1 = C.c_int64(), C.c_int64()
    rc = lib().landau_pair_partition(int(ntiles), int(world), int(rank), C.byref(q0), C.byref(q1))
    if rc:
        raise LandauError(rc, "landau_pair_partition")
    return q0.value, q1.value


def landau3d_inner(xyz, wTD, wTK, G, stream=None):
    """NEXT-4: 3D Cartesian inner integral on device tensors xyz [3][n], wTD [n], wTK [3][n] -> G [9][n]
    (float64, contiguous, on the current CUDA device)."""
    import torch
    n = int(wTD.numel())
    for t, shape in ((xyz, (3, n)), (wTK, (3, n)), (G, (9, n))):
        if tuple(t.shape) != shape or t.dtype != torch.float64 or not t.is_cuda or not t.is_contiguous():
            raise ValueError(f"landau3d_inner: expected a contiguous float64 CUDA tensor of shape {shape}")
    st = (stream or torch.cuda.current_stream()).cuda_stream
    rc = lib().landau3d_inner(n, xyz.data_ptr(), wTD.data_ptr(), wTK.data_ptr(), G.data_ptr(), st)
    if rc:
        raise LandauError(rc, "landau3d_inner")


class Landau3D:
    """NEXT-4: the 3D Cartesian Landau Jacobian on a uniform grid of ncell^3 Q_p cubes over [-R, R]^3
    (include/landau.h, landau3d_*).  species: sequence of (mass, charge).  Argument marshalling only."""

    def __init__(self, ncell, order, R, species, nu=1.0, device=0, stream=None):
        import torch
        self.device = int(device)
        self.nspecies = len(species)
        mass = np.array([m for m, _ in species], dtype=np.float64)
        charge = np.array([e for _, e in species], dtype=np.float64)
        st = stream.cuda_stream if stream is not None else torch.cuda.current_stream(self.device).cuda_stream
        self.stream = stream
        h = C.c_void_p()
        rc = lib().landau3d_create(C.byref(h), int(ncell), int(order), float(R), self.nspecies, _dptr(mass), _dptr(charge),
                                   float(nu), self.device, C.c_void_p(st))
        if rc:
            raise LandauError(rc, "landau3d_create")
        self._h = h
        a, b, c = C.c_int64(), C.c_int64(), C.c_int64()
        lib().landau3d_get_sizes(h, C.byref(a), C.byref(b), C.byref(c))
        self.ndof, self.npoints, self.nnz = a.value, b.value, c.value

    def close(self):
        if getattr(self, "_h", None):
            lib().landau3d_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def pattern(self):
        rp = np.zeros(self.ndof + 1, dtype=np.int64)
        col = np.zeros(self.nnz, dtype=np.int32)
        lib().landau3d_get_pattern(self._h, rp.ctypes.data_as(C.POINTER(C.c_int64)), col.ctypes.data_as(C.POINTER(C.c_int32)))
        return rp, col

    def nodes(self):
        xyz = np.zeros((3, self.ndof))
        lib().landau3d_get_nodes(self._h, _dptr(xyz))
        return xyz

    def jacobian(self, f, J):
        """f [nspecies][ndof] -> J [nspecies][nnz] (contiguous float64 tensors on the handle's GPU)."""
        for t, n, name in ((f, self.nspecies * self.ndof, "f"), (J, self.nspecies * self.nnz, "J")):
            if not t.is_cuda or t.device.index != self.device or t.numel() != n:
                raise ValueError(f"landau3d_jacobian: {name} must hold {n} values on cuda:{self.device}")
        rc = lib().landau3d_jacobian(self._h, _tptr(f), _tptr(J))
        if rc:
            raise LandauError(rc, "landau3d_jacobian")

    def set_timing(self, on):
        lib().landau3d_set_timing(self._h, int(bool(on)))

    def get_timing(self):
        """per-stage ms of the last timed build: field, inner, element, assemble"""
        ms = (C.c_float * 4)()
        lib().landau3d_get_timing(self._h, ms)
        return dict(zip(("field", "inner", "element", "assemble"), [float(x) for x in ms]))


def landau_nccl_unique_id():
    buf = (C.c_ubyte * 128)()
    rc = lib().landau_nccl_unique_id(buf)
    if rc:
        raise LandauError(rc, "landau_nccl_unique_id")
    return bytes(buf)


def _dptr(a):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _tptr(t, dtype=None):
    """device pointer of a torch tensor (contiguous, float64 unless stated)."""
    import torch
    if not t.is_contiguous():
        raise ValueError("tensor must be contiguous")
    if t.dtype != (dtype or torch.float64):
        raise TypeError(f"expected {dtype or torch.float64}, got {t.dtype}")
    return C.c_void_p(t.data_ptr())


def _host_ptr(t, numel, where):
    """host pointer of a CPU float64 contiguous torch tensor with exactly `numel` elements."""
    import torch
    if t.is_cuda or t.dtype != torch.float64 or not t.is_contiguous():
        raise TypeError(f"{where}: expected a contiguous float64 CPU tensor")
    if t.numel() != numel:
        raise ValueError(f"{where}: expected {numel} elements, got {t.numel()}")
    return C.c_void_p(t.data_ptr())


class Landau:
    """One handle (one mesh, FE order and species set; optional batch of states)."""

    def __init__(self, grids, order, mass, charge, grid_of, nu=1.0, device=0, stream=None, dist=None):
        """grids: list of (R, cells[n][3]); mass/charge/grid_of: per species.  device =
        LANDAU_HOST_ONLY builds only the host plan.  stream: torch.cuda.Stream or raw handle (int)."""
        L = lib()
        ncells = np.array([len(c) for _, c in grids], dtype=np.int64)
        cells = np.ascontiguousarray(np.concatenate([np.asarray(c, dtype=np.float64).reshape(-1, 3) for _, c in grids]))
        radius = np.array([R for R, _ in grids], dtype=np.float64)
        self._keep = [ncells, cells, radius]
        mesh = _Mesh(len(grids), ncells.ctypes.data_as(C.POINTER(C.c_int64)), _dptr(cells), _dptr(radius))
        m = np.ascontiguousarray(mass, dtype=np.float64)
        q = np.ascontiguousarray(charge, dtype=np.float64)
        g = np.ascontiguousarray(grid_of, dtype=np.int32)
        self._keep += [m, q, g]
        prm = _Params(int(order), 0, len(m), _dptr(m), _dptr(q), g.ctypes.data_as(C.POINTER(C.c_int32)), float(nu))
        if stream is None and device != LANDAU_HOST_ONLY:
            import torch
            stream = torch.cuda.current_stream(device)
        if stream is not None and not isinstance(stream, int):
            stream = stream.cuda_stream
        dptr = None
        if dist is not None:
            uid = dist.get("nccl_unique_id")
            self._uid = C.create_string_buffer(uid, 128) if uid else None
            dptr = C.byref(_Dist(int(dist["rank"]), int(dist["world"]),
                                 C.cast(self._uid, C.c_void_p) if self._uid else None, int(dist["mode"])))
        h = C.c_void_p()
        rc = L.landau_create(C.byref(h), C.byref(mesh), C.byref(prm), int(device), C.c_void_p(stream or 0), dptr)
        if rc:
            raise LandauError(rc, "landau_create", L.landau_last_error(None).decode())
        self._h = h
        self.device = device
        a, b, c, d = (C.c_int64() for _ in range(4))
        L.landau_get_sizes(h, C.byref(a), C.byref(b), C.byref(c), C.byref(d))
        self.ndof, self.npoints, self.nnz, self.ncoo = a.value, b.value, c.value, d.value
        self.ngrids = len(grids)
        self.nspecies = len(m)
        self.nbatch = 0

    @classmethod
    def from_problem(cls, prob, device=0, stream=None, dist=None):
        return cls(prob.grids, prob.order, prob.mass, prob.charge, prob.grid_of, prob.nu, device, stream, dist)

    def _check(self, rc, where):
        if rc:
            raise LandauError(rc, where, lib().landau_last_error(self._h).decode())

    def close(self):
        if getattr(self, "_h", None):
            lib().landau_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- host-side queries ---------------------------------------------------------------------
    def grid_ndof(self, g):
        n = C.c_int64()
        self._check(lib().landau_get_grid_ndof(self._h, g, C.byref(n)), "landau_get_grid_ndof")
        return n.value

    def nodes(self, g):
        n = self.grid_ndof(g)
        r, z = np.zeros(n), np.zeros(n)
        self._check(lib().landau_get_nodes(self._h, g, _dptr(r), _dptr(z)), "landau_get_nodes")
        return r, z

    def all_nodes(self):
        return [self.nodes(g) for g in range(self.ngrids)]

    def points(self):
        r, z, w = (np.zeros(self.npoints) for _ in range(3))
        self._check(lib().landau_get_points(self._h, _dptr(r), _dptr(z), _dptr(w)), "landau_get_points")
        return r, z, w

    def pattern(self, coo=False):
        if coo:
            row = np.zeros(max(self.ncoo, 1), dtype=np.int32)
            col = np.zeros(max(self.ncoo, 1), dtype=np.int32)
            self._check(lib().landau_get_pattern(self._h, None, None, row.ctypes.data_as(C.POINTER(C.c_int32)),
                                                 col.ctypes.data_as(C.POINTER(C.c_int32))), "landau_get_pattern")
            return row[: self.ncoo], col[: self.ncoo]
        rp = np.zeros(self.ndof + 1, dtype=np.int64)
        col = np.zeros(max(self.nnz, 1), dtype=np.int32)
        self._check(lib().landau_get_pattern(self._h, rp.ctypes.data_as(C.POINTER(C.c_int64)),
                                             col.ctypes.data_as(C.POINTER(C.c_int32)), None, None), "landau_get_pattern")
        return rp, col[: self.nnz]

    # ---- device calls (torch tensors, float64, on this handle's device) --------------------------
    def _dev(self, t, numel, where):
        """Device pointer of a contiguous float64 CUDA tensor on this handle's device holding exactly
        `numel` elements: the library trusts the sizes it is given, so they are checked here."""
        if not t.is_cuda or t.device.index != self.device:
            raise ValueError(f"{where}: tensor must live on cuda:{self.device}")
        if t.numel() != numel:
            raise ValueError(f"{where}: expected {numel} elements, got {t.numel()} (shape {tuple(t.shape)})")
        return _tptr(t)

    def _nvals(self, format):
        if format not in (LANDAU_CSR, LANDAU_COO):
            raise ValueError(f"unknown format {format!r}")
        return self.nnz if format == LANDAU_CSR else self.ncoo

    @staticmethod
    def _nb(t):
        return t.shape[0] if t.dim() >= 2 else 1

    def set_state(self, f):
        self._check(lib().landau_set_state(self._h, self._dev(f, self.ndof, "set_state")), "landau_set_state")
        self.nbatch = 1

    def set_state_batched(self, f):
        nb = self._nb(f)
        self._check(lib().landau_set_state_batched(self._h, nb, self._dev(f, nb * self.ndof, "set_state_batched")),
                    "landau_set_state_batched")
        self.nbatch = nb

    def jacobian(self, values, format=LANDAU_CSR):
        self._check(lib().landau_jacobian(self._h, self._dev(values, self._nvals(format), "jacobian"), format),
                    "landau_jacobian")
        return values

    def jacobian_batched(self, values, format=LANDAU_CSR):
        nb = self._nb(values)
        self._check(lib().landau_jacobian_batched(self._h, nb, self._dev(values, nb * self._nvals(format),
                                                                         "jacobian_batched"), format),
                    "landau_jacobian_batched")
        return values

    def jacobian_host(self, f_host, values_host, format=LANDAU_CSR):
        """f_host: CPU float64 tensor [nbatch, ndof] (pin it for asynchronous copies); values_host
        [nbatch, nnz] (CSR) or [nbatch, ncoo] (COO), CPU float64."""
        nb = self._nb(f_host)
        fp = _host_ptr(f_host, nb * self.ndof, "jacobian_host f")
        vp_ = _host_ptr(values_host, nb * self._nvals(format), "jacobian_host values")
        self._check(lib().landau_jacobian_host(self._h, nb, fp, vp_, format), "landau_jacobian_host")
        return values_host

    def mass(self, shift, values, format=LANDAU_CSR):
        self._check(lib().landau_mass(self._h, float(shift), self._dev(values, self._nvals(format), "mass"), format),
                    "landau_mass")
        return values

    def point_coeffs(self, G):
        self._check(lib().landau_point_coeffs(self._h, self._dev(G, 5 * self.npoints, "point_coeffs")),
                    "landau_point_coeffs")
        return G

    def point_coeffs_batched(self, G):
        nb = G.shape[0]
        self._check(lib().landau_point_coeffs_batched(self._h, nb, self._dev(G, nb * 5 * self.npoints,
                                                                             "point_coeffs_batched")),
                    "landau_point_coeffs_batched")
        return G

    def set_timing(self, enable=True):
        self._check(lib().landau_set_timing(self._h, int(bool(enable))), "landau_set_timing")

    def get_timing(self):
        ms = np.zeros(len(TIMERS))
        n = np.zeros(len(TIMERS), dtype=np.int64)
        self._check(lib().landau_get_timing(self._h, _dptr(ms), n.ctypes.data_as(C.POINTER(C.c_int64))),
                    "landau_get_timing")
        return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(TIMERS)}

    def band_info(self, g):
        B = C.c_int32()
        perm = np.zeros(self.grid_ndof(g), dtype=np.int32)
        self._check(lib().landau_band_info(self._h, g, C.byref(B), perm.ctypes.data_as(C.POINTER(C.c_int32))),
                    "landau_band_info")
        return B.value, perm

    def band_factor_batched(self, shift, J, Ez=0.0):
        nb = self._nb(J)
        Jp = self._dev(J, nb * self.nnz, "band_factor_batched")
        if Ez == 0.0:
            self._check(lib().landau_band_factor_batched(self._h, nb, float(shift), Jp), "landau_band_factor_batched")
        else:
            self._check(lib().landau_band_factor_field_batched(self._h, nb, float(shift), float(Ez), Jp),
                        "landau_band_factor_field_batched")

    def advection(self, Ez, values, format=LANDAU_CSR):
        self._check(lib().landau_advection(self._h, float(Ez), self._dev(values, self._nvals(format), "advection"),
                                           format), "landau_advection")
        return values

    def implicit_step_batched(self, dt, f_old, f_new, Ez=0.0, max_iter=4, rtol=0.0, src=None):
        """One backward-Euler step by quasi-Newton (include/landau.h); src: the FE coefficients of the
        source S_a(t^{n+1}) (same shape as f_old) or None.  Returns (iterations, max rel. change)."""
        nb = self._nb(f_old)
        it, dn = C.c_int32(), C.c_double()
        fo = self._dev(f_old, nb * self.ndof, "implicit_step f_old")
        fn = self._dev(f_new, nb * self.ndof, "implicit_step f_new")
        if src is None:
            rc = lib().landau_implicit_step_batched(self._h, nb, float(dt), float(Ez), fo, fn, int(max_iter),
                                                    float(rtol), C.byref(it), C.byref(dn))
        else:
            sp = self._dev(src, nb * self.ndof, "implicit_step src")
            rc = lib().landau_implicit_step_source_batched(self._h, nb, float(dt), float(Ez), fo, sp, fn, int(max_iter),
                                                           float(rtol), C.byref(it), C.byref(dn))
        self._check(rc, "landau_implicit_step_batched")
        return it.value, dn.value

    def band_solve_batched(self, b, x):
        nb = self._nb(b)
        self._check(lib().landau_band_solve_batched(self._h, nb, self._dev(b, nb * self.ndof, "band_solve b"),
                                                    self._dev(x, nb * self.ndof, "band_solve x")),
                    "landau_band_solve_batched")
        return x

    def set_mirror(self, enable=True):
        """False: plain symmetric kernel; True: mirror kernel (auto: per-vertex for large batches);
        "slots": mirror kernel with HBM partial slots; "vertex": per-vertex mirror kernel."""
        mode = {"slots": 2, "vertex": 3}.get(enable) if isinstance(enable, str) else int(bool(enable))
        if mode is None:
            raise ValueError(f"set_mirror: unknown mode {enable!r}")
        self._check(lib().landau_set_mirror(self._h, mode), "landau_set_mirror")

    def mirror(self):
        """(exactly z-mirror-symmetric mesh, mirror kernels in use) -- see landau_get_mirror."""
        a, b = C.c_int32(), C.c_int32()
        self._check(lib().landau_get_mirror(self._h, C.byref(a), C.byref(b)), "landau_get_mirror")
        return bool(a.value), bool(b.value)

    def vtx_schedule(self):
        """(round weight prefix [nrounds + 1], CTAs of an automatic launch) of the per-vertex kernel."""
        nr, ct = C.c_int32(), C.c_int32()
        self._check(lib().landau_get_vtx_schedule(self._h, C.byref(nr), None, None), "landau_get_vtx_schedule")
        wp = np.zeros(nr.value + 1, dtype=np.int32)
        self._check(lib().landau_get_vtx_schedule(self._h, None, wp.ctypes.data_as(C.POINTER(C.c_int32)),
                                                  C.byref(ct)), "landau_get_vtx_schedule")
        return wp, ct.value

    def vtx_split_vertices(self, nbatch):
        """Batch items whose rounds an automatic-mode build spreads over more than one CTA."""
        first, last = np.zeros(nbatch, dtype=np.int32), np.zeros(nbatch, dtype=np.int32)
        self._check(lib().landau_get_vtx_split(self._h, int(nbatch), first.ctypes.data_as(C.POINTER(C.c_int32)),
                                               last.ctypes.data_as(C.POINTER(C.c_int32))), "landau_get_vtx_split")
        return np.nonzero(first != last)[0]

    def set_tensor_cache(self, enable=True):
        """True: cache the tensors across builds; "recompute": GEMM path, tensors evaluated every build."""
        mode = 2 if enable == "recompute" else int(bool(enable))
        self._check(lib().landau_set_tensor_cache(self._h, mode), "landau_set_tensor_cache")

    def stats(self):
        st = _Stats()
        self._check(lib().landau_get_stats(self._h, C.byref(st)), "landau_get_stats")
        return {k: getattr(st, k) for k, _ in _Stats._fields_}

    def launch_count(self):
        n = C.c_int64()
        self._check(lib().landau_get_launch_count(self._h, C.byref(n)), "landau_get_launch_count")
        return n.value


# ------------------------------------------------------------------------------------------------
# multi-process helpers (host logic only; the data path never leaves the library)
# ------------------------------------------------------------------------------------------------
def batch_range(nbatch, world, rank):
    """Contiguous share [lo, hi) of a batch of independent vertices for one rank (C4 sharding)."""
    return rank * nbatch // world, (rank + 1) * nbatch // world


def chunk_points(ncell, nqp, world):
    """Points per rank chunk of the element split's G exchange (cells are split by landau_partition)."""
    e0, e1 = landau_partition(ncell, world, 0)
    return (e1 - e0) * nqp


def make_dist(mode, group=None):
    """dist descriptor for Landau(...): rank/world from torch.distributed; for the element split, rank 0
    creates the NCCL id through the library and the process group broadcasts it."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    uid = None
    if mode == LANDAU_DIST_ELEMENTS:
        obj = [landau_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        uid = obj[0]
    return {"rank": rank, "world": world, "mode": mode, "nccl_unique_id": uid}
