"""CPU tests of the C ABI (no GPU): the library loads and exports every symbol include/landau.h
declares; the host-side plan (step a-0: nodes, DOF numbering, points, CSR/COO patterns) agrees with
the independent oracle; invalid meshes are rejected; the element partition is a partition."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "landau.h")).read()
    return sorted(set(re.findall(r"^\s*(?:int|void|const char \*)\s*(landau(?:_|3d_)\w+)\s*\(", txt, re.M)))


def test_library_exports_every_declared_symbol():
    syms = header_symbols()
    assert len(syms) >= 20
    out = subprocess.run(["nm", "-D", "--defined-only", L.LIB_PATH], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (landau(?:_|3d_)\w+)", out))
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    lib = ctypes.CDLL(L.LIB_PATH)
    for s in syms:
        getattr(lib, s)


def test_strerror_and_version():
    assert "invalid" in L.landau_strerror(L.LANDAU_EINVAL)
    assert "sm_100a" in L.landau_version()


@pytest.mark.parametrize("nelem,world", [(68, 1), (68, 2), (4352, 8), (7, 3), (3, 8)])
def test_partition_covers_cells_once(nelem, world):
    seen = np.zeros(nelem, dtype=int)
    for r in range(world):
        e0, e1 = L.landau_partition(nelem, world, r)
        assert 0 <= e0 <= e1 <= nelem
        seen[e0:e1] += 1
    assert np.all(seen == 1)
    with pytest.raises(L.LandauError):
        L.landau_partition(nelem, world, world)


@pytest.mark.parametrize("ntiles,world", [(17, 1), (17, 2), (1700, 8), (5, 3), (2, 8), (0, 2)])
def test_pair_partition_covers_items_once_balanced(ntiles, world):
    """Pair split: the ranks' item ranges tile [0, T(T+1)/2) in order, and each rank's weight (2 per
    tile pair, 1 per diagonal item) is within one pair of T^2 / world."""
    items = [(a, b) for b in range(ntiles) for a in range(b + 1)]
    wt = np.array([1 if a == b else 2 for a, b in items], dtype=np.int64)
    prev = 0
    for r in range(world):
        q0, q1 = L.landau_pair_partition(ntiles, world, r)
        assert q0 == prev and q0 <= q1 <= len(items)
        prev = q1
        if len(items) and world <= len(items):
            assert abs(int(wt[q0:q1].sum()) - ntiles * ntiles / world) <= 2
    assert prev == len(items)
    for bad in ((ntiles, world, world), (ntiles, 0, 0), (-1, world, 0)):
        with pytest.raises(L.LandauError):
            L.landau_pair_partition(*bad)


def _host(prob):
    return L.Landau.from_problem(prob, device=L.LANDAU_HOST_ONLY)


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_host_plan_matches_oracle(cfg):
    from oracle.oracle import Oracle
    prob = inputs.CONFIGS[cfg]()
    h = _host(prob)
    o = Oracle(prob)
    assert (h.ndof, h.npoints, h.nnz, h.ncoo) == (o.ndof, o.npoints, o.nnz, o.ncoo)
    for g in range(len(prob.grids)):
        hr, hz = h.nodes(g)
        orr, oz = o.nodes(g)
        np.testing.assert_allclose(hr, orr, rtol=0, atol=1e-14 * prob.grids[g][0])
        np.testing.assert_allclose(hz, oz, rtol=0, atol=1e-14 * prob.grids[g][0])
    hr, hz, hw = h.points()
    orr, oz, ow = o.points()
    np.testing.assert_allclose(hr, orr, rtol=1e-15, atol=0)
    np.testing.assert_allclose(hz, oz, rtol=1e-15, atol=1e-16)
    np.testing.assert_allclose(hw, ow, rtol=4e-15)
    rp, col = h.pattern()
    orp, ocol = o.pattern()
    np.testing.assert_array_equal(rp, orp)
    np.testing.assert_array_equal(col, ocol)
    row, col = h.pattern(coo=True)
    orow, ocol = o.coo_pattern()
    np.testing.assert_array_equal(row, orow)
    np.testing.assert_array_equal(col, ocol)


def test_host_plan_C5_sizes():
    prob = inputs.config5()
    h = _host(prob)
    assert h.npoints == 108800 and len(prob.grids[0][1]) == 4352


def test_invalid_meshes_rejected():
    R = 1.0
    base = inputs.origin_chain(R, 2)
    c0 = [c for c in base if c[0] == 0.0 and c[1] == 0.0][0]
    unbalanced = [c for c in base if c != c0] + inputs.refine_uniform([c0], 2)
    bad = {
        "unbalanced": unbalanced,
        "overlap": base + [(0.0, 0.0, R / 8)],
        "hole": base[1:],
        "off-lattice": [(0.0, -R, R), (0.0, 0.0, R / 2), (R / 2, 0.0, R / 2), (0.1, R / 2, R / 2), (R / 2, R / 2, R / 2)],
        "negative r": [(-R, -R, R), (0.0, 0.0, R)],
    }
    for name, cells in bad.items():
        prob = inputs.Problem("bad", 3, [(R, cells)], [inputs.Species("e", 1.0, -1.0, 0)], fmix=[[(1, 1, 0)]])
        with pytest.raises(L.LandauError) as ei:
            _host(prob)
        assert ei.value.code == L.LANDAU_EINVAL, name
    prob = inputs.Problem("ok", 5, [(R, base)], [inputs.Species("e", 1.0, -1.0, 0)], fmix=[[(1, 1, 0)]])
    with pytest.raises(L.LandauError):
        _host(prob)                       # order 5 unsupported
    prob = inputs.Problem("ok", 3, [(R, base)], [inputs.Species("e", -1.0, -1.0, 0)], fmix=[[(1, 1, 0)]])
    with pytest.raises(L.LandauError):
        _host(prob)                       # negative mass


def test_host_only_handle_refuses_device_calls():
    h = _host(inputs.config1())
    lib = L.lib()
    rc = lib.landau_mass(h._h, 1.0, ctypes.c_void_p(16), L.LANDAU_CSR)
    assert rc == L.LANDAU_EUNSUPPORTED


def test_create_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(L.LandauError) as ei:
        L.Landau.from_problem(inputs.config1(), device=0, stream=0)
    assert ei.value.code == L.LANDAU_ECUDA


def test_argument_errors_without_gpu():
    """Error codes the header documents, checked before any device work: set_mirror outside 0..3 is
    EINVAL and the mirror on a host-only handle (no mirror maps) EUNSUPPORTED; landau3d_inner with
    n < 0 or NULL pointers is EINVAL and with n = 0 a no-op."""
    h = _host(inputs.config1())
    lib = L.lib()
    assert lib.landau_set_mirror(h._h, 7) == L.LANDAU_EINVAL
    assert lib.landau_set_mirror(h._h, -1) == L.LANDAU_EINVAL
    assert lib.landau_set_mirror(h._h, 1) == L.LANDAU_EUNSUPPORTED
    assert lib.landau3d_inner(-1, None, None, None, None, None) == L.LANDAU_EINVAL
    assert lib.landau3d_inner(5, None, None, None, None, None) == L.LANDAU_EINVAL
    assert lib.landau3d_inner(0, None, None, None, None, None) == L.LANDAU_OK


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C5"])
def test_mirror_detection_is_bit_exact(cfg):
    """Every configuration's mesh is exactly z-mirror-symmetric in floating point (dyadic radius,
    cell-centre point formula), so the mirror kernels compute at the caller's own points: each point
    (r, z) has a partner with bit-identical r and z' == -z."""
    h = _host(inputs.CONFIGS[cfg]())
    sym, active = h.mirror()
    assert sym and not active          # host-only handle: detected, no device maps
    r, z, _ = h.points()
    pts = set(zip(r.tolist(), z.tolist()))
    assert all((a, -b) in pts for a, b in zip(r.tolist(), z.tolist()))


@pytest.mark.parametrize("shift", [1e-13, -2e-15, 1e-10])
def test_mirror_detection_refuses_near_symmetric_mesh(shift):
    """A mesh shifted by a few ulps-to-1e-10 R along z is still a valid quadtree (the cell lattice check
    has a 1e-6 tolerance) but no longer exactly mirror-symmetric: the mirror kernels must not be used
    (they would evaluate tensors at (r, -z) instead of the caller's point)."""
    R = inputs.R_E
    cells = [(a, b + shift * R, c) for a, b, c in inputs.c2_mesh(R)]
    prob = inputs.Problem("shifted", 3, [(R, cells)], [inputs.Species("e", 1.0, -1.0, 0)], fmix=[[(1, 1, 0)]])
    h = _host(prob)
    assert h.mirror() == (False, False)
    lib = L.lib()
    assert lib.landau_set_mirror(h._h, 1) == L.LANDAU_EUNSUPPORTED


def test_dyadic_radius_keeps_refinement_exact():
    """inputs.dyadic_radius: a 36-significant-bit R changes the domain by <= 2^-36 relative and makes
    every refinement coordinate an exact double (mirror cells satisfy z0' == -(z0 + h) exactly)."""
    R = inputs.dyadic_radius(5.0 * inputs.VTH_E)
    assert abs(R / (5.0 * inputs.VTH_E) - 1.0) <= 2.0 ** -36
    cells = inputs.refine_uniform(inputs.c2_mesh(R), 3)
    key = set(cells)
    assert all((a, -(b + c), c) in key for a, b, c in cells)


def test_host_allocation_failure_is_enomem(monkeypatch):
    """The header promises that nothing throws or aborts: a std::bad_alloc inside the host plan
    (forced by the LANDAU_TEST_FAIL_ALLOC fault-injection hook) comes back as LANDAU_ENOMEM with a
    message, the process survives, and the next create succeeds."""
    monkeypatch.setenv("LANDAU_TEST_FAIL_ALLOC", "plan")
    with pytest.raises(L.LandauError) as ei:
        _host(inputs.config1())
    assert ei.value.code == L.LANDAU_ENOMEM
    assert "bad_alloc" in L.lib().landau_last_error(None).decode()
    monkeypatch.delenv("LANDAU_TEST_FAIL_ALLOC")
    assert _host(inputs.config1()).npoints == 72


def test_binding_checks_sizes_before_calling():
    """The binding passes raw pointers, so it checks every tensor first: wrong element count, wrong
    dtype or a CPU tensor where a device one is expected raise before the library is called."""
    import torch
    h = _host(inputs.config1())
    with pytest.raises(ValueError):
        h.set_state(torch.zeros(h.ndof))                   # CPU tensor for a device argument
    with pytest.raises(ValueError):
        h._dev(torch.zeros(3), h.ndof, "x")
    with pytest.raises(TypeError):
        h.jacobian_host(torch.zeros(h.ndof, dtype=torch.float32), torch.zeros(h.nnz, dtype=torch.float64))
    with pytest.raises(ValueError):
        h.jacobian_host(torch.zeros((1, h.ndof), dtype=torch.float64), torch.zeros((1, h.nnz - 1), dtype=torch.float64))
    with pytest.raises(ValueError):
        h._nvals(7)
