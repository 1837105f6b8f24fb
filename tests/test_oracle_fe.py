"""Pins P6, P7, P8 (+ hanging-node constraints) of the oracle's FE machinery.

P6: DOF/point counts the paper prints (tests/golden/paper_counts.json).
P7: mass matrix: sum of entries = shift * int r dr dz = shift R^3, symmetric, positive definite.
P8: Gauss-Legendre nodes/weights against numpy's textbook rule; Q_p polynomials are reproduced
    exactly through the hanging-node constraints (value and gradient at every quadrature point).
"""
import json
import os

import numpy as np
import pytest

from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_counts.json")))


def _single(cells, R, p, nq=0):
    return inputs.Problem("t", p, [(R, cells)], [inputs.Species("x", 1.0, 1.0, 0)], fmix=[[(1.0, 1.0, 0.0)]])


def test_p6_mesh_A_counts():
    R = inputs.R_E
    pa = _single(inputs.origin_chain(R, 3), R, 3)
    o = Oracle(pa)
    assert len(pa.grids[0][1]) == GOLD["mesh_A_cells"]["value"]
    assert o.ndof == GOLD["mesh_A_q3_vertices"]["value"]
    assert o.npoints == GOLD["mesh_A_cells"]["value"] * GOLD["q3_points_per_cell"]["value"]
    # 128 integration points within a bit over one thermal radius (R/4 = 1.25 v_th), Fig. 3 text
    r, z, w = o.points()
    assert np.sum(np.maximum(r, np.abs(z)) < R / 4) == GOLD["mesh_A_inner_points"]["value"]
    # the Cartesian equivalent at the finest spacing R/8 has 8 x 16 = 128 cells
    assert len(inputs.uniform_mesh(R, 8)) == GOLD["cartesian_equivalent_cells"]["value"]


def test_p6_table_I_three_grids():
    o = Oracle(inputs.config3())
    assert o.npoints == GOLD["three_grids_N"]["value"]
    assert round(o.npoints ** 2 / 1e6, 1) == GOLD["three_grids_tensors_M"]["value"]
    assert [o.grid_ndof(g) for g in range(3)] == [GOLD["mesh_A_q3_vertices"]["value"]] * 3
    # ten grids of 20 Q3 cells: N = 3200, N^2 = 10.2M
    n10 = 10 * GOLD["mesh_A_cells"]["value"] * GOLD["q3_points_per_cell"]["value"]
    assert n10 == GOLD["ten_grids_N"]["value"] and round(n10 ** 2 / 1e6, 1) == GOLD["ten_grids_tensors_M"]["value"]


def test_config_sizes():
    """Sizes quoted in SURVEY.md §8(d) (regression of the generator recipe, survey S3)."""
    o1 = Oracle(inputs.config1())
    assert (o1.ndof, o1.npoints, o1.nnz) == (45, 72, 561)
    o2 = Oracle(inputs.config2())
    assert len(inputs.c2_mesh()) == 68 and o2.npoints == 1088 and o2.grid_ndof(0) == 601


@pytest.mark.parametrize("p", [2, 3, 4])
def test_p8_gauss_points_and_weights(p):
    R = 2.0
    o = Oracle(_single([(0.0, -R, R), (0.0, 0.0, R)], R, p))
    r, z, w = o.points()
    x, wx = np.polynomial.legendre.leggauss(p + 1)
    n = p + 1
    rr = R * (x + 1) / 2
    for c, z0 in enumerate([-R, 0.0]):
        sl = slice(c * n * n, (c + 1) * n * n)
        er = np.tile(rr, n)
        ez = np.repeat(z0 + R * (x + 1) / 2, n)
        ew = np.outer(wx, wx).ravel() * (R / 2) ** 2 * er
        np.testing.assert_allclose(r[sl], er, rtol=1e-15, atol=1e-15)
        np.testing.assert_allclose(z[sl], ez, rtol=1e-15, atol=1e-15)
        np.testing.assert_allclose(w[sl], ew, rtol=2e-15)


@pytest.mark.parametrize("p", [2, 3, 4])
@pytest.mark.parametrize("mesh", ["A", "chain", "C1"])
def test_p8_polynomial_reproduction_through_constraints(p, mesh):
    """f in Q_p is interpolated at the DOF nodes; the constrained (hanging) nodes must reproduce it, so
    f and grad f at every quadrature point are exact.  A wrong constraint weight or index breaks it."""
    R = 3.0
    cells = {"A": inputs.origin_chain(R, 3), "chain": inputs.origin_chain(R, 6),
             "C1": inputs.uniform_mesh(R, 2)}[mesh]
    o = Oracle(_single(cells, R, p))
    nr, nz = o.nodes(0)
    rng = np.random.default_rng(p)
    A = rng.normal(size=(p + 1, p + 1))

    def poly(r, z, dr=0, dz=0):
        out = np.zeros_like(r)
        for a in range(p + 1):
            for b in range(p + 1):
                ca = np.prod(range(a - dr + 1, a + 1)) if a >= dr else 0.0
                cb = np.prod(range(b - dz + 1, b + 1)) if b >= dz else 0.0
                if ca and cb:
                    out = out + A[a, b] * ca * cb * (r / R) ** (a - dr) * (z / R) ** (b - dz) / R ** (dr + dz)
        return out

    f = poly(nr, nz)
    TD, TKr, TKz = o.point_fields(f)
    r, z, w = o.points()
    scale = np.abs(A).sum()
    np.testing.assert_allclose(TD, poly(r, z), atol=1e-13 * scale)
    np.testing.assert_allclose(TKr, poly(r, z, 1, 0), atol=1e-12 * scale / R)
    np.testing.assert_allclose(TKz, poly(r, z, 0, 1), atol=1e-12 * scale / R)


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_p7_mass(cfg):
    prob = inputs.CONFIGS[cfg]()
    o = Oracle(prob)
    shift = 2.5
    M = o.mass(shift)
    rp, col = o.pattern()
    Mc = o.mass_coo(shift)
    row_of = np.repeat(np.arange(o.ndof), np.diff(rp))
    start = 0
    for a, sp in enumerate(prob.species):
        R = prob.grids[sp.grid][0]
        nd = o.grid_ndof(sp.grid)
        rows = (row_of >= start) & (row_of < start + nd)
        # partition of unity: sum_kl M_kl = shift * int_0^R int_-R^R r dz dr = shift R^3
        np.testing.assert_allclose(M[rows].sum(), shift * R ** 3, rtol=1e-13)
        start += nd
    np.testing.assert_allclose(Mc.sum(), M.sum(), rtol=1e-13)
    # symmetric and positive definite (dense check on the small configs)
    if o.ndof <= 1300:
        D = np.zeros((o.ndof, o.ndof))
        D[row_of, col] = M
        np.testing.assert_allclose(D, D.T, atol=1e-15 * np.abs(D).max())
        assert np.linalg.eigvalsh(D).min() > 0


def test_p7_mass_second_moment():
    """psi^T M 1 with psi = r^2 + z^2 (exact in Q_p, p >= 2): int r (r^2+z^2) = 5 R^5 / 6."""
    for p in (2, 3, 4):
        R = 1.7
        o = Oracle(_single(inputs.origin_chain(R, 4), R, p))
        M = o.mass(1.0)
        rp, col = o.pattern()
        row_of = np.repeat(np.arange(o.ndof), np.diff(rp))
        nr, nz = o.nodes(0)
        psi = nr ** 2 + nz ** 2
        val = np.sum(M * psi[row_of])
        np.testing.assert_allclose(val, 5 * R ** 5 / 6, rtol=1e-13)


def test_csr_pattern_structure():
    o = Oracle(inputs.config3())
    rp, col = o.pattern()
    for i in range(o.ndof):
        seg = col[rp[i]:rp[i + 1]]
        assert np.all(np.diff(seg) > 0)
    # block diagonal: species blocks never couple
    row_of = np.repeat(np.arange(o.ndof), np.diff(rp))
    blk = np.searchsorted(np.cumsum([193, 193, 193]), row_of, side="right")
    blkc = np.searchsorted(np.cumsum([193, 193, 193]), col, side="right")
    assert np.all(blk == blkc)
    # structurally symmetric
    S = set(zip(row_of.tolist(), col.tolist()))
    assert all((c, r) in S for (r, c) in S)


def test_invalid_meshes_rejected():
    R = 1.0
    bad_balance = inputs.refine_origin(inputs.refine_origin([(0.0, -R, R), (0.0, 0.0, R)], 1), 1)
    # refine only one cell twice more -> 4:1 neighbour
    bad = [c for c in bad_balance]
    c0 = [c for c in bad if c[0] == 0.0 and c[1] == 0.0][0]
    bad.remove(c0)
    sub = inputs.refine_uniform([c0], 2)
    with pytest.raises(ValueError):
        Oracle(_single(bad + sub, R, 3))
    with pytest.raises(ValueError):
        Oracle(_single([(0.0, -R, R), (0.0, 0.0, R), (0.0, 0.0, R / 2)], R, 3))   # overlap
