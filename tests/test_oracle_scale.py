"""Pins of the oracle's condition scale O10: J^abs and G^abs are the same finite sums
as J and G with every product replaced by its absolute value (reading R-4: O3-O8).  They are
the denominators of every GPU parity assertion (|J_gpu - J_ora| <= 1e-11 J^abs), so an inflated scale
would silently loosen parity; these tests fix them from outside the oracle:

* an independent brute-force |.| assembly on C1 (uniform Q2 mesh, no hanging nodes): numpy Gauss
  points and Lagrange tables, DOFs matched by node coordinates, the Landau tensors by numerical
  azimuthal quadrature of Eq. 3 (tests/_brute.py, no elliptic integrals), sums by math.fsum;
* J^abs >= |J| and G^abs >= |G| entrywise on C1-C3 (triangle inequality; C2/C3 have hanging nodes);
* J^abs and G^abs depend on |f| only (flipping the signs of coefficients leaves them unchanged while
  J changes), and are linear in |f|.
"""
import math

import numpy as np
import pytest

from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs
from tests._brute import tensors_quadrature


def _lagrange_tables(p, x):
    """values and derivatives of the equispaced degree-p Lagrange basis on [-1, 1] at points x."""
    nodes = np.linspace(-1.0, 1.0, p + 1)
    V = np.zeros((len(x), p + 1))
    D = np.zeros((len(x), p + 1))
    for a in range(p + 1):
        others = np.delete(nodes, a)
        poly = np.poly1d(others, r=True) / np.prod(nodes[a] - others)
        V[:, a] = poly(x)
        D[:, a] = poly.deriv()(x)
    return V, D


def _brute_abs_scale_C1(f):
    """(G^abs [5][N], J^abs as a dict (row, col) -> value) of C1 computed from scratch."""
    prob = inputs.config1()
    o = Oracle(prob)
    (R, cells), = prob.grids
    sp = prob.species[0]
    p = prob.order
    S = p + 1
    xg, wg = np.polynomial.legendre.leggauss(S)
    V, D = _lagrange_tables(p, xg)
    nr, nz = o.nodes(0)
    dof_of = {(round(a / R * 1e9), round(b / R * 1e9)): k for k, (a, b) in enumerate(zip(nr, nz))}
    xi = np.linspace(-1.0, 1.0, S)
    e2, im = sp.charge ** 2, 1.0 / sp.mass
    fD, fK = -prob.nu * e2 * im * im, prob.nu * e2 * im
    pts, cell_dofs, tabs = [], [], []
    for (r0, z0, h) in cells:
        dofs = []
        for b in range(S):               # node n = b S + a (a along r, b along z)
            for a in range(S):
                key = (round((r0 + 0.5 * h * (1 + xi[a])) / R * 1e9), round((z0 + 0.5 * h * (1 + xi[b])) / R * 1e9))
                dofs.append(dof_of[key])
        cell_dofs.append(dofs)
        phi, gr, gz = [], [], []
        for qz in range(S):              # point q = qz S + qr
            for qr in range(S):
                r = r0 + 0.5 * h * (1 + xg[qr])
                z = z0 + 0.5 * h * (1 + xg[qz])
                w = wg[qr] * wg[qz] * 0.25 * h * h * r
                pts.append((r, z, w))
                phi.append([V[qr, a] * V[qz, b] for b in range(S) for a in range(S)])
                gr.append([2 / h * D[qr, a] * V[qz, b] for b in range(S) for a in range(S)])
                gz.append([2 / h * V[qr, a] * D[qz, b] for b in range(S) for a in range(S)])
        tabs.append((np.array(phi), np.array(gr), np.array(gz)))
    r, z, w = (np.array(c) for c in zip(*pts))
    # O3/O4 with |.|: T^abs = e^2 sum |phi| |f|, T_K^abs = e^2 (m0/m) sum |grad phi| |f|
    TD, TKr, TKz = [], [], []
    for dofs, (phi, gr, gz) in zip(cell_dofs, tabs):
        fa = np.abs(f[dofs])
        TD += list(e2 * (np.abs(phi) @ fa))
        TKr += list(e2 * im * (np.abs(gr) @ fa))
        TKz += list(e2 * im * (np.abs(gz) @ fa))
    TD, TKr, TKz = np.array(TD), np.array(TKr), np.array(TKz)
    N = r.size
    ii, jj = np.meshgrid(np.arange(N), np.arange(N), indexing="ij")
    ii, jj = ii.ravel(), jj.ravel()
    keep = ~((r[ii] == r[jj]) & (z[ii] == z[jj]))
    ii, jj = ii[keep], jj[keep]
    U = np.abs(tensors_quadrature(r[ii], z[ii], r[jj], z[jj]))
    wd, wkr, wkz = w[jj] * TD[jj], w[jj] * TKr[jj], w[jj] * TKz[jj]
    comps = [wd * U[0], wd * U[1], wd * U[2], U[3] * wkr + U[1] * wkz, U[4] * wkr + U[2] * wkz]
    Ga = np.stack([np.array([math.fsum(c[ii == i]) for i in range(N)]) for c in comps])
    # O6-O8 with |.|
    Ja = {}
    q0 = 0
    for dofs, (phi, gr, gz) in zip(cell_dofs, tabs):
        nq = phi.shape[0]
        for q in range(nq):
            Arr, Arz, Azz = (abs(fD) * Ga[c, q0 + q] for c in range(3))
            AKr, AKz = abs(fK) * Ga[3, q0 + q], abs(fK) * Ga[4, q0 + q]
            for k in range(len(dofs)):
                gkr, gkz = abs(gr[q, k]), abs(gz[q, k])
                for l in range(len(dofs)):
                    glr, glz, pl = abs(gr[q, l]), abs(gz[q, l]), abs(phi[q, l])
                    v = gkr * (Arr * glr + Arz * glz) + gkz * (Arz * glr + Azz * glz) + (gkr * AKr + gkz * AKz) * pl
                    Ja.setdefault((dofs[k], dofs[l]), []).append(abs(w[q0 + q]) * v)
        q0 += nq
    return Ga, {key: math.fsum(v) for key, v in Ja.items()}, (r, z, w)


def _signed_state(o, seed=7):
    f = o.coefficients()
    s = np.where(np.random.default_rng(seed).random(f.size) < 0.5, -1.0, 1.0)
    return f, f * s


def test_O10_matches_bruteforce_abs_assembly_C1():
    prob = inputs.config1()
    o = Oracle(prob)
    f, fs = _signed_state(o)
    Gb, Jb, (r, z, w) = _brute_abs_scale_C1(fs)
    ro, zo, wo = o.points()
    np.testing.assert_allclose(r, ro, rtol=1e-15)
    np.testing.assert_allclose(w, wo, rtol=1e-14)
    G, Ga = o.point_coeffs(fs)
    assert np.max(np.abs(Ga - Gb) / Gb) < 1e-14   # measured 6e-16
    J, Ja = o.jacobian(fs)
    rp, col = o.pattern()
    row = np.repeat(np.arange(o.ndof), np.diff(rp))
    ref = np.array([Jb[(int(a), int(b))] for a, b in zip(row, col)])
    assert len(Jb) == o.nnz
    assert np.max(np.abs(Ja - ref) / ref) < 1e-14   # measured 1.1e-15


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_O10_bounds_and_sign_invariance(cfg):
    o = Oracle(inputs.CONFIGS[cfg]())
    f, fs = _signed_state(o)
    J, Ja = o.jacobian(f)
    Js, Jas = o.jacobian(fs)
    G, Ga = o.point_coeffs(fs)
    eps = 1e-15
    assert np.all(np.abs(J) <= Ja * (1 + eps)) and np.all(np.abs(Js) <= Jas * (1 + eps))
    assert np.all(np.abs(G) <= Ga * (1 + eps))
    # |.| scale sees |f| only; J itself does change with the signs
    assert np.max(np.abs(Jas - Ja) / Ja) < 1e-14
    assert np.max(np.abs(Js - J)) > 1e-3 * np.max(np.abs(J))
    # and is positively homogeneous of degree one in f
    J2, Ja2 = o.jacobian(2.0 * fs)
    assert np.max(np.abs(Ja2 - 2.0 * Jas) / Jas) < 1e-14
