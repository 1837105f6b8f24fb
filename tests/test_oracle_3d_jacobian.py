"""Pins of the oracle's 3D Cartesian Jacobian O13 (NEXT-4 completed: "a full 3D model is supported in
the library", PAPER.md:1@7997-8072; oracle.h O13).  Its inner integral (O12) is pinned by P13
(tests/test_oracle_3d.py); these tests fix the rest from outside the oracle:

* P15 the point fields (O3/O4) of a polynomial f in Q_p equal T_D = sum e^2 f, T_K = sum e^2 (m0/m) grad f
  evaluated analytically at the Gauss points (the nodal interpolant of a Q_p function is exact);
* P16 the element matrices and assembly (O7/O8) with a manufactured G: G_D = I, G_K = 0 gives
  fD x the Q_p stiffness matrix, whose action on x^2 at interior nodes is -2 fD int phi_k = -2 fD times a
  product of closed-form Newton-Cotes weights (Simpson 1/3, 4/3, 1/3 for Q2; 3/8-rule 1/4, 3/4, 3/4, 1/4
  for Q3, times h/2); G_D = 0, G_K = e_x gives fK int d_x phi_k phi_l, whose action on 1 is 0 and on x is
  -fK int phi_k at interior nodes;
* P17 the whole Jacobian conserves density per species and momentum and energy summed over species
  (Sigma_a m_a psi^T J_a f_a = 0 for psi = v_x, v_y, v_z, |v|^2, all in Q_p): the discrete Landau form's
  exact conservation (PAPER.md:1@2223), which fails for a wrong species factor, tensor or pairing;
* the pattern is the tensor product of the 1-D patterns, |J| <= J^abs entrywise.
"""
import numpy as np
import pytest

from oracle.oracle import Oracle3D
from paper_conf_ipps_adamsbkw22_b200 import inputs

NC = {2: [1.0 / 3.0, 4.0 / 3.0, 1.0 / 3.0], 3: [0.25, 0.75, 0.75, 0.25]}   # int_{-1}^{1} l_a, equispaced


def _oracle(ncell, order, species=((1.0, -1.0), (4.0, 1.0)), R=None):
    return Oracle3D(ncell, order, inputs.R_E if R is None else R, list(species))


def _weights_1d(ncell, order, h):
    """int phi_i over the lattice line: sum over the cells holding node i of (h/2) NC[a]"""
    M = ncell * order + 1
    W = np.zeros(M)
    for c in range(ncell):
        for a in range(order + 1):
            W[c * order + a] += 0.5 * h * NC[order][a]
    return W


@pytest.mark.parametrize("ncell,order", [(2, 2), (2, 3), (3, 2)])
def test_P15_fields_of_a_Qp_polynomial_are_exact(ncell, order):
    sp = ((1.0, -1.0), (4.0, 1.0))
    o = _oracle(ncell, order, sp)
    x, y, z = o.nodes()
    c = [0.7, -0.3, 0.2, 0.05, -0.11]
    poly = lambda x, y, z: c[0] + c[1] * x + c[2] * y * z + c[3] * x ** order * y ** (order - 1) + c[4] * z ** order
    grad = lambda x, y, z: (c[1] + order * c[3] * x ** (order - 1) * y ** (order - 1),
                            c[2] * z + (order - 1) * c[3] * x ** order * y ** (order - 2),
                            c[2] * y + order * c[4] * z ** (order - 1))
    f = np.stack([poly(x, y, z), 2.0 * poly(x, y, z) - 1.0])   # species 1: 2 f - 1 (still in Q_p)
    T = o.fields(f)
    (px, py, pz), w = o.points()
    fv, g = poly(px, py, pz), np.array(grad(px, py, pz))
    TD = 1.0 * fv + 1.0 * (2.0 * fv - 1.0)
    TK = 1.0 / 1.0 * g + 1.0 / 4.0 * (2.0 * g)
    scale = np.abs(TD).max()
    assert np.max(np.abs(T[0] - TD)) <= 1e-13 * scale
    assert np.max(np.abs(T[1:] - TK)) <= 1e-13 * np.abs(TK).max()
    assert abs(w.sum() - (2.0 * inputs.R_E) ** 3) <= 1e-13 * (2.0 * inputs.R_E) ** 3


@pytest.mark.parametrize("ncell,order", [(2, 2), (3, 2), (2, 3), (3, 3)])
def test_P16_stiffness_and_advection_closed_forms(ncell, order):
    e, m, nu = -1.0, 1.0, 1.0
    o = _oracle(ncell, order, ((m, e),))
    R = inputs.R_E
    h = 2.0 * R / ncell
    fD, fK = -nu * e * e / (m * m), nu * e * e / m
    x, y, z = o.nodes()
    rp, col = o.pattern()
    row = np.repeat(np.arange(o.ndof), np.diff(rp))
    M = ncell * order + 1
    ix = np.arange(o.ndof) % M
    iy = (np.arange(o.ndof) // M) % M
    iz = np.arange(o.ndof) // (M * M)
    W = _weights_1d(ncell, order, h)
    intphi = W[ix] * W[iy] * W[iz]
    interior_x = (ix > 0) & (ix < M - 1)
    G = np.zeros((9, o.npoints))
    G[0] = G[3] = G[5] = 1.0                                  # G_D = I, G_K = 0
    J = o.assemble(G)[0]
    act = np.bincount(row, J * (x ** 2)[col], minlength=o.ndof)
    assert np.max(np.abs(act[interior_x] - (-2.0 * fD * intphi[interior_x]))) <= 1e-12 * np.abs(fD * intphi).max()
    # the stiffness matrix is symmetric and annihilates constants
    Jd = np.zeros((o.ndof, o.ndof))
    Jd[row, col] = J
    assert np.max(np.abs(Jd - Jd.T)) <= 1e-13 * np.abs(Jd).max()
    assert np.max(np.abs(Jd.sum(axis=1))) <= 1e-13 * np.abs(Jd).max()
    G = np.zeros((9, o.npoints))
    G[6] = 1.0                                                # G_D = 0, G_K = e_x
    A = o.assemble(G)[0]
    one = np.bincount(row, A, minlength=o.ndof)
    lin = np.bincount(row, A * x[col], minlength=o.ndof)
    assert np.max(np.abs(one[interior_x])) <= 1e-13 * np.abs(A).max()
    assert np.max(np.abs(lin[interior_x] - (-fK * intphi[interior_x]))) <= 1e-12 * np.abs(fK * intphi).max()


def _moments(o, prob, J, Ja, f):
    rp, col = o.pattern()
    row = np.repeat(np.arange(o.ndof), np.diff(rp))
    xyz = o.nodes()
    v2 = (xyz ** 2).sum(axis=0)
    dens, tot = [], np.zeros(8)
    for a, (m, _) in enumerate(prob.species):
        cs, csa = np.bincount(col, J[a], minlength=o.ndof), np.bincount(col, Ja[a], minlength=o.ndof)
        dens.append(np.max(np.abs(cs) / csa))
        Jf = np.bincount(row, J[a] * f[a][col], minlength=o.ndof)
        Jaf = np.bincount(row, Ja[a] * np.abs(f[a][col]), minlength=o.ndof)
        for c in range(3):
            tot[2 * c] += m * xyz[c] @ Jf
            tot[2 * c + 1] += m * np.abs(xyz[c]) @ Jaf
        tot[6] += m * v2 @ Jf
        tot[7] += m * v2 @ Jaf
    return max(dens), max(abs(tot[2 * c]) / tot[2 * c + 1] for c in range(3)), abs(tot[6]) / tot[7]


@pytest.mark.parametrize("ncell,order", [(2, 2), (2, 3)])
def test_P17_conservation_and_scale(ncell, order):
    prob = inputs.config3d(ncell, order)
    o = Oracle3D(prob.ncell, prob.order, prob.R, prob.species, prob.nu)
    f = inputs.coefficients3d(prob, o.nodes())
    J, Ja = o.jacobian(f)
    d, mom, en = _moments(o, prob, J, Ja, f)
    assert d < 1e-15 and mom < 1e-15 and en < 1e-15, (d, mom, en)   # measured ~1e-17 .. 1e-19
    assert np.all(np.abs(J) <= Ja * (1 + 1e-15))
    # the |.| scale depends on |f| only
    s = np.where(np.random.default_rng(3).random(f.shape) < 0.5, -1.0, 1.0)
    _, Ja2 = o.jacobian(f * s)
    assert np.max(np.abs(Ja2 - Ja) / Ja) < 1e-14


def test_pattern_is_the_tensor_product_of_1d_patterns():
    for ncell, order in ((1, 2), (2, 2), (3, 3)):
        o = _oracle(ncell, order)
        M = ncell * order + 1
        cnt1 = []
        for i in range(M):
            cells = [c for c in range(ncell) if c * order <= i <= (c + 1) * order]
            cnt1.append((max(cells) + 1) * order - min(cells) * order + 1)
        assert o.nnz == sum(cnt1) ** 3
        rp, col = o.pattern()
        assert np.all(np.diff(rp) > 0)
        for r in range(0, o.ndof, max(1, o.ndof // 7)):
            assert np.all(np.diff(col[rp[r]:rp[r + 1]]) > 0)
        A = np.zeros((o.ndof, o.ndof), dtype=bool)
        A[np.repeat(np.arange(o.ndof), np.diff(rp)), col] = True
        assert np.array_equal(A, A.T)
