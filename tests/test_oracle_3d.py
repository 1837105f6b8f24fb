"""Pins of oracle O12: the inner integral with the 3D Cartesian Landau tensor
of Eq. 3 (PAPER.md:1@7593), U(u) = (|u|^2 I - u u^T)/|u|^3, evaluated straight from the definition.

P13a  what Eq. 3 fixes for any u: U u = 0, tr U = 2/|u|, U symmetric with eigenvalues 0 (along u)
      and 1/|u| (twice), U(lambda u) = U(u)/|lambda|;
P13b  the azimuthal integral of the 3D tensor over a source ring is the axisymmetric tensor of O5
      (elliptic integrals, itself pinned to mpmath quadrature in test_oracle_tensor): two
      independent formulas for the same integral (Eq. 3 and the reduction of @7997-8072);
P13c  the 3D inner integral of ring-discretised sources equals the axisymmetric inner integral O5
      at targets off the rings (the whole sum, G_D and the G_K contraction, component by component);
P13d  rotation covariance: rotating every point and T_K by Q maps G_D -> Q G_D Q^T, G_K -> Q G_K
      (catches a transposed or mislabelled component).
"""
import numpy as np
import pytest

from oracle import oracle as O

IDX = [(0, 0), (0, 1), (0, 2), (1, 1), (1, 2), (2, 2)]


def U3(u):
    t = O.tensor3d(u)
    M = np.zeros((3, 3))
    for k, (a, b) in enumerate(IDX):
        M[a, b] = M[b, a] = t[k]
    return M


def test_P13a_tensor_invariants():
    rng = np.random.default_rng(1)
    for _ in range(50):
        u = rng.normal(size=3) * 10.0 ** rng.uniform(-3, 2)
        M = U3(u)
        s = np.linalg.norm(u)
        assert np.allclose(M, M.T)
        assert np.linalg.norm(M @ u) <= 1e-14 * np.linalg.norm(M) * s
        assert abs(np.trace(M) - 2.0 / s) <= 1e-14 * 2.0 / s
        ev = np.sort(np.linalg.eigvalsh(M))
        assert abs(ev[0]) <= 1e-14 / s and np.allclose(ev[1:], 1.0 / s, rtol=1e-13)
        lam = rng.uniform(0.1, 10.0) * rng.choice([-1.0, 1.0])
        assert np.allclose(U3(lam * u), M / abs(lam), rtol=1e-13, atol=0.0)


@pytest.mark.parametrize("r,z,rb,zb", [(1.0, 0.3, 0.7, -0.4), (0.2, 1.5, 1.1, 0.9), (2.0, -1.0, 0.05, 0.6),
                                       (0.8, 0.0, 0.3, 0.0)])
def test_P13b_ring_integral_is_the_axisymmetric_tensor(r, z, rb, zb):
    """Target at (r, 0, z), sources at (rb cos phi, rb sin phi, zb): the trapezoid rule in phi (exact
    up to rounding for these smooth periodic integrands at M = 4096) reproduces O5's
    U^D_rr = int U_xx, U^D_rz = int U_xz, U^D_zz = int U_zz, U^K_rr = int (U_xx cos + U_xy sin),
    U^K_zr = int (U_zx cos + U_zy sin)."""
    M = 4096
    phi = 2.0 * np.pi * np.arange(M) / M
    acc = np.zeros(5)
    for p in phi:
        T = U3([r - rb * np.cos(p), -rb * np.sin(p), z - zb])
        acc += [T[0, 0], T[0, 2], T[2, 2], T[0, 0] * np.cos(p) + T[0, 1] * np.sin(p),
                T[2, 0] * np.cos(p) + T[2, 1] * np.sin(p)]
    acc *= 2.0 * np.pi / M
    ref = O.tensor(r, z, rb, zb)
    assert np.allclose(acc, ref, rtol=1e-11, atol=1e-12 * np.abs(ref).max())


def test_P13c_inner3d_of_rings_is_the_axisymmetric_inner_integral():
    """2D sources (r_j, z_j, w_j, T_D, T_Kr, T_Kz) become M-point rings with weights w_j 2 pi / M and
    T_K = T_Kr e_r(phi) + T_Kz e_z; targets (weight 0) sit at azimuth 0 off every ring.  Then the 3D
    G_D xx, xz, zz and G_K x, z at a target are O5's G_D rr, rz, zz and G_K r, z."""
    rng = np.random.default_rng(7)
    ns, nt, M = 6, 4, 2048
    rs, zs = rng.uniform(0.3, 2.0, ns), rng.uniform(-1.5, 1.5, ns)
    ws, TD, TKr, TKz = rng.uniform(0.5, 1.5, ns), rng.normal(size=ns), rng.normal(size=ns), rng.normal(size=ns)
    rt, zt = rng.uniform(0.3, 2.0, nt), rng.uniform(-1.5, 1.5, nt)
    # 2D reference: sources + weightless targets
    r2, z2 = np.concatenate([rs, rt]), np.concatenate([zs, zt])
    w2 = np.concatenate([ws, np.zeros(nt)])
    pad = np.zeros(nt)
    G2 = O.inner(r2, z2, w2, np.concatenate([TD, pad]), np.concatenate([TKr, pad]), np.concatenate([TKz, pad]),
                 targets=np.arange(ns, ns + nt))
    # 3D: rings + targets
    phi = 2.0 * np.pi * np.arange(M) / M
    c, s = np.cos(phi), np.sin(phi)
    x = np.concatenate([np.outer(rs, c).ravel(), rt])
    y = np.concatenate([np.outer(rs, s).ravel(), np.zeros(nt)])
    z = np.concatenate([np.repeat(zs, M), zt])
    wq = np.concatenate([np.repeat(ws * 2.0 * np.pi / M, M), np.zeros(nt)])
    wTD = wq * np.concatenate([np.repeat(TD, M), np.zeros(nt)])
    wTK = np.stack([wq * np.concatenate([np.outer(TKr, c).ravel(), pad]),
                    wq * np.concatenate([np.outer(TKr, s).ravel(), pad]),
                    wq * np.concatenate([np.repeat(TKz, M), pad])])
    G3, _ = O.inner3d(x, y, z, wTD, wTK)
    G3t = G3[:, ns * M:]
    got = np.stack([G3t[0], G3t[2], G3t[5], G3t[6], G3t[8]])
    assert np.allclose(got, G2, rtol=1e-10, atol=1e-11 * np.abs(G2).max())
    # and nothing out of the (r, z) plane at azimuth 0: G_D xy, yz and G_K y vanish by symmetry
    assert np.abs(G3t[[1, 4, 7]]).max() <= 1e-12 * np.abs(G2).max()


def test_P13d_rotation_covariance():
    rng = np.random.default_rng(3)
    n = 40
    X = rng.normal(size=(3, n))
    wTD = rng.uniform(0.1, 1.0, n)
    wTK = rng.normal(size=(3, n))
    G, _ = O.inner3d(X[0], X[1], X[2], wTD, wTK)
    Q, _ = np.linalg.qr(rng.normal(size=(3, 3)))
    Xq, wTKq = Q @ X, Q @ wTK
    Gq, _ = O.inner3d(Xq[0], Xq[1], Xq[2], wTD, wTKq)

    def mat(Gc, i):
        Mx = np.zeros((3, 3))
        for k, (a, b) in enumerate(IDX):
            Mx[a, b] = Mx[b, a] = Gc[k, i]
        return Mx

    for i in range(n):
        assert np.allclose(mat(Gq, i), Q @ mat(G, i) @ Q.T, rtol=1e-12, atol=1e-12 * np.abs(G[:6, i]).max())
        assert np.allclose(Gq[6:, i], Q @ G[6:, i], rtol=1e-12, atol=1e-12 * np.abs(G[6:, i]).max())
