"""Independent brute-force evaluation of the axisymmetric Landau tensors straight from Eq. 3.

U(u) = (|u|^2 I - u u^T) / |u|^3 (PAPER.md:1@7593, Eq. 3) with u = v - vbar(phi), target at azimuth 0,
source at azimuth phi; U^D_ab = int e_a.U.e_b dphi, U^K_ab = int e_a.U.ebar_b(phi) dphi (SURVEY §8(c)
O5).  Integrated numerically over phi (the integrand is even in phi, so 2 * int_0^pi), with no
elliptic integrals and no closed form -- so it pins the oracle's closed forms and series.
"""
import numpy as np
import mpmath as mp

_X16, _W16 = np.polynomial.legendre.leggauss(24)


def _panels():
    # geometric grading toward phi = 0 (where |u| is smallest), then uniform panels to pi
    edges = [0.0] + [np.pi * 2.0 ** (-k) for k in range(44, 3, -1)]
    edges += list(np.linspace(np.pi / 16, np.pi, 16)[1:])
    return np.array(edges)


_E = _panels()
_a, _b = _E[:-1], _E[1:]
_PHI = (0.5 * (_b - _a)[:, None] * _X16[None, :] + 0.5 * (_a + _b)[:, None]).ravel()
_WPHI = (0.5 * (_b - _a)[:, None] * _W16[None, :]).ravel()


def integrand(r, z, rb, zb, phi):
    """5 components (U^D_rr, U^D_rz, U^D_zz, U^K_rr, U^K_zr) of the phi-integrand, from Eq. 3."""
    c, s = np.cos(phi), np.sin(phi)
    ux, uy, uz = r - rb * c, -rb * s, (z - zb) + 0 * c
    u2 = ux * ux + uy * uy + uz * uz
    n3 = u2 * np.sqrt(u2)
    # e_r = (1,0,0), e_z = (0,0,1), ebar_r = (c, s, 0)
    Urr = (u2 - ux * ux) / n3
    Urz = (-ux * uz) / n3
    Uzz = (u2 - uz * uz) / n3
    UKrr = (u2 * c - ux * (ux * c + uy * s)) / n3
    UKzr = (-uz * (ux * c + uy * s)) / n3
    return np.stack([Urr, Urz, Uzz, UKrr, UKzr])


def tensors_quadrature(r, z, rb, zb):
    """Vectorised over pairs: arrays r, z, rb, zb of shape [n] -> [5, n]."""
    r, z, rb, zb = (np.asarray(a, dtype=np.float64)[:, None] for a in (r, z, rb, zb))
    vals = integrand(r, z, rb, zb, _PHI[None, :])       # [5, n, nphi]
    return 2.0 * np.einsum("cnp,p->cn", vals, _WPHI)


def tensor_mpmath(r, z, rb, zb, dps=30):
    """One pair at `dps` digits with mpmath tanh-sinh quadrature (splits near the phi = 0 peak)."""
    mp.mp.dps = dps
    r, z, rb, zb = map(mp.mpf, (r, z, rb, zb))

    def comp(k):
        def f(phi):
            c, s = mp.cos(phi), mp.sin(phi)
            ux, uy, uz = r - rb * c, -rb * s, z - zb
            u2 = ux * ux + uy * uy + uz * uz
            n3 = u2 * mp.sqrt(u2)
            return [(u2 - ux * ux) / n3, (-ux * uz) / n3, (u2 - uz * uz) / n3,
                    (u2 * c - ux * (ux * c + uy * s)) / n3, (-uz * (ux * c + uy * s)) / n3][k]
        pts = [0, mp.mpf("1e-8"), mp.mpf("1e-6"), mp.mpf("1e-4"), mp.mpf("1e-2"), mp.mpf("0.3"), mp.pi]
        return 2 * mp.quad(f, pts)

    return np.array([float(comp(k)) for k in range(5)])
