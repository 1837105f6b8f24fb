"""Pins P1, P2: the oracle's U^D, U^K against Eq. 3 itself.

P1: brute-force azimuthal quadrature of Eq. 3 (PAPER.md:1@7593) at 30 digits, on a stress set that
    covers the series branch (s < 1/4), the closed-form branch, near-coincident pairs, near-axis
    points and the branch switch.
P2: exact identities that follow from U(u) u = 0 and U(v, vbar) = U(vbar, v) -- true for any values
    of K and E, so they pin signs, indices and the component assembly rather than elliptic accuracy.
"""
import numpy as np
import pytest

from oracle.oracle import tensor
from tests._brute import tensor_mpmath, tensors_quadrature

STRESS = [
    (1.0, 0.3, 0.7, -0.2),          # generic, closed form
    (1e-4, 0.5, 2.0, 0.1),          # s ~ 1e-4, series
    (1.5e-4, 0.1, 3e-4, -0.2),      # both near the axis
    (0.5, 0.0, 0.5, 1e-5),          # near-coincident, s -> 1
    (0.3, 0.1, 0.30001, 0.1),       # near-coincident in r
    (2.0, 1.0, 2.0 + 1.4e-5, 1.0),  # separation 1.4e-5 far from the axis
    (2.0, 1.0, 1e-3, -1.0),         # s ~ 8e-4
    (1.0, 0.0, 0.1267, 0.0),        # just below the switch s = 1/4
    (1.0, 0.0, 0.1268, 0.0),        # just above
    (0.2, 0.2, 0.25, 0.21),
    (3.7, -2.2, 0.05, 4.1),         # s ~ 5.6e-3
    (4.0, 0.0, 1e-5, 0.0),          # s ~ 5e-6
]


@pytest.mark.parametrize("pair", STRESS)
def test_p1_tensor_vs_mpmath_quadrature(pair):
    a = tensor(*pair)
    b = tensor_mpmath(*pair)
    scale = np.abs(b).max()
    err = np.abs(a - b)
    assert np.all(err <= 1e-14 * scale + 1e-14 * np.abs(b)), (pair, a, b, err / scale)
    # component-wise relative accuracy wherever the component is not itself a cancellation remnant
    big = np.abs(b) > 1e-6 * scale
    assert np.all(err[big] <= 2e-13 * np.abs(b[big])), (pair, err / np.abs(b))


def test_p1_random_pairs_vs_graded_quadrature():
    rng = np.random.default_rng(7)
    n = 400
    r = 10.0 ** rng.uniform(-4, 0.6, n)
    rb = 10.0 ** rng.uniform(-4, 0.6, n)
    z = rng.uniform(-4, 4, n)
    zb = z + rng.choice([-1, 1], n) * 10.0 ** rng.uniform(-5, 0.5, n)
    ours = np.stack([tensor(*p) for p in zip(r, z, rb, zb)], axis=1)
    ref = tensors_quadrature(r, z, rb, zb)
    scale = np.abs(ref).max(axis=0)
    rel = np.abs(ours - ref) / scale
    assert rel.max() < 1e-12, rel.max()


def _pairs(n, seed):
    rng = np.random.default_rng(seed)
    r = 10.0 ** rng.uniform(-4, 0.7, n)
    rb = 10.0 ** rng.uniform(-4, 0.7, n)
    z = rng.uniform(-5, 5, n)
    zb = rng.uniform(-5, 5, n)
    return r, z, rb, zb


def test_p2_null_space_identity():
    """U^D_ij (r_i, z_i) = U^K_ij (r_j, z_j): int e_a.U.(v - vbar) dphi = 0 (energy conservation)."""
    for r, z, rb, zb in zip(*_pairs(2000, 1)):
        Drr, Drz, Dzz, Krr, Kzr = tensor(r, z, rb, zb)
        lhs = np.array([Drr * r + Drz * z, Drz * r + Dzz * z])
        rhs = np.array([Krr * rb + Drz * zb, Kzr * rb + Dzz * zb])
        scale = np.array([abs(Drr * r) + abs(Drz * z) + abs(Krr * rb) + abs(Drz * zb),
                          abs(Drz * r) + abs(Dzz * z) + abs(Kzr * rb) + abs(Dzz * zb)])
        assert np.all(np.abs(lhs - rhs) <= 1e-13 * scale), (r, z, rb, zb, lhs, rhs)


def test_p2_transpose_identity():
    """U^K_ji = (U^K_ij)^T and U^D_zz symmetric (rotational symmetry + U(v, vbar) = U(vbar, v))."""
    for r, z, rb, zb in zip(*_pairs(2000, 2)):
        ij = tensor(r, z, rb, zb)
        ji = tensor(rb, zb, r, z)
        pairs = [(ji[3], ij[3]), (ji[4], ij[1]), (ji[1], ij[4]), (ji[2], ij[2])]
        for a, b in pairs:
            assert abs(a - b) <= 1e-13 * (abs(a) + abs(b)) + 1e-300, (r, z, rb, zb, a, b)


def test_branch_continuity_at_switch():
    """The series (s < 1/4) and the closed form (s >= 1/4) agree across the switch."""
    r = 1.0
    s_lo = 0.25 * (1 - 1e-12)
    # s = 2 r rb / (r^2 + rb^2) -> rb = (1 - sqrt(1 - s^2)) / s
    for s in (s_lo, 0.25 * (1 + 1e-12)):
        rb = (1 - np.sqrt(1 - s * s)) / s
        a = tensor(r, 0.3, rb, 0.3)
        b = tensor_mpmath(r, 0.3, rb, 0.3)
        assert np.abs(a - b).max() <= 1e-14 * np.abs(b).max()
