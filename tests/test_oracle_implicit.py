"""Oracle pins for NEXT-3: the E_z advection matrix of Eq. 4 (O11) and the backward-Euler
step by the paper's quasi-Newton iteration (PAPER.md:1@10500-10978), checked against what the FE space
and the conservation properties of the collision operator fix -- not against the oracle itself.

P11 advection: Q_p (p >= 2) reproduces z and z^2, so  A_E z = M 1  and  A_E z^2 = 2 M z  hold to
    roundoff (a transposed operand, a wrong sign or a wrong 2/h scale fails them).
P12 implicit step: 1^T J_a = 0 (density conservation of C, pinned by P4), so every quasi-Newton
    iterate satisfies  1^T [M (f^{k+1} - f^n)/dt + eta_a A_E f^{k+1}] = 0  per species exactly; at
    convergence momentum and energy satisfy the same balance summed over species with m_a psi^T
    (psi = z, r^2 + z^2), and without a field the step conserves all three.  The iteration converges
    linearly (@10978).
"""
import numpy as np
import pytest
import scipy.sparse as sps

from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs


def _mats(o):
    rp, col = o.pattern()
    n = o.ndof
    M = sps.csr_matrix((o.mass(1.0), col, rp), shape=(n, n))
    A = sps.csr_matrix((o.advection(), col, rp), shape=(n, n))
    return M, A


def _nodes(o, prob):
    r = np.concatenate([o.nodes(int(g))[0] for g in prob.grid_of])
    z = np.concatenate([o.nodes(int(g))[1] for g in prob.grid_of])
    return r, z


@pytest.mark.parametrize("cfg", ["config1", "config2", "config3"])
def test_P11_advection_reproduces_dz_of_polynomials(cfg):
    prob = getattr(inputs, cfg)()
    o = Oracle(prob)
    M, A = _mats(o)
    r, z = _nodes(o, prob)
    one = np.ones(o.ndof)
    scale = np.abs(M).sum(axis=1).max() * (1 + np.abs(z).max())
    assert np.abs(A @ z - M @ one).max() <= 1e-13 * scale
    assert np.abs(A @ (z * z) - 2 * M @ z).max() <= 1e-13 * scale * np.abs(z).max()
    # d_z of a function of r alone vanishes; the transpose does not reproduce d_z
    assert np.abs(A @ (r * r)).max() <= 1e-13 * scale * np.abs(r).max() ** 2
    assert np.abs(A.T @ z - M @ one).max() > 1e-3 * np.abs(M @ one).max()


def test_P11_advection_coo_assembles_to_csr():
    prob = inputs.config3()
    o = Oracle(prob)
    row, col = o.coo_pattern()
    rp, ccol = o.pattern()
    Acoo = sps.coo_matrix((o.advection_coo(), (row, col)), shape=(o.ndof, o.ndof)).tocsr()
    Acoo.sort_indices()
    Acsr = o.advection()
    assert np.abs(Acoo.data - Acsr).max() <= 1e-14 * np.abs(Acsr).max()


def _balances(o, prob, f_old, f, dt, Ez):
    """per-species density residual and species-summed momentum / energy residuals of
    M (f - f_old)/dt + eta A_E f, each relative to the magnitude of its terms"""
    M, A = _mats(o)
    rows = o.species_rows()
    m = np.asarray(prob.mass, float)[rows]
    eta = Ez * (np.asarray(prob.charge, float) / np.asarray(prob.mass, float))[rows]
    R = M @ (f - f_old) / dt + eta * (A @ f)
    Rabs = np.abs(M) @ (np.abs(f) + np.abs(f_old)) / dt + np.abs(eta) * (np.abs(A) @ np.abs(f))
    r, z = _nodes(o, prob)
    dens = max(abs(R[rows == a].sum()) / Rabs[rows == a].sum() for a in range(len(prob.mass)))
    mom = abs((m * z * R).sum()) / (m * np.abs(z) * Rabs).sum()
    en = abs((m * (r * r + z * z) * R).sum()) / (m * (r * r + z * z) * Rabs).sum()
    return dens, mom, en


@pytest.mark.parametrize("cfg,Ez", [("config1", 0.0), ("config1", 0.1), ("config3", 0.0), ("config3", 0.1)])
def test_P12_implicit_step_balances(cfg, Ez):
    prob = getattr(inputs, cfg)()
    o = Oracle(prob)
    f0 = o.coefficients()
    dt = 0.05 if cfg == "config1" else 0.01
    its = o.implicit_step(f0, dt, Ez, iters=10)
    # density balance at every iterate (1^T J = 0 exactly)
    for f in its:
        assert _balances(o, prob, f0, f, dt, Ez)[0] <= 1e-13
    # linear convergence, then momentum and energy balance at the converged iterate
    d = [np.linalg.norm(its[k] - its[k - 1]) / np.linalg.norm(its[k]) for k in range(1, len(its))]
    assert d[4] < 1e-3 * d[0]
    dens, mom, en = _balances(o, prob, f0, its[-1], dt, Ez)
    assert mom <= 1e-12 and en <= 1e-12, (mom, en)
    # the step changes f (it is not the identity), and without a field it conserves the moments
    assert np.linalg.norm(its[-1] - f0) > 1e-4 * np.linalg.norm(f0)
    if Ez == 0.0:
        M, _ = _mats(o)
        rows = o.species_rows()
        r, z = _nodes(o, prob)
        m = np.asarray(prob.mass, float)[rows]
        Mf0, Mf = M @ f0, M @ its[-1]
        e0 = (m * (r * r + z * z) * Mf0).sum()
        assert abs((m * (r * r + z * z) * Mf).sum() - e0) <= 1e-12 * abs(e0)


def test_P12_negative_control_first_iterate_not_converged():
    """Momentum/energy balance holds only at convergence: the first iterate (J about f^n, not f^{n+1})
    violates it by far more than roundoff -- so the balance test above really checks convergence."""
    prob = inputs.config1()
    o = Oracle(prob)
    f0 = o.coefficients()
    its = o.implicit_step(f0, 0.05, 0.0, iters=1)
    dens, mom, en = _balances(o, prob, f0, its[0], 0.05, 0.0)
    assert dens <= 1e-13 and en > 1e-8


# ---------------------------------------------------------------------------------------------------
# P14: the thermal-quench source S_a(t) of Eq. 1 / Eq. 4 (PAPER.md:1@6337, @8216, @34560, @35736)
# ---------------------------------------------------------------------------------------------------
def _source(o, prob, f0, t0, t1, t_pulse, factor=5.0):
    """sigma for the step [t0, t1]: the cold-Maxwellian shape scaled so that the whole pulse injects
    factor x the initial discrete density of each species (reading R-7), divided by the step."""
    M, _ = _mats(o)
    rows = o.species_rows()
    shape = inputs.quench_source_shape(prob, o.all_nodes())
    Ms, Mf0 = M @ shape, M @ f0
    scale = np.array([Mf0[rows == a].sum() / Ms[rows == a].sum() for a in range(len(prob.species))])[rows]
    return factor * inputs.quench_pulse_fraction(t0, t1, t_pulse) / (t1 - t0) * scale * shape


@pytest.mark.parametrize("cfg,Ez", [("config1", 0.0), ("config3", 0.1)])
def test_P14_source_density_balance_every_iterate(cfg, Ez):
    """With the source, each quasi-Newton iterate satisfies the per-species density balance
    1^T [M (f^{k+1} - f^n)/dt + eta A_E f^{k+1}] = 1^T M sigma exactly (1^T J = 0); without the source
    term in the step the same balance misses by the injected amount (negative control)."""
    prob = getattr(inputs, cfg)()
    o = Oracle(prob)
    f0 = o.coefficients()
    dt = 0.02
    sig = _source(o, prob, f0, 0.0, dt, 4 * dt)
    M, A = _mats(o)
    rows = o.species_rows()
    eta = Ez * (np.asarray(prob.charge, float) / np.asarray(prob.mass, float))[rows]
    Msig = M @ sig
    for f in o.implicit_step(f0, dt, Ez, iters=3, src=sig):
        R = M @ (f - f0) / dt + eta * (A @ f)
        for a in range(len(prob.species)):
            sel = rows == a
            scale = (np.abs(M) @ (np.abs(f) + np.abs(f0)))[sel].sum() / dt
            assert abs(R[sel].sum() - Msig[sel].sum()) <= 1e-13 * scale
    f = o.implicit_step(f0, dt, Ez, iters=1)[0]
    R = M @ (f - f0) / dt + eta * (A @ f)
    assert abs(R[rows == 0].sum() - Msig[rows == 0].sum()) > 1e-3 * abs(Msig[rows == 0].sum())


def test_P14_pulse_injects_five_times_the_initial_density():
    """A whole pulse (4 backward-Euler steps, cumulative sinusoidal profile) injects exactly five times
    each species' initial density (@35736: "the total mass injected by the model is five times the
    initial density, which is observed to high accuracy"): with 1^T J = 0 and no field the discrete
    density after the pulse is 6 x the initial one to roundoff, whatever the iterates' convergence."""
    prob = inputs.config3()
    o = Oracle(prob)
    f = o.coefficients()
    f0 = f.copy()
    M, _ = _mats(o)
    rows = o.species_rows()
    dt, K = 0.01, 4
    for n in range(K):
        sig = _source(o, prob, f0, n * dt, (n + 1) * dt, K * dt)
        f = o.implicit_step(f, dt, 0.0, iters=2, src=sig)[-1]
    Mf0, Mf = M @ f0, M @ f
    for a in range(len(prob.species)):
        n0, n1 = Mf0[rows == a].sum(), Mf[rows == a].sum()
        assert abs(n1 - 6.0 * n0) <= 1e-12 * n1, (a, n1 / n0)
