"""Seeded, synthetic input generators shared by the CUDA path's tests/bench and the oracle's tests.

This module holds NONE of the method's arithmetic (no basis functions, quadrature, DOF numbering,
constraints, Landau tensor or assembly).  It only produces what a user hands to ``landau_create`` /
``landau_set_state``:

* velocity-space meshes: leaf cells ``(r0, z0, h)`` of a 2:1-balanced quadtree over
  ``[0, R] x [-R, R]`` (two R x R roots), built by explicit refinement rules;
* species tables (mass in m_e, charge in e, grid index), App. A units (PAPER.md:1@58269);
* analytic distributions f_alpha(r, z) (sums of drifting Maxwellians, Amb-18) that are evaluated at
  node coordinates supplied by the caller (the library's or the oracle's own node list), multiplied
  by ``(1 + 0.01 xi)`` where ``xi ~ U(-1, 1)`` comes from a counter-based splitmix64 keyed by the
  node's exact lattice position, so both sides get identical coefficients at identical nodes.

Recipes are the ones in DESIGN.md §"Input recipe".
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

# App. A (PAPER.md:1@58430): v0 = (8 k T_e / (pi m_e))^(1/2).  A Maxwellian of temperature T and mass
# m (in m_e) has exp(-v^2/theta) with theta = (pi/4) (T/T_e) (m_e/m)  (Amb-18).
VTH_E = math.sqrt(math.pi) / 2.0          # electron thermal speed sqrt(theta_e) in units of v0
M_D = 3670.48                             # deuterium mass in m_e
M_W = 335120.0                            # tungsten (183.84 u) in m_e


def theta(T: float, m: float) -> float:
    return 0.25 * math.pi * T / m


def vth(T: float, m: float) -> float:
    return math.sqrt(theta(T, m))


# ----------------------------------------------------------------------------------------------
# meshes
# ----------------------------------------------------------------------------------------------

def dyadic_radius(R: float, bits: int = 36) -> float:
    """R rounded to `bits` significant binary digits (relative change <= 2^-bits ~ 1.5e-11).
    Every cell coordinate R * k / 2^L with k < 2^(53 - bits) is then an exact double, so the
    refinement sums are exact and the mesh is exactly mirror-symmetric under z -> -z in floating
    point (the library's mirror kernels require bit-exact mirrored points)."""
    m, e = math.frexp(R)
    return math.ldexp(round(m * 2.0 ** bits), e - bits)


def _roots(R: float):
    return [(0.0, -R, R), (0.0, 0.0, R)]


def _split(c):
    r0, z0, h = c
    g = 0.5 * h
    return [(r0, z0, g), (r0 + g, z0, g), (r0, z0 + g, g), (r0 + g, z0 + g, g)]


def refine_uniform(cells, times: int = 1):
    for _ in range(times):
        out = []
        for c in cells:
            out.extend(_split(c))
        cells = out
    return cells


def refine_origin(cells, times: int = 1):
    """Refine every cell whose closed square contains the origin (r, z) = (0, 0)."""
    for _ in range(times):
        out = []
        for c in cells:
            r0, z0, h = c
            if r0 == 0.0 and (z0 == 0.0 or z0 + h == 0.0):
                out.extend(_split(c))
            else:
                out.append(c)
        cells = out
    return cells


def uniform_mesh(R: float, nr: int):
    """nr x 2nr uniform cells on [0,R] x [-R,R] (h = R/nr)."""
    h = R / nr
    return [(i * h, -R + j * h, h) for j in range(2 * nr) for i in range(nr)]


def origin_chain(R: float, k: int):
    """Two R x R roots, then k successive refinements of the cells touching the origin: 2 + 6k cells.

    k = 3 is 'mesh A' (20 cells, = one uniform refinement followed by two origin refinements),
    the paper's 20-cell Maxwellian grid (PAPER.md:1@26927, Table I text @29286)."""
    return refine_origin(_roots(R), k)


@dataclass
class Species:
    name: str
    mass: float     # m_e units
    charge: float   # e units
    grid: int


@dataclass
class Problem:
    """Everything landau_create/landau_set_state need, plus the analytic f recipe."""
    name: str
    order: int
    grids: list                      # list of (R, cells[n][3])
    species: list                    # list[Species]
    nu: float = 1.0
    # f recipe per species: list of (density, T, drift_z) Maxwellian components
    fmix: list = field(default_factory=list)
    seed: int = 0
    noise: float = 0.01

    @property
    def radius(self):
        return np.array([g[0] for g in self.grids], dtype=np.float64)

    @property
    def ncells(self):
        return np.array([len(g[1]) for g in self.grids], dtype=np.int64)

    @property
    def cells(self):
        return np.ascontiguousarray(np.concatenate([np.asarray(g[1], dtype=np.float64).reshape(-1, 3)
                                                    for g in self.grids]), dtype=np.float64)

    @property
    def mass(self):
        return np.array([s.mass for s in self.species], dtype=np.float64)

    @property
    def charge(self):
        return np.array([s.charge for s in self.species], dtype=np.float64)

    @property
    def grid_of(self):
        return np.array([s.grid for s in self.species], dtype=np.int32)

    @property
    def npoints(self):
        return int(self.ncells.sum()) * (self.order + 1) ** 2


# ----------------------------------------------------------------------------------------------
# counter-based noise: splitmix64 keyed by (seed, species, exact node lattice position)
# ----------------------------------------------------------------------------------------------
_M64 = (1 << 64) - 1


def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = (x + np.uint64(0x9E3779B97F4A7C15)).astype(np.uint64)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def lattice_key(x: np.ndarray, R: float) -> np.ndarray:
    """Exact integer lattice coordinate of a node coordinate in [-R, R]: every node of a Q_p
    (p in 2,3,4) quadtree cell of level <= 22 is an integer multiple of R / (12 * 2^22)."""
    return np.rint((np.asarray(x, dtype=np.float64) + R) / R * (12.0 * 2.0 ** 22)).astype(np.int64)


def xi_noise(seed: int, species: int, r: np.ndarray, z: np.ndarray, R: float) -> np.ndarray:
    """xi ~ U(-1, 1), a pure function of (seed, species, node position)."""
    kr = lattice_key(r, R).astype(np.uint64)
    kz = lattice_key(z, R).astype(np.uint64)
    with np.errstate(over="ignore"):
        h = _splitmix64(np.uint64(seed) * np.uint64(0x100000001B3) + np.uint64(species + 1))
        h = _splitmix64(h ^ kr)
        h = _splitmix64(h ^ (kz * np.uint64(0x9E3779B97F4A7C15)))
    u = (h >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)   # [0, 1)
    return 2.0 * u - 1.0


def maxwellian(r, z, n, T, m, u=0.0):
    """n (pi theta)^(-3/2) exp(-(r^2 + (z-u)^2)/theta), theta = (pi/4) T/m  (App. A units, Amb-18)."""
    th = theta(T, m)
    return n * (math.pi * th) ** -1.5 * np.exp(-(np.asarray(r) ** 2 + (np.asarray(z) - u) ** 2) / th)


def maxwellian_grad(r, z, n, T, m, u=0.0):
    th = theta(T, m)
    f = maxwellian(r, z, n, T, m, u)
    return -2.0 * np.asarray(r) / th * f, -2.0 * (np.asarray(z) - u) / th * f


def f_species(prob: Problem, a: int, r, z, with_noise: bool = True):
    sp = prob.species[a]
    val = np.zeros_like(np.asarray(r, dtype=np.float64))
    for (n, T, u) in prob.fmix[a]:
        val = val + maxwellian(r, z, n, T, sp.mass, u)
    if with_noise and prob.noise != 0.0:
        R = prob.grids[sp.grid][0]
        val = val * (1.0 + prob.noise * xi_noise(prob.seed, a, r, z, R))
    return val


def coefficients(prob: Problem, nodes_per_grid, with_noise: bool = True) -> np.ndarray:
    """FE coefficient vector (species-major) = nodal interpolant of f at the given DOF nodes.

    ``nodes_per_grid[g] = (r[ndof_g], z[ndof_g])`` comes from whoever owns the numbering (the CUDA
    library via landau_get_nodes, or the oracle)."""
    out = []
    for a, sp in enumerate(prob.species):
        r, z = nodes_per_grid[sp.grid]
        out.append(f_species(prob, a, r, z, with_noise))
    return np.ascontiguousarray(np.concatenate(out), dtype=np.float64)


# ----------------------------------------------------------------------------------------------
# NEXT-3 thermal-quench source S_a(t) of Eq. 1 / Eq. 4 (PAPER.md:1@6337, @8216): "a pulse of cold ions
# is injected with the source term" (@34560), "the profile n_e is the prescribed sinusoidal source
# function", "the total mass injected by the model is five times the initial density" (@35736).
# Readings (R-7): every species is injected (quasi-neutral: electrons with the ions), as a
# Maxwellian at the cold temperature Tc of the quench bulk, with the cumulative sinusoidal profile
# P(t) = (1 - cos(pi t / t_pulse)) / 2 (0 -> 1 over the pulse); a backward-Euler step [t, t + dt]
# injects (P(t + dt) - P(t)) of the total, so the injected amounts telescope exactly.
# ----------------------------------------------------------------------------------------------
def quench_pulse_fraction(t0: float, t1: float, t_pulse: float) -> float:
    """Fraction of the pulse's total injection that falls in [t0, t1] (cumulative sinusoidal profile)."""
    P = lambda t: 0.5 * (1.0 - math.cos(math.pi * min(max(t, 0.0), t_pulse) / t_pulse))
    return P(t1) - P(t0)


def quench_source_shape(prob: Problem, nodes_per_grid, Tc: float = 0.1, density=None) -> np.ndarray:
    """FE coefficients (species-major, the caller's DOF numbering) of the cold Maxwellians a quench
    pulse injects: species a at temperature Tc with density[a] (default: the initial density of the
    species' recipe, sum of its Maxwellian components).  The step's source is sigma = fraction x
    factor x shape (factor = 5 for the paper's five-fold injection)."""
    out = []
    for a, sp in enumerate(prob.species):
        r, z = nodes_per_grid[sp.grid]
        n = density[a] if density is not None else sum(c[0] for c in prob.fmix[a])
        out.append(maxwellian(r, z, n, Tc, sp.mass))
    return np.ascontiguousarray(np.concatenate(out), dtype=np.float64)


# ----------------------------------------------------------------------------------------------
# the five configurations of BASELINE.json (concretised in SURVEY.md §8(d))
# ----------------------------------------------------------------------------------------------
R_E = dyadic_radius(5.0 * VTH_E)   # 5 v_th,e (PAPER.md:1@26988), dyadic-rounded (exact mirror)


def config1() -> Problem:
    """C1: electrons, Q2, uniform 2x4 cells on [0,R]x[-R,R], Maxwellian T_e = 1."""
    return Problem("C1", 2, [(R_E, uniform_mesh(R_E, 2))],
                   [Species("e", 1.0, -1.0, 0)], fmix=[[(1.0, 1.0, 0.0)]], seed=20219, noise=0.01)


C2_CHAIN = 11   # 2 + 6*11 = 68 cells


def c2_mesh(R: float = R_E):
    return origin_chain(R, C2_CHAIN)


def _quench_mix(Tc: float, nh: float):
    ne_c = 5.0
    return [[(ne_c, Tc, 0.0), (nh, 1.0, 0.5 * VTH_E)], [(ne_c + nh, Tc, 0.0)]]


def config2(seed: int = 20220, Tc: float = 0.1, nh: float = 1.0) -> Problem:
    """C2: e + D on one Q3 AMR grid (68 cells), thermal-quench f: cold bulk + drifting hot tail."""
    return Problem("C2", 3, [(R_E, c2_mesh())],
                   [Species("e", 1.0, -1.0, 0), Species("D", M_D, 1.0, 0)],
                   fmix=_quench_mix(Tc, nh), seed=seed)


def config3() -> Problem:
    """C3: e, D, W(Z=10), each on its own mesh-A grid with R_s = 5 v_th,s, all at T = T_e."""
    sp = [Species("e", 1.0, -1.0, 0), Species("D", M_D, 1.0, 1), Species("W", M_W, 10.0, 2)]
    dens = [1.0, 0.9, 0.01]
    grids = []
    for s in sp:
        R = dyadic_radius(5.0 * vth(1.0, s.mass))
        grids.append((R, origin_chain(R, 3)))
    return Problem("C3", 3, grids, sp, fmix=[[(n, 1.0, 0.0)] for n in dens], seed=20221)


def config4_vertex(b: int, nbatch: int = 1024) -> Problem:
    """C4 vertex b: C2 mesh; T_c = 0.05 * 10^(b/(nbatch-1)), n_h = 0.5 + b/(nbatch-1), seed 20220 + b."""
    t = b / max(nbatch - 1, 1)
    return config2(seed=20220 + b, Tc=0.05 * 10.0 ** t, nh=0.5 + t)


def config5() -> Problem:
    """C5: C2 mesh refined uniformly 3x (4352 cells), Q4, e + D thermal-quench f (N = 108,800)."""
    p = config2()
    p.name = "C5"
    p.order = 4
    p.grids = [(R_E, refine_uniform(c2_mesh(), 3))]
    return p


def config2ncu() -> Problem:
    """C2-ncu: the C2 problem on its mesh refined uniformly once (272 cells, N = 4,352),
    the analogue of the paper's 320-cell problem sized to fill the GPU for Nsight Compute (@40473)."""
    p = config2()
    p.name = "C2ncu"
    p.grids = [(R_E, refine_uniform(c2_mesh(), 1))]
    return p


CONFIGS = {"C1": config1, "C2": config2, "C3": config3, "C5": config5, "C2ncu": config2ncu}


# ------------------------------------------------------------------------------------------------
# NEXT-4 (3D Cartesian variant): a point set and synthetic fields for the 3D inner integral
# ------------------------------------------------------------------------------------------------
def points3d(ncell: int = 4, order: int = 3, R: float = R_E):
    """Tensor-product Gauss-Legendre points ((order+1)^3 per cube) of a uniform ncell^3 grid of cubes on
    [-R, R]^3: xyz [3][n] and the quadrature weights w [n] (cube-major, then z, y, x)."""
    q = order + 1
    g, gw = np.polynomial.legendre.leggauss(q)
    h = 2.0 * R / ncell
    c0 = -R + h * np.arange(ncell)
    X, Y, Z, W = [], [], [], []
    for cz in c0:
        for cy in c0:
            for cx in c0:
                for a in range(q):
                    for b in range(q):
                        for c in range(q):
                            X.append(cx + 0.5 * h * (g[c] + 1.0))
                            Y.append(cy + 0.5 * h * (g[b] + 1.0))
                            Z.append(cz + 0.5 * h * (g[a] + 1.0))
                            W.append(gw[a] * gw[b] * gw[c] * (0.5 * h) ** 3)
    return np.array([X, Y, Z]), np.array(W)


def fields3d(xyz, w, seed: int = 20222):
    """Synthetic w T_D [n] and w T_K [3][n] with the shape of the thermal-quench case (a cold bulk
    plus a drifting hot tail, electrons): a Maxwellian mix g(v) and its gradient, times the weights,
    times (1 + 0.01 xi) with xi ~ U(-1, 1) from a seeded generator."""
    x, y, z = xyz
    rng = np.random.default_rng(seed)
    g = np.zeros_like(x)
    grad = np.zeros_like(xyz)
    for n, T, u in ((5.0, 0.1, 0.0), (1.0, 1.0, 0.5 * VTH_E)):
        th = theta(T, 1.0)
        f = n * (math.pi * th) ** -1.5 * np.exp(-(x ** 2 + y ** 2 + (z - u) ** 2) / th)
        g += f
        grad += np.array([-2.0 * x / th * f, -2.0 * y / th * f, -2.0 * (z - u) / th * f])
    xi = 1.0 + 0.01 * rng.uniform(-1.0, 1.0, size=x.size)
    return w * g * xi, w * grad * xi


# ------------------------------------------------------------------------------------------------
# NEXT-4 completed: a 3D Cartesian Jacobian configuration (uniform ncell^3 Q_p cubes over [-R, R]^3)
# ------------------------------------------------------------------------------------------------
@dataclass
class Problem3D:
    name: str
    ncell: int
    order: int
    R: float
    species: list            # [(mass, charge)]
    fmix: list               # per species [(n, T, u_z)]: Maxwellians drifting along z
    seed: int = 20223
    noise: float = 0.01
    nu: float = 1.0


def config3d(ncell: int = 4, order: int = 3) -> Problem3D:
    """Electrons with the thermal-quench shape of C2 (cold bulk + drifting hot tail) and a light
    synthetic ion (m = 4 m_e, T = 4 T_e, so that its Maxwellian is resolved on the electron-scale grid:
    the test exercises the species factors, not a physical mass ratio), on [-R_E, R_E]^3."""
    return Problem3D("C3D", ncell, order, R_E, [(1.0, -1.0), (4.0, 1.0)],
                     fmix=[[(5.0, 0.1, 0.0), (1.0, 1.0, 0.5 * VTH_E)], [(6.0, 4.0, 0.0)]])


def coefficients3d(prob: Problem3D, xyz, with_noise: bool = True) -> np.ndarray:
    """[S][ndof] nodal values of each species' Maxwellian mix at the DOF nodes xyz [3][ndof] (whoever
    owns the numbering), times (1 + noise xi), xi ~ U(-1, 1) from a seeded generator per species."""
    x, y, z = (np.asarray(c, dtype=np.float64) for c in xyz)
    out = []
    for a, (m, _) in enumerate(prob.species):
        v = np.zeros_like(x)
        for (n, T, u) in prob.fmix[a]:
            th = theta(T, m)
            v = v + n * (math.pi * th) ** -1.5 * np.exp(-(x ** 2 + y ** 2 + (z - u) ** 2) / th)
        if with_noise and prob.noise != 0.0:
            v = v * (1.0 + prob.noise * np.random.default_rng(prob.seed + a).uniform(-1.0, 1.0, size=x.size))
        out.append(v)
    return np.ascontiguousarray(np.stack(out), dtype=np.float64)
