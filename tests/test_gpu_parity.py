"""GPU parity: the CUDA path (through the C ABI) against the independent C oracle on the same seeded
inputs (SURVEY.md §8(c) parity metric):

  * point-level G (step a-2):   |G_gpu - G_ora| <= 1e-12 G^abs           (every point, every component)
  * Jacobian entries (a-1..a-5): |J_gpu - J_ora| <= 1e-11 J^abs          (every stored entry, CSR and COO)
  * conservation of the GPU Jacobian: density, momentum, energy <= 1e-13 (normalised by |psi|^T |J| |f|)
  * mass (a-6):                  |M_gpu - M_ora| <= 1e-14 max_row |M|
  * determinism: repeated builds are bitwise identical (no atomics, Amb-15)

Each side computes its own coefficients from its own DOF node list with the shared generator.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from oracle.oracle import Oracle  # noqa: E402
from paper_conf_ipps_adamsbkw22_b200 import inputs  # noqa: E402
from paper_conf_ipps_adamsbkw22_b200 import landau as L  # noqa: E402

DEV = "cuda:0"


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


_cache = {}


def setup(cfg):
    if cfg not in _cache:
        prob = inputs.CONFIGS[cfg]() if isinstance(cfg, str) else cfg
        h = L.Landau.from_problem(prob, device=0)
        o = Oracle(prob)
        f_gpu = inputs.coefficients(prob, h.all_nodes())
        f_ora = o.coefficients()
        _cache[cfg] = (prob, h, o, f_gpu, f_ora)
    return _cache[cfg]


def gpu_jacobian(h, f, fmt=L.LANDAU_CSR):
    ft = torch.tensor(f, device=DEV)
    h.set_state(ft)
    out = torch.full((h.nnz if fmt == L.LANDAU_CSR else h.ncoo,), float("nan"), dtype=torch.float64, device=DEV)
    h.jacobian(out, fmt)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def gpu_G(h, f):
    h.set_state(torch.tensor(f, device=DEV))
    G = torch.full((5, h.npoints), float("nan"), dtype=torch.float64, device=DEV)
    h.point_coeffs(G)
    torch.cuda.synchronize()
    return G.cpu().numpy()


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_point_coeffs_parity(cfg):
    prob, h, o, fg, fo = setup(cfg)
    G = gpu_G(h, fg)
    Go, Ga = o.point_coeffs(fo)
    err = np.abs(G - Go) / Ga
    assert np.all(np.isfinite(G))
    assert err.max() <= 1e-12, (cfg, err.max(), np.unravel_index(err.argmax(), err.shape))


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_jacobian_csr_parity(cfg):
    prob, h, o, fg, fo = setup(cfg)
    J = gpu_jacobian(h, fg)
    Jo, Ja = o.jacobian(fo)
    assert np.all(np.isfinite(J))
    bad = np.abs(J - Jo) > 1e-11 * Ja
    assert not bad.any(), (cfg, np.max(np.abs(J - Jo) / Ja), np.abs(J - Jo).max() / np.abs(Jo).max())
    # the summary numbers of SURVEY §8(c)
    big = np.abs(Jo) >= 1e-3 * Ja
    rel = np.abs(J - Jo)[big] / np.abs(Jo)[big]
    assert np.mean(rel <= 1e-11) > 0.999


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_jacobian_coo_parity(cfg):
    prob, h, o, fg, fo = setup(cfg)
    J = gpu_jacobian(h, fg, L.LANDAU_COO)
    Jo, Ja = o.jacobian_coo(fo)
    assert np.all(np.abs(J - Jo) <= 1e-11 * Ja)


def _conservation(prob, h, J, f):
    rp, col = h.pattern()
    row = np.repeat(np.arange(h.ndof), np.diff(rp))
    nodes = h.all_nodes()
    start = 0
    tot = np.zeros(4)
    dens = []
    for a, s in enumerate(prob.species):
        nd = h.grid_ndof(s.grid)
        sel = (row >= start) & (row < start + nd)
        rr, cc = row[sel] - start, col[sel] - start
        fa = f[start:start + nd]
        Jf = np.bincount(rr, J[sel] * fa[cc], minlength=nd)
        Jaf = np.bincount(rr, np.abs(J[sel]) * np.abs(fa[cc]), minlength=nd)
        nr, nz = nodes[s.grid]
        dens.append(abs(Jf.sum()) / Jaf.sum())
        v2 = nr ** 2 + nz ** 2
        tot += s.mass * np.array([nz @ Jf, np.abs(nz) @ Jaf, v2 @ Jf, v2 @ Jaf])
        start += nd
    return max(dens), abs(tot[0]) / tot[1], abs(tot[2]) / tot[3]


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_conservation_of_gpu_jacobian(cfg):
    prob, h, o, fg, fo = setup(cfg)
    J = gpu_jacobian(h, fg)
    d, m, e = _conservation(prob, h, J, fg)
    assert d < 1e-13 and m < 1e-13 and e < 1e-13, (d, m, e)


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_mass_parity(cfg):
    prob, h, o, fg, fo = setup(cfg)
    shift = 3.25
    for fmt, ref in ((L.LANDAU_CSR, o.mass(shift)), (L.LANDAU_COO, o.mass_coo(shift))):
        out = torch.full((h.nnz if fmt == L.LANDAU_CSR else h.ncoo,), float("nan"), dtype=torch.float64, device=DEV)
        h.mass(shift, out, fmt)
        M = out.cpu().numpy()
        if fmt == L.LANDAU_CSR:
            rp, _ = h.pattern()
            rowmax = np.maximum.reduceat(np.abs(ref), rp[:-1])
            scale = np.repeat(rowmax, np.diff(rp))
        else:
            scale = np.abs(ref).max()
        assert np.all(np.abs(M - ref) <= 1e-14 * scale)


def test_determinism_bitwise():
    prob, h, o, fg, fo = setup("C2")
    a = gpu_jacobian(h, fg)
    b = gpu_jacobian(h, fg)
    assert np.array_equal(a.view(np.uint64), b.view(np.uint64))


def test_zero_state_gives_zero_jacobian():
    prob, h, o, fg, fo = setup("C2")
    J = gpu_jacobian(h, np.zeros_like(fg))
    assert np.all(J == 0.0)


def test_host_entry_point_matches_device_path():
    prob, h, o, fg, fo = setup("C2")
    J = gpu_jacobian(h, fg)
    fh = torch.tensor(fg).reshape(1, -1).pin_memory()
    vh = torch.empty((1, h.nnz), dtype=torch.float64).pin_memory()
    h.jacobian_host(fh, vh)
    assert np.array_equal(vh.numpy()[0], J)


def test_batched_vertices_C4_recipe():
    """C4: independent vertex grids sharing the C2 mesh, batched in one launch per kernel."""
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    verts = [0, 341, 682, 1023]
    probs = [inputs.config4_vertex(b) for b in verts]
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(p, nodes) for p in probs]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((len(verts), h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    torch.cuda.synchronize()
    Jb = out.cpu().numpy()
    for k, p in enumerate(probs):
        o = Oracle(p)
        Jo, Ja = o.jacobian(o.coefficients())
        assert np.all(np.abs(Jb[k] - Jo) <= 1e-11 * Ja), verts[k]
    # batch item k equals the single-vertex build (split-j grouping may differ: not bitwise)
    single = gpu_jacobian(h, F[2].cpu().numpy())
    assert np.abs(single - Jb[2]).max() <= 1e-13 * np.abs(Jb[2]).max()


def test_C5_sampled_elements():
    """C5 (Q4, 4352 cells, N = 108,800) at full size: the oracle computes every pair for the points of
    32 seeded-random cells (800 targets); compare point-level G there and the COO element blocks of those cells."""
    prob = inputs.config5()
    h = L.Landau.from_problem(prob, device=0)
    o = Oracle(prob)
    fg = inputs.coefficients(prob, h.all_nodes())
    fo = o.coefficients()
    rng = np.random.default_rng(2022)
    ncell = len(prob.grids[0][1])
    cells = np.sort(rng.choice(ncell, 32, replace=False))   # 32 elements, 800 targets
    nqp = (prob.order + 1) ** 2
    targets = (cells[:, None] * nqp + np.arange(nqp)[None, :]).ravel()
    G = gpu_G(h, fg)
    Go, Ga = o.point_coeffs(fo, targets)
    assert np.max(np.abs(G[:, targets] - Go) / Ga) <= 1e-12
    Jc = gpu_jacobian(h, fg, L.LANDAU_COO)
    mask = np.zeros(ncell, dtype=np.uint8)
    mask[cells] = 1
    Jo, Ja = o.jacobian_coo(fo, mask)
    sel = np.isfinite(Jo)
    assert sel.sum() > 0
    assert np.all(np.abs(Jc[sel] - Jo[sel]) <= 1e-11 * Ja[sel])


def test_error_codes():
    prob = inputs.config1()
    h = L.Landau.from_problem(prob, device=0)
    out = torch.empty(h.nnz, dtype=torch.float64, device=DEV)
    with pytest.raises(L.LandauError) as ei:
        h.jacobian(out)
    assert ei.value.code == L.LANDAU_ESTATE
    h.set_state(torch.zeros(h.ndof, dtype=torch.float64, device=DEV))
    with pytest.raises(ValueError):
        h.jacobian(out, 7)                 # the binding refuses an unknown format ...
    import ctypes                          # ... and so does the library itself
    assert L.lib().landau_jacobian(h._h, ctypes.c_void_p(out.data_ptr()), 7) == L.LANDAU_EINVAL
    with pytest.raises(L.LandauError) as ei:
        h.jacobian_batched(torch.empty((2, h.nnz), dtype=torch.float64, device=DEV))
    assert ei.value.code == L.LANDAU_ESTATE


def test_launch_counter_and_timers():
    prob, h, o, fg, fo = setup("C2")
    n0 = h.launch_count()
    h.set_timing(True)
    gpu_jacobian(h, fg)
    t = h.get_timing()
    h.set_timing(False)   # the cached handle goes back to the untimed (fused single-build) path
    assert h.launch_count() > n0
    assert t["inner"][1] == 1 and t["inner"][0] > 0


def test_element_split_mode_single_rank():
    """LANDAU_DIST_ELEMENTS at world = 1: NCCL communicator, the all-gather of G and the chunked layout
    run on the device and give the same Jacobian, bit for bit, as the plain handle."""
    prob, h, o, fg, fo = setup("C2")
    dist = {"rank": 0, "world": 1, "mode": L.LANDAU_DIST_ELEMENTS, "nccl_unique_id": L.landau_nccl_unique_id()}
    hd = L.Landau.from_problem(prob, device=0, dist=dist)
    # a handle with a communicator never runs the fused single-build kernel: compare with the plain
    # handle's multi-kernel build (stage timers on select it), bit for bit, and with its fused build
    # within rounding (the fused kernel groups the source splits differently)
    h.set_timing(True)
    a = gpu_jacobian(h, fg)
    h.set_timing(False)
    a_fused = gpu_jacobian(h, fg)
    b = gpu_jacobian(hd, fg)
    assert np.array_equal(a.view(np.uint64), b.view(np.uint64))
    _, Ja = o.jacobian(fo)
    assert np.max(np.abs(a_fused - b) / Ja) <= 1e-14
    hd.set_timing(True)
    gpu_jacobian(hd, fg)
    tm = hd.get_timing()
    assert tm["allgather"][1] == 1 and tm["allgather"][0] > 0.0   # one timed exchange step per build
    Gd = gpu_G(hd, fg)
    h.set_timing(True)   # the split rule of the multi-kernel build, as on the communicator handle
    Gh = gpu_G(h, fg)
    h.set_timing(False)
    assert np.array_equal(Gd, Gh)


@pytest.mark.parametrize("cfg,fmt", [("C1", L.LANDAU_CSR), ("C2", L.LANDAU_CSR), ("C3", L.LANDAU_CSR), ("C2", L.LANDAU_COO)])
def test_fused_single_build_matches_direct_launches(cfg, fmt):
    """Single builds run as one cooperative kernel (kernels_single.cuh: fields, mirror-directed inner
    integral, split reduction, element matrices, assembly separated by grid barriers), replayed from a
    CUDA graph; with per-stage timers the same build runs as six separate kernels.  Both agree up to the
    grouping of the inner integral's split sums (the fused kernel adds 8 splits per CTA first), replays
    repeat bit for bit, and the fused build matches the oracle."""
    prob, h, o, fg, fo = setup(cfg)
    h.set_timing(True)           # timers force the multi-kernel path
    a = gpu_jacobian(h, fg, fmt)
    t = h.get_timing()
    assert t["inner"][1] == 1 and t["element"][1] == 1
    h.set_timing(False)          # fused single kernel (captured on first use, replayed after)
    n0 = h.launch_count()
    b = gpu_jacobian(h, fg, fmt)
    c = gpu_jacobian(h, fg, fmt)
    assert h.launch_count() - n0 == 2   # one kernel per build
    assert np.array_equal(b.view(np.uint64), c.view(np.uint64))
    Jo, Ja = o.jacobian(fo) if fmt == L.LANDAU_CSR else o.jacobian_coo(fo)
    assert np.all(np.abs(b - Jo) <= 1e-11 * Ja)
    assert np.all(np.abs(a - b) <= 1e-14 * Ja)


@pytest.mark.parametrize("mirror", [True, False, "vertex"])
def test_symmetric_kernel_batch_C4(mirror):
    """A batch large enough for the symmetric inner kernel (each unordered pair evaluated once, both
    targets updated; with mirror=True also each z-mirrored pair from the same tensor): vertices
    against the oracle, conservation, and bitwise determinism."""
    nb = 24
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    h.set_mirror(mirror)
    verts = [int(round(k * 1023 / (nb - 1))) for k in range(nb)]
    probs = [inputs.config4_vertex(b) for b in verts]
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(p, nodes) for p in probs]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.set_timing(True)
    h.jacobian_batched(out)
    t = h.get_timing()
    h.set_timing(False)
    # the slot kernels reduce their partial slots; the per-vertex kernel sums in shared memory
    assert t["reduce"][1] == (0 if mirror == "vertex" else 1)
    assert h.stats()["inner_path"] == {True: 3, False: 1, "vertex": 4}[mirror]
    Jb = out.cpu().numpy()
    for k in (0, nb // 2, nb - 1):
        o = Oracle(probs[k])
        fo = o.coefficients()
        Jo, Ja = o.jacobian(fo)
        assert np.all(np.abs(Jb[k] - Jo) <= 1e-11 * Ja), verts[k]
        d, m, e = _conservation(probs[k], h, Jb[k], inputs.coefficients(probs[k], nodes))
        assert d < 1e-13 and m < 1e-13 and e < 1e-13, (d, m, e)
    h.jacobian_batched(out)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), Jb.view(np.uint64))
    G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
    h.point_coeffs_batched(G)
    o = Oracle(probs[5])
    Go, Ga = o.point_coeffs(o.coefficients())
    assert np.max(np.abs(G[5].cpu().numpy() - Go) / Ga) <= 1e-12


def test_host_entry_pipelined_chunks_match_device_batch():
    """landau_jacobian_host splits a large batch into chunks whose uploads, builds and downloads
    overlap on three streams; every vertex must come back equal to the device-side batch up to the
    summation grouping (a chunk's stream-K split differs from the whole batch's: vertices cut between
    CTAs add their partials in another grouping), and bitwise repeatable."""
    nb = 130
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    F = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 1024 // nb)][:nb])
    Fd = torch.tensor(F, device=DEV)
    h.set_state_batched(Fd)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    ref = out.cpu().numpy()
    fh = torch.tensor(F).pin_memory()
    vh = torch.full((nb, h.nnz), float("nan"), dtype=torch.float64).pin_memory()
    h.jacobian_host(fh, vh)
    got = vh.numpy().copy()
    assert np.all(np.abs(got - ref) <= 1e-14 * np.abs(ref).max(axis=1, keepdims=True))
    h.jacobian_host(fh, vh)
    assert np.array_equal(vh.numpy().view(np.uint64), got.view(np.uint64))


def test_symmetric_kernel_with_coincident_points():
    """Two species on two identical grids: every point has a distinct twin with identical (r, z), so
    the library must take the masked symmetric kernel (Amb-3: coincident pairs contribute nothing)."""
    R = inputs.R_E
    mesh = inputs.origin_chain(R, 3)
    prob = inputs.Problem("twin", 3, [(R, mesh), (R, mesh)],
                          [inputs.Species("e", 1.0, -1.0, 0), inputs.Species("D", inputs.M_D, 1.0, 1)],
                          fmix=[[(1.0, 1.0, 0.0)], [(1.0, 0.5, 0.0)]], seed=99)
    h = L.Landau.from_problem(prob, device=0)
    nodes = h.all_nodes()
    nb = 48
    fs = []
    for b in range(nb):
        p = inputs.Problem("twin", 3, prob.grids, prob.species, fmix=[[(1.0 + 0.01 * b, 1.0, 0.0)], [(1.0, 0.5, 0.0)]],
                           seed=99 + b)
        fs.append(inputs.coefficients(p, nodes))
    h.set_state_batched(torch.tensor(np.stack(fs), device=DEV))
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    torch.cuda.synchronize()
    assert h.stats()["inner_path"] == 3   # the twin mesh is z-symmetric too: masked mirror kernel
    Jb = out.cpu().numpy()
    h.set_mirror(False)
    out2 = torch.empty_like(out)
    h.jacobian_batched(out2)
    torch.cuda.synchronize()
    assert h.stats()["inner_path"] == 1   # masked plain symmetric kernel
    assert np.abs(out2.cpu().numpy() - Jb).max() <= 1e-13 * np.abs(Jb).max()
    h.set_mirror("vertex")
    out3 = torch.empty_like(out)
    h.jacobian_batched(out3)
    torch.cuda.synchronize()
    assert h.stats()["inner_path"] == 4   # masked per-vertex mirror kernel
    assert np.abs(out3.cpu().numpy() - Jb).max() <= 1e-13 * np.abs(Jb).max()
    for b in (0, nb - 1):
        p = inputs.Problem("twin", 3, prob.grids, prob.species, fmix=[[(1.0 + 0.01 * b, 1.0, 0.0)], [(1.0, 0.5, 0.0)]],
                           seed=99 + b)
        o = Oracle(p)
        Jo, Ja = o.jacobian(o.coefficients())
        assert np.all(np.abs(Jb[b] - Jo) <= 1e-11 * Ja)


def _adhoc(order, mesh, species_grid=(0, 0)):
    R = inputs.R_E
    sp = [inputs.Species("e", 1.0, -1.0, species_grid[0]), inputs.Species("D", inputs.M_D, 1.0, species_grid[1])]
    grids = [(R, mesh)] * (max(species_grid) + 1)
    return inputs.Problem(f"Q{order}", order, grids, sp, fmix=[[(1.0, 1.0, 0.0), (0.3, 0.2, 0.4)], [(1.3, 0.5, 0.0)]],
                          seed=4242 + order)


@pytest.mark.parametrize("order,mesh", [(4, "A"), (2, "C2"), (4, "chain6")])
def test_full_parity_other_orders(order, mesh):
    """Full-Jacobian parity (every CSR entry, every G) for Q2 and Q4 AMR meshes with hanging nodes."""
    R = inputs.R_E
    cells = {"A": inputs.origin_chain(R, 3), "C2": inputs.c2_mesh(), "chain6": inputs.origin_chain(R, 6)}[mesh]
    prob = _adhoc(order, cells)
    h = L.Landau.from_problem(prob, device=0)
    o = Oracle(prob)
    fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
    G = gpu_G(h, fg)
    Go, Ga = o.point_coeffs(fo)
    assert np.max(np.abs(G - Go) / Ga) <= 1e-12
    J = gpu_jacobian(h, fg)
    Jo, Ja = o.jacobian(fo)
    assert np.all(np.abs(J - Jo) <= 1e-11 * Ja)
    d, m, e = _conservation(prob, h, J, fg)
    assert max(d, m, e) < 1e-13, (d, m, e)


def test_tensor_cache_gemm_path_C4():
    """NEXT-4 tensor cache: the batch's inner integral as FP64 GEMMs over cached tensor matrices
    matches the oracle and the pairwise (symmetric) kernel."""
    nb = 24
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    verts = [int(round(k * 1023 / (nb - 1))) for k in range(nb)]
    probs = [inputs.config4_vertex(b) for b in verts]
    F = torch.tensor(np.stack([inputs.coefficients(p, nodes) for p in probs]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    ref = out.cpu().numpy()
    h.set_tensor_cache(True)
    h.jacobian_batched(out)
    torch.cuda.synchronize()
    assert h.stats()["inner_path"] == 2
    Jc = out.cpu().numpy()
    assert np.abs(Jc - ref).max() <= 1e-12 * np.abs(ref).max()
    for k in (0, nb - 1):
        o = Oracle(probs[k])
        Jo, Ja = o.jacobian(o.coefficients())
        assert np.all(np.abs(Jc[k] - Jo) <= 1e-11 * Ja)
    h.jacobian_batched(out)      # cached tensors reused: bitwise repeatable
    assert np.array_equal(out.cpu().numpy().view(np.uint64), Jc.view(np.uint64))
    h.set_tensor_cache("recompute")   # tensors re-evaluated in the build: the same values
    h.jacobian_batched(out)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), Jc.view(np.uint64))
    h.set_tensor_cache(False)
    h.jacobian_batched(out)
    assert h.stats()["inner_path"] in (1, 3)


def test_more_error_codes_and_coo_batched():
    prob = inputs.config2()
    h = L.Landau.from_problem(prob, device=0)
    lib = L.lib()
    import ctypes
    assert lib.landau_set_state_batched(h._h, 0, ctypes.c_void_p(16)) == L.LANDAU_EINVAL
    assert lib.landau_set_state_batched(h._h, 2, None) == L.LANDAU_EINVAL
    assert lib.landau_mass(h._h, 1.0, None, L.LANDAU_CSR) == L.LANDAU_EINVAL
    assert lib.landau_point_coeffs(h._h, None) == L.LANDAU_EINVAL
    assert "set_state" in lib.landau_last_error(h._h).decode() or lib.landau_last_error(h._h)
    # batched COO = per-vertex COO
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in (3, 700)]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((2, h.ncoo), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out, L.LANDAU_COO)
    torch.cuda.synchronize()
    for k in range(2):
        single = gpu_jacobian(h, F[k].cpu().numpy(), L.LANDAU_COO)
        assert np.abs(single - out[k].cpu().numpy()).max() <= 1e-13 * np.abs(single).max()
    # COO summed into the CSR pattern equals the CSR output
    import scipy.sparse as sps
    row, col = h.pattern(coo=True)
    rp, ccol = h.pattern()
    Jcoo = gpu_jacobian(h, F[0].cpu().numpy(), L.LANDAU_COO)
    Jcsr = gpu_jacobian(h, F[0].cpu().numpy(), L.LANDAU_CSR)
    A = sps.coo_matrix((Jcoo, (row, col)), shape=(h.ndof, h.ndof)).tocsr()
    A.sort_indices()
    assert np.abs(A.data - Jcsr).max() <= 1e-14 * np.abs(Jcsr).max()


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_band_lu_solve_matches_sparse_direct(cfg):
    """NEXT-2: the GPU band LU of A = shift M - J (RCM order, no pivoting) solves A x = b like a sparse
    direct solve (scipy SuperLU) of the oracle's own A, for an implicit-step shift."""
    import scipy.sparse as sps
    import scipy.sparse.linalg as spla
    prob, h, o, fg, fo = setup(cfg)
    J = gpu_jacobian(h, fg)
    Jo, _ = o.jacobian(fo)
    Mo = o.mass(1.0)
    shift = 1.0 * np.abs(Jo).max() / np.abs(Mo).max()
    rp, col = o.pattern()
    Ao = sps.csr_matrix((shift * Mo - Jo, col, rp), shape=(o.ndof, o.ndof))
    rng = np.random.default_rng(11)
    bvec = rng.standard_normal(o.ndof)
    x_ref = spla.spsolve(Ao.tocsc(), bvec)
    Jt = torch.tensor(J, device=DEV).reshape(1, -1)
    h.band_factor_batched(shift, Jt)
    bt = torch.tensor(bvec, device=DEV).reshape(1, -1)
    xt = torch.empty_like(bt)
    h.band_solve_batched(bt, xt)
    torch.cuda.synchronize()
    x = xt.cpu().numpy()[0]
    assert np.linalg.norm(x - x_ref) <= 1e-9 * np.linalg.norm(x_ref)
    # residual with the GPU's own A
    Ag = sps.csr_matrix((shift * Mo - J, col, rp), shape=(o.ndof, o.ndof))
    assert np.linalg.norm(Ag @ x - bvec) <= 1e-12 * (abs(Ag).sum(axis=1).max() * np.abs(x).max() * np.sqrt(o.ndof))


def test_band_lu_batched_C4():
    """Batched band factor/solve over vertices: each item matches its own sparse direct solve."""
    import scipy.sparse as sps
    import scipy.sparse.linalg as spla
    nb = 6
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 171)][:nb]),
                     device=DEV)
    h.set_state_batched(F)
    J = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(J)
    M = torch.empty(h.nnz, dtype=torch.float64, device=DEV)
    h.mass(1.0, M)
    torch.cuda.synchronize()
    Jn, Mn = J.cpu().numpy(), M.cpu().numpy()
    shift = 2.0 * np.abs(Jn).max() / np.abs(Mn).max()
    h.band_factor_batched(shift, J)
    b = torch.tensor(np.random.default_rng(5).standard_normal((nb, h.ndof)), device=DEV)
    x = torch.empty_like(b)
    h.band_solve_batched(b, x)
    torch.cuda.synchronize()
    rp, col = h.pattern()
    for k in range(nb):
        A = sps.csr_matrix((shift * Mn - Jn[k], col, rp), shape=(h.ndof, h.ndof)).tocsc()
        xr = spla.spsolve(A, b[k].cpu().numpy())
        assert np.linalg.norm(x[k].cpu().numpy() - xr) <= 1e-9 * np.linalg.norm(xr), k
    # solve in place (b aliases x)
    b2 = b.clone()
    h.band_solve_batched(b2, b2)
    assert torch.equal(b2, x)


# ------------------------------------------------------------------------------------------------
# NEXT-3: E_z advection matrix and the quasi-Newton implicit step
# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_advection_parity(cfg):
    """A_E (Eq. 4's field term) with its species factor E_z e_a / m_a, CSR and COO, against the oracle."""
    prob, h, o, fg, fo = setup(cfg)
    Ez = 0.37
    eta = Ez * (np.asarray(prob.charge, float) / np.asarray(prob.mass, float))
    rows = o.species_rows()
    rp, col = o.pattern()
    per_entry = eta[np.repeat(rows, np.diff(rp))]
    ref = per_entry * o.advection()
    out = torch.full((h.nnz,), float("nan"), dtype=torch.float64, device=DEV)
    h.advection(Ez, out)
    torch.cuda.synchronize()
    assert np.abs(out.cpu().numpy() - ref).max() <= 1e-14 * np.abs(ref).max()
    row, ccol = o.coo_pattern()
    refc = eta[rows[row]] * o.advection_coo()
    outc = torch.full((h.ncoo,), float("nan"), dtype=torch.float64, device=DEV)
    h.advection(Ez, outc, L.LANDAU_COO)
    torch.cuda.synchronize()
    assert np.abs(outc.cpu().numpy() - refc).max() <= 1e-14 * np.abs(refc).max()


@pytest.mark.parametrize("cfg", ["C1", "C3"])
def test_band_lu_with_field_matches_sparse_direct(cfg):
    import scipy.sparse as sps
    import scipy.sparse.linalg as spla
    prob, h, o, fg, fo = setup(cfg)
    J = gpu_jacobian(h, fg)
    Mo, Ao = o.mass(1.0), o.advection()
    rows = o.species_rows()
    rp, col = o.pattern()
    Ez, shift = 0.2, 10.0
    eta = Ez * (np.asarray(prob.charge, float) / np.asarray(prob.mass, float))[np.repeat(rows, np.diff(rp))]
    A = sps.csr_matrix((shift * Mo + eta * Ao - J, col, rp), shape=(o.ndof, o.ndof))
    bvec = np.random.default_rng(3).standard_normal(o.ndof)
    x_ref = spla.spsolve(A.tocsc(), bvec)
    h.band_factor_batched(shift, torch.tensor(J, device=DEV).reshape(1, -1), Ez=Ez)
    x = torch.empty((1, o.ndof), dtype=torch.float64, device=DEV)
    h.band_solve_batched(torch.tensor(bvec, device=DEV).reshape(1, -1), x)
    torch.cuda.synchronize()
    assert np.linalg.norm(x.cpu().numpy()[0] - x_ref) <= 1e-9 * np.linalg.norm(x_ref)


@pytest.mark.parametrize("cfg,dt,Ez", [("C1", 0.05, 0.0), ("C1", 0.05, 0.1), ("C3", 0.01, 0.1), ("C2", 0.02, 0.05)])
def test_implicit_step_matches_oracle_iterates(cfg, dt, Ez):
    """Every quasi-Newton iterate of the device step equals the oracle's iterate (same iteration count)."""
    prob, h, o, fg, fo = setup(cfg)
    its = o.implicit_step(fo, dt, Ez, iters=3)
    f_old = torch.tensor(fg, device=DEV).reshape(1, -1)
    f_new = torch.empty_like(f_old)
    for k in (1, 3):
        n_it, dn = h.implicit_step_batched(dt, f_old, f_new, Ez=Ez, max_iter=k, rtol=0.0)
        torch.cuda.synchronize()
        assert n_it == k
        x = f_new.cpu().numpy()[0]
        assert np.linalg.norm(x - its[k - 1]) <= 1e-10 * np.linalg.norm(its[k - 1]), (k, np.linalg.norm(x - its[k - 1]))
        prev = its[k - 2] if k > 1 else fo
        assert abs(dn - np.linalg.norm(its[k - 1] - prev) / np.linalg.norm(its[k - 1])) <= 1e-6 * dn


@pytest.mark.parametrize("cfg,dt,Ez", [("C1", 0.05, 0.1), ("C2", 0.02, 0.0), ("C3", 0.01, 0.1)])
def test_implicit_step_with_quench_source_matches_oracle(cfg, dt, Ez):
    """NEXT-3 with the source S_a(t) of Eq. 4 (a cold Maxwellian pulse, reading R-7): every device
    iterate equals the oracle's iterate with the same source (each side interpolates the shape at its
    own DOF nodes), and the device iterate satisfies the per-species density balance
    1^T [M (f^1 - f^0)/dt + eta A_E f^1] = 1^T M sigma."""
    import scipy.sparse as sps
    prob, h, o, fg, fo = setup(cfg)
    frac = 5.0 * inputs.quench_pulse_fraction(0.0, dt, 4 * dt) / dt   # rate for the first step of a 4-step pulse
    sig_o = frac * inputs.quench_source_shape(prob, o.all_nodes())
    sig_g = frac * inputs.quench_source_shape(prob, h.all_nodes())
    its = o.implicit_step(fo, dt, Ez, iters=2, src=sig_o)
    f_old = torch.tensor(fg, device=DEV).reshape(1, -1)
    f_new = torch.empty_like(f_old)
    n_it, dn = h.implicit_step_batched(dt, f_old, f_new, Ez=Ez, max_iter=2, rtol=0.0,
                                       src=torch.tensor(sig_g, device=DEV).reshape(1, -1))
    torch.cuda.synchronize()
    x = f_new.cpu().numpy()[0]
    assert n_it == 2 and np.linalg.norm(x - its[1]) <= 1e-10 * np.linalg.norm(its[1])
    M = torch.empty(h.nnz, dtype=torch.float64, device=DEV)
    A = torch.empty(h.nnz, dtype=torch.float64, device=DEV)
    h.mass(1.0, M)
    h.advection(Ez, A)
    rp, col = h.pattern()
    Mm = sps.csr_matrix((M.cpu().numpy(), col, rp), shape=(h.ndof, h.ndof))
    Am = sps.csr_matrix((A.cpu().numpy(), col, rp), shape=(h.ndof, h.ndof))
    R = Mm @ (x - fg) / dt + Am @ x - Mm @ sig_g
    start = 0
    for sp in prob.species:
        nd = h.grid_ndof(sp.grid)
        sl = slice(start, start + nd)
        assert abs(R[sl].sum()) <= 1e-12 * (np.abs(Mm) @ np.abs(x))[sl].sum() / dt
        start += nd


def test_implicit_step_converges_and_conserves_C4_batch():
    """Batched step over vertices with a tolerance: stops when every item's relative change <= rtol;
    the converged step conserves density, momentum and energy of every vertex (no field)."""
    import scipy.sparse as sps
    nb = 4
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    # the quasi-Newton iteration converges linearly, slowly for the coldest vertices: hotter ones here
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in (600, 700, 800, 1023)]),
                     device=DEV)
    Fn = torch.empty_like(F)
    dt = 0.002
    n_it, dn = h.implicit_step_batched(dt, F, Fn, max_iter=40, rtol=1e-12)
    torch.cuda.synchronize()
    assert n_it < 40 and dn <= 1e-12
    M = torch.empty(h.nnz, dtype=torch.float64, device=DEV)
    h.mass(1.0, M)
    rp, col = h.pattern()
    Mm = sps.csr_matrix((M.cpu().numpy(), col, rp), shape=(h.ndof, h.ndof))
    ng = h.grid_ndof(0)
    r, z = np.concatenate([nodes[0][0]] * 2), np.concatenate([nodes[0][1]] * 2)
    m = np.repeat(np.asarray(prob0.mass, float), ng)
    for k in range(nb):
        f0, f1 = F[k].cpu().numpy(), Fn[k].cpu().numpy()
        d0, d1 = Mm @ f0, Mm @ f1
        for a in range(2):
            sl = slice(a * ng, (a + 1) * ng)
            assert abs(d1[sl].sum() - d0[sl].sum()) <= 1e-12 * abs(d0[sl].sum())
        psi = r * r + z * z
        assert abs((m * psi * (d1 - d0)).sum()) <= 1e-10 * (m * psi * np.abs(d0)).sum()
        assert abs((m * z * (d1 - d0)).sum()) <= 1e-10 * (m * np.abs(z) * np.abs(d0)).sum()
        assert np.linalg.norm(f1 - f0) > 1e-6 * np.linalg.norm(f0)


def test_mirror_kernel_C3_C5_sampled_and_unsupported_mesh():
    """Mirror kernel on the three-grid impurity case (C3, batched) against the oracle's point
    coefficients; a mesh that is not z-symmetric refuses set_mirror(True) and still builds."""
    prob, h0, o, fg, fo = setup("C3")
    h = L.Landau.from_problem(prob, device=0)
    nb = 64   # enough items for the batched (symmetric) path
    F = torch.tensor(np.stack([fg] * nb), device=DEV)
    h.set_state_batched(F)
    G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
    Go, Ga = o.point_coeffs(fo)
    for mode, path in ((True, 4), ("slots", 3)):   # automatic (per-vertex, stream-K) and the slot kernel
        h.set_mirror(mode)
        h.point_coeffs_batched(G)
        torch.cuda.synchronize()
        assert h.stats()["inner_path"] == path
        for k in (0, nb // 2 + 1, nb - 1):
            assert np.max(np.abs(G[k].cpu().numpy() - Go) / Ga) <= 1e-12, (mode, k)
    # an asymmetric mesh: the uniform 2 x 4 mesh with one upper cell split into four
    R = inputs.R_E
    cells = inputs.uniform_mesh(R, 2)
    top = max(cells, key=lambda c: (c[1], c[0]))
    cells.remove(top)
    cells += inputs._split(top)
    asym = inputs.Problem("asym", 2, [(R, cells)], [inputs.Species("e", 1.0, -1.0, 0)],
                          fmix=[[(1.0, 1.0, 0.3)]], seed=7)
    ha = L.Landau.from_problem(asym, device=0)
    assert not _mesh_is_mirror(ha)
    with pytest.raises(L.LandauError):
        ha.set_mirror(True)
    oa = Oracle(asym)
    fa = oa.coefficients()
    J = gpu_jacobian(ha, inputs.coefficients(asym, ha.all_nodes()))
    Jo, Ja = oa.jacobian(fa)
    assert np.all(np.abs(J - Jo) <= 1e-11 * Ja)


def _mesh_is_mirror(h):
    r, z, _ = h.points()
    a = sorted(zip(r, z))
    b = sorted(zip(r, -z))
    return np.allclose(np.array(a), np.array(b), atol=1e-12)


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_vertex_kernel_point_coeffs(cfg):
    """Per-vertex mirror kernel (one CTA per batch item, sums in shared memory, round-robin tile
    schedule) on a ragged tile set (C1: H = 36, two tiles), an odd tile count (C3: 15, three grids)
    and the C2 mesh (17): point coefficients of every item against the oracle, single items and
    batches, bitwise reproducible, and equal to the slot kernel up to summation order."""
    prob, h0, o, fg, fo = setup(cfg)
    h = L.Landau.from_problem(prob, device=0)
    h.set_mirror("vertex")
    Go, Ga = o.point_coeffs(fo)
    for nb in (1, 5):
        F = torch.tensor(np.stack([fg * (1.0 + 0.1 * k) for k in range(nb)]), device=DEV)
        h.set_state_batched(F)
        G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
        h.point_coeffs_batched(G)
        torch.cuda.synchronize()
        assert h.stats()["inner_path"] == 4
        Gn = G.cpu().numpy()
        for k in range(nb):   # G is linear in f
            assert np.max(np.abs(Gn[k] - (1.0 + 0.1 * k) * Go) / ((1.0 + 0.1 * k) * Ga)) <= 1e-12, (nb, k)
        h.point_coeffs_batched(G)
        assert np.array_equal(G.cpu().numpy().view(np.uint64), Gn.view(np.uint64))
    h.set_mirror("slots")
    G2 = torch.empty_like(G)
    h.point_coeffs_batched(G2)
    torch.cuda.synchronize()
    assert np.max(np.abs(G2.cpu().numpy() - Gn) / Ga) <= 1e-13
    J = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.set_mirror("vertex")
    h.jacobian_batched(J)
    Jo, Ja = o.jacobian(fo)
    assert np.all(np.abs(J[0].cpu().numpy() - Jo) <= 1e-11 * Ja)


def test_vertex_kernel_stream_k_small_wave():
    """Automatic mode on a batch just above one vertex per SM (S + 5 vertices): the per-vertex kernel's
    stream-K split gives every SM an equal share of the (vertex, round) work, so some vertices are cut
    between CTAs and their partials are combined in CTA order.  Split and unsplit vertices against
    the oracle, the whole batch against the slot kernel, and bitwise repeatability."""
    S = torch.cuda.get_device_properties(0).multi_processor_count
    nb = S + 5
    prob0 = inputs.config4_vertex(0)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    verts = [(k * 1023) // (nb - 1) for k in range(nb)]
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in verts]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.set_timing(True)
    h.jacobian_batched(out)
    t = h.get_timing()
    h.set_timing(False)
    assert h.stats()["inner_path"] == 4
    assert t["inner"][1] == 1 and t["reduce"][1] == 0   # one inner launch, no slot reduction
    split = h.vtx_split_vertices(nb)
    assert 0 < len(split) < nb
    unsplit = np.setdiff1d(np.arange(nb), split)
    Jb = out.cpu().numpy()
    for k in (int(split[0]), int(split[-1]), int(unsplit[0]), nb - 1):
        o = Oracle(inputs.config4_vertex(verts[k]))
        Jo, Ja = o.jacobian(o.coefficients())
        assert np.all(np.abs(Jb[k] - Jo) <= 1e-11 * Ja), verts[k]
    h.jacobian_batched(out)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), Jb.view(np.uint64))
    h.set_mirror("slots")
    out2 = torch.empty_like(out)
    h.jacobian_batched(out2)
    assert h.stats()["inner_path"] == 3
    assert np.abs(out2.cpu().numpy() - Jb).max() <= 1e-13 * np.abs(Jb).max()


def test_vertex_kernel_headline_batch_1024():
    """The headline configuration as bench.py runs it: 1024 C4 vertices in automatic mode (every CTA
    loops over about seven vertices' rounds).  Vertices handled at the start, middle and end of CTA
    ranges -- including vertices split between two CTAs -- against the oracle at 1e-11 J^abs; vertices
    that ran whole on one CTA are bitwise equal to a lone build of that vertex (the same summation
    order), split ones equal to it within 1e-14 of the condition scale; and the point coefficients of
    sampled vertices against the oracle at 1e-12 G^abs."""
    nb = 1024
    prob0 = inputs.config4_vertex(0, nb)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b, nb), nodes) for b in range(nb)]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    torch.cuda.synchronize()
    assert h.stats()["inner_path"] == 4
    split = set(int(x) for x in h.vtx_split_vertices(nb))
    S = h.vtx_schedule()[1]
    assert 0 < len(split) < S
    sample = [0, 148, 500, 1023] + sorted(split)[:2] + sorted(split)[-1:]
    Jb = out.cpu().numpy()
    G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
    h.point_coeffs_batched(G)
    Gb = G.cpu().numpy()
    lone = L.Landau.from_problem(prob0, device=0)
    lone.set_mirror("vertex")
    for b in sample:
        o = Oracle(inputs.config4_vertex(b, nb))
        fo = o.coefficients()
        Jo, Ja = o.jacobian(fo)
        assert np.all(np.abs(Jb[b] - Jo) <= 1e-11 * Ja), b
        if b in (0, 500):
            Go, Ga = o.point_coeffs(fo)
            assert np.max(np.abs(Gb[b] - Go) / Ga) <= 1e-12, b
        Jl = gpu_jacobian(lone, F[b].cpu().numpy())
        assert lone.stats()["inner_path"] == 4
        if b in split:
            assert np.all(np.abs(Jl - Jb[b]) <= 1e-14 * Ja), b
        else:
            assert np.array_equal(Jl.view(np.uint64), Jb[b].view(np.uint64)), b
    h.jacobian_batched(out)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), Jb.view(np.uint64))


def test_mirror_directed_kernel_unsplit():
    """The mirror-symmetric directed kernel writes G directly when one source split suffices (a batch
    large enough to fill the GPU with target tiles alone); the pair kernels are switched off in a
    child process (LANDAU_SYM=0 is read once per process) so the path runs, and each item is checked
    against the oracle."""
    import os
    import subprocess
    import sys
    code = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
nb = 160
p0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(p0, device=0)
nodes = h.all_nodes()
verts = [0, 511, 1023]
F = np.stack([inputs.coefficients(inputs.config4_vertex(verts[k % 3]), nodes) for k in range(nb)])
h.set_state_batched(torch.tensor(F, device="cuda"))
G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device="cuda")
h.point_coeffs_batched(G)
torch.cuda.synchronize()
st = h.stats()
assert st["inner_path"] == 5 and st["nsplit"] == 1, st
for k in range(3):
    o = Oracle(inputs.config4_vertex(verts[k]))
    Go, Ga = o.point_coeffs(o.coefficients())
    e = float(np.max(np.abs(G[k].cpu().numpy() - Go) / Ga))
    assert e <= 1e-12, (k, e)
print("ok")
'''
    env = dict(os.environ, LANDAU_SYM="0")
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600, env=env,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert out.returncode == 0 and out.stdout.strip().endswith("ok"), out.stderr[-3000:]


@pytest.mark.parametrize("world", [2, 3])
def test_pair_split_partials_sum_to_G(world, monkeypatch):
    """Pair split (LANDAU_DIST_ELEMENTS on a mirror mesh): each rank runs only its landau_pair_partition
    share of the slot kernel's items and the ranks' partial G are summed by the all-reduce.  One GPU
    emulates the ranks (LANDAU_PAIR_SPLIT_EMULATE, read at create): the partials must add up to the
    full G, which matches the oracle."""
    prob, h0, o, fg, fo = setup("C3")
    nb = 64   # enough items for the slot kernel
    F = torch.tensor(np.stack([fg] * nb), device=DEV)

    def G_of(env):
        if env:
            monkeypatch.setenv("LANDAU_PAIR_SPLIT_EMULATE", env)
        else:
            monkeypatch.delenv("LANDAU_PAIR_SPLIT_EMULATE", raising=False)
        h = L.Landau.from_problem(prob, device=0)
        h.set_mirror("slots")
        h.set_state_batched(F)
        G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
        h.point_coeffs_batched(G)
        torch.cuda.synchronize()
        assert h.stats()["inner_path"] == 3
        ev = h.stats()["pair_evaluations"]
        h.close()
        return G.cpu().numpy(), ev

    Gfull, evfull = G_of(None)
    parts = [G_of(f"{world}:{r}") for r in range(world)]
    assert sum(e for _, e in parts) == evfull
    Gsum = sum(g for g, _ in parts)
    Go, Ga = o.point_coeffs(fo)
    assert np.max(np.abs(Gsum[0] - Go) / Ga) <= 1e-12
    assert np.max(np.abs(Gsum - Gfull) / Ga) <= 1e-13


@pytest.mark.parametrize("ncell,order,sub", [(3, 3, None), (2, 2, 173), (1, 2, 1)])
def test_inner3d_matches_oracle(ncell, order, sub):
    """NEXT-4: the 3D Cartesian inner integral (Eq. 3 directly) against oracle O12 on every point:
    several target tiles and source splits, a ragged size (173 points), a single point, and a twin
    point (coincident pairs excluded)."""
    from oracle import oracle as O
    xyz, w = inputs.points3d(ncell, order)
    wTD, wTK = inputs.fields3d(xyz, w)
    if sub is not None:
        xyz, wTD, wTK = xyz[:, :sub].copy(), wTD[:sub].copy(), wTK[:, :sub].copy()
    if xyz.shape[1] > 4:   # a twin of point 3 (distinct index, identical coordinates)
        xyz = np.concatenate([xyz, xyz[:, 3:4]], axis=1)
        wTD = np.concatenate([wTD, wTD[3:4]])
        wTK = np.concatenate([wTK, wTK[:, 3:4]], axis=1)
    n = xyz.shape[1]
    G = torch.full((9, n), float("nan"), dtype=torch.float64, device=DEV)
    L.landau3d_inner(torch.tensor(xyz, device=DEV), torch.tensor(wTD, device=DEV), torch.tensor(wTK, device=DEV), G)
    torch.cuda.synchronize()
    Go, Ga = O.inner3d(xyz[0], xyz[1], xyz[2], wTD, wTK)
    Gg = G.cpu().numpy()
    assert np.all(np.isfinite(Gg))
    assert np.max(np.abs(Gg - Go) / np.maximum(Ga, 1e-300)) <= 1e-13


def test_bench_gpu_arm_json_line():
    """The driver's contract for the GPU arm: one JSON line with the base keys, roofline, cpu_baseline,
    e2e, clocks and a non-zero launch count of this library's kernels."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--steps", "3", "--warmup", "3",
                          "--cpu-sample", "2", "--c5-cells", "2"],
                         capture_output=True, text=True, timeout=900, cwd=root)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"):
        assert k in d, k
    assert d["value"] > 0 and d["steps"] == 3 and d["warmup"] == 3 and d["scaling"] == "strong"
    assert d["config"]["vertices"] == 1024
    for name in ("C1", "C2", "C3", "C5"):
        assert d["configs"][name]["value"] > 0, name
    assert d["configs"]["C5"]["parity"]["max_dJ_over_Jabs"] <= 1e-11
    assert d["configs"]["C2"]["parity_max_dJ_over_Jabs"] <= 1e-11
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1 and r["peak"] > 30
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0 and d["e2e"]["value"] > 0
    assert d["gpu_launches"] > 0 and d["config"]["workload"].startswith("C4")


def _balanced_random_mesh(rng, R, nsplit, mirror):
    """Two R x R roots refined at random (mirror: every split applied to the z -> -z image too), then
    2:1-balanced by splitting any cell with an edge neighbour more than one level finer."""
    cells = [(0.0, -R, R), (0.0, 0.0, R)]
    for _ in range(nsplit):
        c = cells[rng.integers(len(cells))]
        if c[2] < R / 32:
            continue
        todo = {c}
        if mirror:
            todo.add((c[0], -c[1] - c[2], c[2]))
        cells = [x for x in cells if x not in todo] + [y for x in todo if x in cells for y in inputs._split(x)]
    while True:
        bad = None
        for a in cells:
            for b in cells:
                if a[2] <= 2 * b[2]:
                    continue
                ra, za, ha = a
                rb, zb, hb = b
                touch_r = (abs(ra + ha - rb) < 1e-12 or abs(rb + hb - ra) < 1e-12) and zb < za + ha and zb + hb > za
                touch_z = (abs(za + ha - zb) < 1e-12 or abs(zb + hb - za) < 1e-12) and rb < ra + ha and rb + hb > ra
                if touch_r or touch_z:
                    bad = a
                    break
            if bad:
                break
        if bad is None:
            return cells
        todo = {bad}
        if mirror:
            todo.add((bad[0], -bad[1] - bad[2], bad[2]))
        cells = [x for x in cells if x not in todo] + [y for x in todo if x in cells for y in inputs._split(x)]


@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5, 6])
def test_random_meshes_every_inner_path(seed):
    """Random 2:1-balanced quadtrees with hanging nodes (mirror-symmetric for odd seeds, asymmetric for
    even ones), orders p = 2, 3, 4, one or two species: point coefficients of a small batch through the
    inner kernels the mesh admits (per-vertex, mirror-directed, directed) against the oracle, and one
    item's Jacobian."""
    rng = np.random.default_rng(1000 + seed)
    R = inputs.R_E
    mirror = seed % 2 == 1
    cells = _balanced_random_mesh(rng, R, int(rng.integers(3, 9)), mirror)
    order = 2 + seed % 3
    species = [inputs.Species("e", 1.0, -1.0, 0)]
    fmix = [[(1.0, 1.0, 0.2)]]
    if seed > 2:
        species.append(inputs.Species("D", inputs.M_D, 1.0, 0))
        fmix.append([(1.0, 1.0, 0.0)])
    prob = inputs.Problem(f"rand{seed}", order, [(R, cells)], species, fmix=fmix, seed=seed)
    o = Oracle(prob)
    fo = o.coefficients()
    Go, Ga = o.point_coeffs(fo)
    h = L.Landau.from_problem(prob, device=0)
    fg = inputs.coefficients(prob, h.all_nodes())
    nb = 5
    F = torch.tensor(np.stack([fg * (1.0 + 0.05 * k) for k in range(nb)]), device=DEV)
    modes = ["vertex", "slots", True, False] if mirror else [False]
    paths = set()
    for mode in modes:
        if mirror:
            h.set_mirror(mode)
        h.set_state_batched(F)
        G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
        h.point_coeffs_batched(G)
        torch.cuda.synchronize()
        paths.add(h.stats()["inner_path"])
        Gn = G.cpu().numpy()
        for k in (0, nb - 1):
            sc = 1.0 + 0.05 * k
            assert np.max(np.abs(Gn[k] - sc * Go) / (sc * Ga)) <= 1e-12, (mode, k)
    if mirror:
        assert {4, 5} <= paths, paths   # per-vertex and mirror-directed kernels both exercised
    J = gpu_jacobian(h, fg)
    Jo, Ja = o.jacobian(fo)
    assert np.all(np.abs(J - Jo) <= 1e-11 * Ja)


def test_pair_split_partials_sum_with_item_runs(monkeypatch):
    """The pair split on a batch large enough for the slot kernel's i-tile runs on every rank (C4 mesh,
    2048 vertices, slot mode): three emulated ranks' partial G sum to the full G of one handle (the
    same sums in another grouping)."""
    prob = inputs.config4_vertex(0)
    nb = 2048   # each emulated rank still has >= 16 items per resident warp: the run item set
    base = L.Landau.from_problem(prob, device=0)
    nodes = base.all_nodes()
    F1 = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 4)])
    F = torch.tensor(np.concatenate([F1 * (1.0 + 0.01 * k) for k in range(nb // F1.shape[0])]), device=DEV)

    def G_of(env):
        if env:
            monkeypatch.setenv("LANDAU_PAIR_SPLIT_EMULATE", env)
        else:
            monkeypatch.delenv("LANDAU_PAIR_SPLIT_EMULATE", raising=False)
        h = L.Landau.from_problem(prob, device=0)
        h.set_mirror("slots")
        h.set_state_batched(F)
        G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device=DEV)
        h.point_coeffs_batched(G)
        torch.cuda.synchronize()
        assert h.stats()["inner_path"] == 3
        h.close()
        return G.cpu().numpy()

    Gfull = G_of(None)
    Gsum = sum(G_of(f"3:{r}") for r in range(3))
    scale = np.abs(Gfull).max(axis=2, keepdims=True)
    assert np.max(np.abs(Gsum - Gfull) / scale) <= 1e-12


def test_vertex_kernel_smem_limit_survives_smaller_handles():
    """The per-vertex kernel's dynamic shared-memory limit is a per-function attribute shared by all
    handles: creating a handle with a smaller mesh after a larger one must not break the larger
    handle's launches (regression: the bench's Newton sub-line failed after the C1 config line)."""
    big = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
    small = L.Landau.from_problem(inputs.config1(), device=0)   # 10.7 KB vs 91 KB of shared memory
    big.set_mirror("vertex")
    f = inputs.coefficients(inputs.config4_vertex(0), big.all_nodes())
    F = torch.tensor(np.stack([f] * 4), device=DEV)
    big.set_state_batched(F)
    out = torch.empty((4, big.nnz), dtype=torch.float64, device=DEV)
    big.jacobian_batched(out)
    torch.cuda.synchronize()
    assert big.stats()["inner_path"] == 4 and np.all(np.isfinite(out.cpu().numpy()))
    small.close()


_TAIL_CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
fmt, nb, path = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3]
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
h.set_mirror("slots")
nodes = h.all_nodes()
verts = [(k * 1023) // (nb - 1) for k in range(nb)]
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in verts]), device="cuda")
h.set_state_batched(F)
out = torch.full((nb, h.nnz if fmt == 0 else h.ncoo), float("nan"), dtype=torch.float64, device="cuda")
h.set_timing(True)
h.jacobian_batched(out, fmt)
t = h.get_timing()
np.save(path, out.cpu().numpy())
print("stages", t["element"][1], t["assemble"][1])
'''


@pytest.mark.parametrize("fmt", [L.LANDAU_CSR, L.LANDAU_COO])
def test_fused_tail_kernel_equals_two_kernel_path(fmt, tmp_path):
    """Batches of >= 16 small meshes run a-4 + a-5 as one kernel (tail_kernel: each phase's element
    matrices in shared memory, then the gather); LANDAU_TAIL=0 runs element_sf_kernel + assemble_kernel.
    On the same G (slot kernel for a-2, batch-invariant) every value agrees bit for bit (same
    contractions; a slot straddling two phases continues one fma chain in the same order); and the
    tail's values match the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    nb = 20
    res = {}
    for tail in ("1", "0"):
        path = str(tmp_path / f"J{tail}.npy")
        out = subprocess.run([sys.executable, "-c", _TAIL_CHILD, str(fmt), str(nb), path], capture_output=True,
                             text=True, timeout=600, cwd=root, env=dict(os.environ, LANDAU_TAIL=tail))
        assert out.returncode == 0, out.stderr[-3000:]
        res[tail] = (np.load(path), out.stdout.split())
    assert res["1"][1][-2:] == ["1", "0"] and res["0"][1][-2:] == ["1", "1"]   # fused vs element + assemble
    Jt, J2 = res["1"][0], res["0"][0]
    assert np.all(np.isfinite(Jt))
    assert np.array_equal(Jt.view(np.uint64), J2.view(np.uint64))
    verts = [(k * 1023) // (nb - 1) for k in range(nb)]
    o = Oracle(inputs.config4_vertex(verts[7]))
    Jo, Ja = o.jacobian(o.coefficients()) if fmt == L.LANDAU_CSR else o.jacobian_coo(o.coefficients())
    assert np.all(np.abs(Jt[7] - Jo) <= 1e-11 * Ja)


def test_rz_cancellation_stress_uniform_density():
    """The two tensor components whose azimuthal integrands change sign (U^D_rz, U^K_zr) are the only
    ones whose GPU error grows beyond roundoff of G^abs (profiles/r02_parity_analysis.md): with a
    uniform density (f = 1 on every DOF, G_rz a sum of nearly cancelling ring integrals) the C2 G_D,rz
    error reaches ~7e-13 G^abs, still inside the 1e-12 parity bound, while rr, zz and both K
    components stay at roundoff."""
    prob, h, o, fg, fo = setup("C2")
    G = gpu_G(h, np.ones_like(fg))
    Go, Ga = o.point_coeffs(np.ones_like(fo))
    e = np.max(np.abs(G - Go) / Ga, axis=1)
    assert e[1] <= 1e-12, e
    assert e[0] <= 1e-14 and e[2] <= 1e-14 and e[3] <= 1e-14 and e[4] <= 1e-14, e


_BAND_CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
path, nb = sys.argv[1], int(sys.argv[2])
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 1024 // nb)]),
                 device="cuda")
h.set_state_batched(F)
J = torch.empty((nb, h.nnz), dtype=torch.float64, device="cuda")
h.jacobian_batched(J)
Mv = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
h.mass(1.0, Mv)
shift = float(J.abs().max()) / float(Mv.abs().max())
h.band_factor_batched(shift, J)
b = torch.tensor(np.random.default_rng(5).standard_normal((nb, h.ndof)), device="cuda")
x = torch.empty_like(b)
h.band_solve_batched(b, x)
np.savez(path, x=x.cpu().numpy(), b=b.cpu().numpy(), J=J.cpu().numpy(), shift=shift)
'''


def test_band_factorisation_kernels_match():
    """The three band factorisations solve the same C4 systems: the default blocked DMMA kernel
    (band_lu_mma_kernel: 8-column panels, rank-8 trailing updates on the FP64 tensor cores), the
    register-tile rank-2 kernel (LANDAU_BAND_MMA=0) and the opt-in column-warp kernel
    (LANDAU_BAND_CW=1); each agrees with a sparse direct solve of the same A = shift M - J (the
    eliminations round differently), and the Jacobians they factor are identical."""
    import os
    import subprocess
    import sys
    import tempfile
    import scipy.sparse as sps
    import scipy.sparse.linalg as spla
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    variants = {"mma": {}, "rt": {"LANDAU_BAND_MMA": "0"}, "cw": {"LANDAU_BAND_CW": "1"}}
    res = {}
    with tempfile.TemporaryDirectory() as td:
        for name, env in variants.items():
            path = os.path.join(td, f"x_{name}.npz")
            out = subprocess.run([sys.executable, "-c", _BAND_CHILD, path, "4"], capture_output=True, text=True,
                                 timeout=600, cwd=root, env=dict(os.environ, **env))
            assert out.returncode == 0, out.stderr[-3000:]
            res[name] = dict(np.load(path))
    o = Oracle(inputs.config4_vertex(0))
    rp, col = o.pattern()
    M = o.mass(1.0)
    for k in range(4):
        J = res["mma"]["J"][k]
        A = sps.csr_matrix((res["mma"]["shift"] * M - J, col, rp), shape=(o.ndof, o.ndof))
        x_ref = spla.spsolve(A.tocsc(), res["mma"]["b"][k])
        for name in variants:
            assert np.array_equal(J, res[name]["J"][k])
            assert np.max(np.abs(res[name]["x"][k] - x_ref)) <= 1e-10 * np.max(np.abs(x_ref)), name


@pytest.mark.parametrize("ncell,order", [(2, 2), (2, 3), (3, 3)])
def test_jacobian3d_matches_oracle(ncell, order):
    """NEXT-4 completed: the 3D Cartesian Jacobian (landau3d_*: field3d_kernel, inner3d_kernel,
    element3d_kernel, assemble_kernel) equals the oracle's O13 to 1e-11 of its |.| scale on two
    species, conserves density, momentum and energy like the oracle, and repeats bit for bit."""
    from oracle.oracle import Oracle3D
    from tests.test_oracle_3d_jacobian import _moments
    prob = inputs.config3d(ncell, order)
    h = L.Landau3D(prob.ncell, prob.order, prob.R, prob.species, prob.nu, device=0)
    o = Oracle3D(prob.ncell, prob.order, prob.R, prob.species, prob.nu)
    assert (h.ndof, h.npoints, h.nnz) == (o.ndof, o.npoints, o.nnz)
    rp, col = h.pattern()
    orp, ocol = o.pattern()
    assert np.array_equal(rp, orp) and np.array_equal(col, ocol)
    assert np.max(np.abs(h.nodes() - o.nodes())) <= 1e-14 * prob.R
    f = inputs.coefficients3d(prob, h.nodes())
    ft = torch.tensor(f, device=DEV)
    J = torch.full((len(prob.species), h.nnz), float("nan"), dtype=torch.float64, device=DEV)
    h.jacobian(ft, J)
    torch.cuda.synchronize()
    Jg = J.cpu().numpy()
    Jo, Ja = o.jacobian(f)
    assert np.all(np.isfinite(Jg))
    assert np.max(np.abs(Jg - Jo) / Ja) <= 1e-11
    d, mom, en = _moments(o, prob, Jg, Ja, f)
    assert d < 1e-13 and mom < 1e-13 and en < 1e-13, (d, mom, en)
    J2 = torch.empty_like(J)
    h.jacobian(ft, J2)
    torch.cuda.synchronize()
    assert torch.equal(J, J2)
    h.close()


_STEP_CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
path, nb = sys.argv[1], int(sys.argv[2])
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 1024 // nb)]),
                 device="cuda")
Src = torch.tensor(np.stack([inputs.quench_source_shape(inputs.config4_vertex(b), nodes)
                             for b in range(0, 1024, 1024 // nb)]), device="cuda")
Fn = torch.empty_like(F)
h.implicit_step_batched(0.002, F, Fn, Ez=0.1, max_iter=3, src=Src)
state = "ok"
try:   # the fused factorisation stored U only: the public solve must refuse it
    h.band_solve_batched(F, torch.empty_like(F))
    state = "solved"
except Exception as e:
    state = type(e).__name__ + ":" + str(e)[:80]
np.savez(path, f=Fn.cpu().numpy(), state=np.array(state))
'''


def test_implicit_step_fused_forward_elimination():
    """The implicit step's fused factorisation (the DMMA band kernel also eliminates the right-hand side
    forward and stores U alone; the solve runs only the backward pass) gives the same iterates as the
    separate factor + full solve (LANDAU_BAND_FUSED=0), up to rounding; after a fused factorisation the
    public band solve refuses to run (LANDAU_ESTATE), since the L factor was not stored."""
    import os
    import subprocess
    import sys
    import tempfile
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = {}
    with tempfile.TemporaryDirectory() as td:
        for fused in ("1", "0"):
            path = os.path.join(td, f"f{fused}.npz")
            out = subprocess.run([sys.executable, "-c", _STEP_CHILD, path, "8"], capture_output=True, text=True,
                                 timeout=600, cwd=root, env=dict(os.environ, LANDAU_BAND_FUSED=fused))
            assert out.returncode == 0, out.stderr[-3000:]
            res[fused] = dict(np.load(path))
    a, b = res["1"]["f"], res["0"]["f"]
    assert np.max(np.abs(a - b)) <= 1e-11 * np.max(np.abs(b))
    assert "(-5)" in str(res["1"]["state"])   # LANDAU_ESTATE
    assert str(res["0"]["state"]) == "solved"


_C3_STEP_CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
path = sys.argv[1]
p = inputs.CONFIGS["C3"]()
h = L.Landau.from_problem(p, device=0)
f = torch.tensor(np.stack([inputs.coefficients(p, h.all_nodes())] * 3), device="cuda")
fn = torch.empty_like(f)
h.implicit_step_batched(0.01, f, fn, Ez=0.05, max_iter=2)
J = torch.empty((3, h.nnz), dtype=torch.float64, device="cuda")
h.set_state_batched(f)
h.jacobian_batched(J)
h.band_factor_batched(50.0, J)
x = torch.empty_like(f)
h.band_solve_batched(f, x)
np.savez(path, fn=fn.cpu().numpy(), x=x.cpu().numpy())
'''


def test_band_per_species_launches_match():
    """Species blocks on grids of different bandwidth are factored by one DMMA launch per species (each
    with its own window size); forced on a C3 problem (LANDAU_BAND_PER_SPECIES=1: three grids, one
    launch each) it gives the same implicit-step iterates and band solutions as the single launch over
    all blocks, up to rounding."""
    import os
    import subprocess
    import sys
    import tempfile
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = {}
    with tempfile.TemporaryDirectory() as td:
        for ps in ("0", "1"):
            path = os.path.join(td, f"p{ps}.npz")
            out = subprocess.run([sys.executable, "-c", _C3_STEP_CHILD, path], capture_output=True, text=True,
                                 timeout=600, cwd=root, env=dict(os.environ, LANDAU_BAND_PER_SPECIES=ps))
            assert out.returncode == 0, out.stderr[-3000:]
            res[ps] = dict(np.load(path))
    for k in ("fn", "x"):
        a, b = res["1"][k], res["0"][k]
        assert np.max(np.abs(a - b)) <= 1e-12 * np.max(np.abs(b)), k
