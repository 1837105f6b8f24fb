# small workloads for compute-sanitizer: every kernel of the library on C1, C3 and a 16-vertex C4 batch
# (symmetric, mirror-slot, per-vertex and mirror-directed inner kernels; band LU, solve and the implicit
# step with and without the quench source; the 3D Cartesian inner integral; one emulated rank of the pair
# split), the fused single-build kernel (C1, C3 without timers), the element/assembly kernels (timed
# builds), a 200-vertex batch (more vertices than SMs: the per-vertex kernel loops over several
# vertices per CTA and splits some between CTAs) and a 640-vertex one (the headline's canonical-order
# variant), the pipelined host entry point, the 3D Cartesian Jacobian.  Argument "tail":
# LANDAU_TAIL=1 (the fused tail kernel); "bandcw": LANDAU_BAND_CW=1 (the column-warp band factorisation).
import os, sys
if len(sys.argv) > 1 and sys.argv[1] == "tail":
    os.environ["LANDAU_TAIL"] = "1"
if len(sys.argv) > 1 and sys.argv[1] == "bandcw":   # the opt-in column-warp band factorisation
    os.environ["LANDAU_BAND_CW"] = "1"
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
for name in ("C1", "C3"):
    p = inputs.CONFIGS[name]()
    h = L.Landau.from_problem(p, device=0)
    f = torch.tensor(inputs.coefficients(p, h.all_nodes()), device="cuda")
    h.set_state(f)
    for fmt, n in ((L.LANDAU_CSR, h.nnz), (L.LANDAU_COO, h.ncoo)):
        v = torch.empty(n, dtype=torch.float64, device="cuda")
        h.jacobian(v, fmt)
        h.mass(2.0, v, fmt)
    G = torch.empty((5, h.npoints), dtype=torch.float64, device="cuda")
    h.point_coeffs(G)
    h.set_timing(True)   # the multi-kernel single build (field, mdir, reduce, element, assemble)
    v = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    h.jacobian(v)
    h.set_timing(False)
p0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(p0, device=0)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(16)]), device="cuda")
os.environ["LANDAU_SYM_MIN_ITEMS_PER_SM"] = "0"
h.set_state_batched(F)
v = torch.empty((16, h.nnz), dtype=torch.float64, device="cuda")
h.jacobian_batched(v)
print("stats", h.stats())
fh = F.cpu().pin_memory(); vh = torch.empty((16, h.nnz), dtype=torch.float64).pin_memory()
h.jacobian_host(fh, vh)
for mode in ("slots", "vertex"):   # mirror slot kernel + reduction; per-vertex kernel
    h.set_mirror(mode)
    h.set_state_batched(F)   # the host entry left its own (chunked) state behind
    h.jacobian_batched(v)
    print("stats", mode, h.stats())
M = torch.empty(h.nnz, dtype=torch.float64, device="cuda"); h.mass(1.0, M)   # band LU, solve, implicit step
shift = 2.0 * v.abs().max().item() / M.abs().max().item()
h.band_factor_batched(shift, v)
b = torch.randn((16, h.ndof), dtype=torch.float64, device="cuda"); x = torch.empty_like(b)
h.band_solve_batched(b, x)
fn = torch.empty_like(F)
h.implicit_step_batched(0.002, F, fn, Ez=0.1, max_iter=2)
src = torch.tensor(np.stack([inputs.quench_source_shape(inputs.config4_vertex(b), nodes) for b in range(16)]), device="cuda")
h.implicit_step_batched(0.002, F, fn, Ez=0.1, max_iter=2, src=src)
torch.cuda.synchronize()
print("ok")
# more vertices than SMs: several vertices per CTA, some split between CTAs (automatic mode)
h.set_mirror(True)
nb = 200
F2 = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(nb)]), device="cuda")
h.set_state_batched(F2)
v2 = torch.empty((nb, h.nnz), dtype=torch.float64, device="cuda")
h.jacobian_batched(v2)
torch.cuda.synchronize()
print("stats 200", h.stats(), "split", len(h.vtx_split_vertices(nb)))
# the headline's variant: >= 4 vertices per CTA (canonical round order, several whole vertices per CTA)
nb = 640
F4 = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b % 200), nodes) for b in range(nb)]), device="cuda")
h.set_state_batched(F4)
v4 = torch.empty((nb, h.nnz), dtype=torch.float64, device="cuda")
h.jacobian_batched(v4)
torch.cuda.synchronize()
print("stats 640", h.stats(), "split", len(h.vtx_split_vertices(nb)))
# the end-to-end entry point: pipelined chunks (H2D, build, D2H on three streams)
fh = F4[:256].cpu().pin_memory()
vh = torch.empty((256, h.nnz), dtype=torch.float64).pin_memory()
h.jacobian_host(fh, vh)
print("ok host chunks")
# NEXT-4: the 3D Cartesian inner integral (split-j and direct)
xyz3, w3 = inputs.points3d(2, 2)
wTD3, wTK3 = inputs.fields3d(xyz3, w3)
G3 = torch.empty((9, w3.size), dtype=torch.float64, device="cuda")
L.landau3d_inner(torch.tensor(xyz3, device="cuda"), torch.tensor(wTD3, device="cuda"), torch.tensor(wTK3, device="cuda"), G3)
# pair split (one emulated rank of two) on C3 through the slot kernel
os.environ["LANDAU_PAIR_SPLIT_EMULATE"] = "2:1"
p3 = inputs.CONFIGS["C3"]()
h3 = L.Landau.from_problem(p3, device=0)
h3.set_mirror("slots")
f3 = torch.tensor(np.stack([inputs.coefficients(p3, h3.all_nodes())] * 4), device="cuda")
h3.set_state_batched(f3)
Gp = torch.empty((4, 5, h3.npoints), dtype=torch.float64, device="cuda")
h3.point_coeffs_batched(Gp)
torch.cuda.synchronize()
print("ok 3d + pair split")
# NEXT-4 completed: the whole 3D Jacobian (field3d, inner3d, element3d, assembly), Q2 and Q3
for nc, order in ((2, 2), (2, 3)):
    p3d = inputs.config3d(nc, order)
    h3d = L.Landau3D(p3d.ncell, p3d.order, p3d.R, p3d.species, p3d.nu, device=0)
    F3d = torch.tensor(inputs.coefficients3d(p3d, h3d.nodes()), device="cuda")
    J3d = torch.empty((len(p3d.species), h3d.nnz), dtype=torch.float64, device="cuda")
    h3d.jacobian(F3d, J3d)
    torch.cuda.synchronize()
    h3d.close()
print("ok 3d jacobian")
