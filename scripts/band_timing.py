import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
nb = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
p0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(p0, device=0)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b % 1024), nodes) for b in range(nb)]), device="cuda")
h.set_state_batched(F)
J = torch.empty((nb, h.nnz), dtype=torch.float64, device="cuda")
h.jacobian_batched(J)
M = torch.empty(h.nnz, dtype=torch.float64, device="cuda"); h.mass(1.0, M)
shift = 2.0 * J.abs().max().item() / M.abs().max().item()
b = torch.randn((nb, h.ndof), dtype=torch.float64, device="cuda"); x = torch.empty_like(b)
for _ in range(2):
    h.band_factor_batched(shift, J); h.band_solve_batched(b, x)
torch.cuda.synchronize()
h.set_timing(True)
for _ in range(5):
    h.jacobian_batched(J); h.band_factor_batched(shift, J); h.band_solve_batched(b, x)
t = h.get_timing()
print({k: round(v[0] / 5, 3) for k, v in t.items()}, "B", h.band_info(0)[0])
