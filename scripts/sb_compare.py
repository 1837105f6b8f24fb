"""C2 Jacobian (CSR) and G of the current library configuration, saved to gpurun_out/<tag>.npz."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_adamsbkw22_b200 import inputs, landau as L
prob = inputs.config2()
h = L.Landau.from_problem(prob, device=0)
f = torch.tensor(inputs.coefficients(prob, h.all_nodes()), device="cuda:0")
h.set_state(f)
J = torch.empty(h.nnz, dtype=torch.float64, device="cuda:0")
h.jacobian(J)
G = torch.empty((5, h.npoints), dtype=torch.float64, device="cuda:0")
h.point_coeffs(G)
torch.cuda.synchronize()
np.savez(f"gpurun_out/{sys.argv[1]}.npz", J=J.cpu().numpy(), G=G.cpu().numpy(), path=h.stats()["inner_path"])
