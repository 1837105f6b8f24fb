import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
p0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(p0, device=0)
nodes = h.all_nodes()
for nb in (8, 64, 148, 1024):
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(nb)]), device="cuda")
    Fn = torch.empty_like(F)
    try:
        print(nb, h.implicit_step_batched(0.002, F, Fn, max_iter=2, rtol=0.0), h.stats()["inner_path"], flush=True)
    except Exception as e:
        print(nb, "ERR", e, flush=True)
        h = L.Landau.from_problem(p0, device=0)
