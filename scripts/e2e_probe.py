import os, sys, statistics, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
B = 1024
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
base = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 8)])
F = np.concatenate([base] * 8)[:B]
f_pin = torch.tensor(F).pin_memory()
v_pin = torch.empty((B, h.nnz), dtype=torch.float64).pin_memory()
for _ in range(3): h.jacobian_host(f_pin, v_pin)
ts = []
import time
for _ in range(10):
    torch.cuda.synchronize(); t = time.perf_counter(); h.jacobian_host(f_pin, v_pin); ts.append(time.perf_counter() - t)
print("chunks", os.environ.get("LANDAU_HOST_CHUNKS", "16 (default)"), "e2e ms %.3f" % (1e3 * statistics.median(ts)), "builds/s %.3e" % (B / statistics.median(ts)))
