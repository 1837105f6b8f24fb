import os, sys, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
prob0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(prob0, device=0)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(1024)]), device="cuda")
vals = torch.empty((1024, h.nnz), dtype=torch.float64, device="cuda")
flush = torch.empty(256 * 1024 * 1024 // 8, dtype=torch.float64, device="cuda")
h.set_state_batched(F)
tc = len(sys.argv) > 1 and sys.argv[1] == "tc"
if tc:
    h.set_tensor_cache(True)
for _ in range(3):
    h.jacobian_batched(vals)
torch.cuda.synchronize()
tot = 0.0
for k in range(20):
    flush.fill_(k)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); h.jacobian_batched(vals); b.record(); torch.cuda.synchronize()
    tot += a.elapsed_time(b)
print(os.environ.get("LANDAU_CHUNK_MB", "0"), "tc" if tc else "pair", round(tot / 20, 4), "ms per build of 1024")
