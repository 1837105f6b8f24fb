"""Inner-kernel time of the per-vertex kernel vs batch size and mode (stream-K overhead study)."""
import sys, os, statistics
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
p0 = inputs.config4_vertex(0)
h = L.Landau.from_problem(p0, device=0)
nodes = h.all_nodes()
base = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 8)])
for mode, B in [("auto", 1024), ("auto", 296), ("auto", 148), ("vertex", 148), ("auto", 128), ("vertex", 128), ("vertex", 1), ("vertex", 8), ("auto", 64)]:
    h.set_mirror(True if mode == "auto" else mode)
    F = torch.tensor(np.concatenate([base] * (B // 128 + 1))[:B], device="cuda")
    G = torch.empty((B, 5, h.npoints), dtype=torch.float64, device="cuda")
    h.set_state_batched(F)
    for _ in range(3):
        h.point_coeffs_batched(G)
    h.set_timing(True)
    for _ in range(10):
        h.point_coeffs_batched(G)
    t = h.get_timing()
    h.set_timing(False)
    print(mode, B, h.stats()["inner_path"], "inner ms %.4f" % (t["inner"][0] / t["inner"][1]), flush=True)
