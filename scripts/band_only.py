"""C4 batch (1024 vertices, 2048 band matrices): Jacobian, then the band factorisation timed with CUDA
events on the library stream (median of 5), for ncu and for quick kernel comparisons."""
import statistics
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_adamsbkw22_b200 import inputs, landau as L
nb = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
prob0 = inputs.config4_vertex(0, nb)
s = torch.cuda.Stream()
h = L.Landau.from_problem(prob0, device=0, stream=s)
nodes = h.all_nodes()
F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b, nb), nodes) for b in range(nb)]), device="cuda")
with torch.cuda.stream(s):
    h.set_state_batched(F)
    J = torch.empty((nb, h.nnz), dtype=torch.float64, device="cuda")
    h.jacobian_batched(J)
    ts = []
    for it in range(6):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        h.band_factor_batched(500.0, J)
        e1.record(s)
        s.synchronize()
        ts.append(e0.elapsed_time(e1))
print("band factor ms (median of 5 after 1):", statistics.median(ts[1:]), ts)
