"""Single-build latency of C1/C2/C3: graph-replayed step time and the per-stage breakdown (timers force
direct launches, so the stage sum exceeds the graph time by the launch gaps)."""
import sys, os, statistics
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
for name in ("C1", "C2", "C3"):
    p = inputs.CONFIGS[name]()
    h = L.Landau.from_problem(p, device=0)
    f = torch.tensor(inputs.coefficients(p, h.all_nodes()), device="cuda")
    v = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    m = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    def step(full=True):
        h.set_state(f); h.jacobian(v)
        if full: h.mass(1e3, m)
    for full in (True, False):
        for _ in range(5): step(full)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(50)]
        for a, b in ev:
            a.record(); step(full); b.record()
        torch.cuda.synchronize()
        print(name, "graph step" if full else "graph set_state+jacobian", "%.1f us" % (1e3 * statistics.median(a.elapsed_time(b) for a, b in ev)))
    h.set_timing(True)
    for _ in range(20): step()
    t = h.get_timing()
    print(name, {k: round(1e3 * v[0] / 20, 2) for k, v in t.items() if v[0]}, "path", h.stats()["inner_path"], "nsplit", h.stats()["nsplit"])
