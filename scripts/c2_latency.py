import os, sys
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
name = sys.argv[1] if len(sys.argv) > 1 else "C2"
p = inputs.CONFIGS[name]()
h = L.Landau.from_problem(p, device=0)
f = torch.tensor(inputs.coefficients(p, h.all_nodes()), device="cuda")
v = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
if os.environ.get("TC") == "1":
    h.set_tensor_cache(True)
h.set_state(f)
for _ in range(5):
    h.jacobian(v)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(200):
    h.jacobian(v)
b.record(); torch.cuda.synchronize()
print(name, os.environ.get("LANDAU_INNER_VARIANT", "1"), "TC" if os.environ.get("TC") == "1" else "", round(a.elapsed_time(b) / 200 * 1e3, 1), "us per jacobian (graph replay, back to back)")
