"""C2 point-coefficient error (vs the oracle, relative to G^abs) of every inner-kernel path, at the worst
point and overall: which formulation carries the 8e-14 of the mirror kernels?"""
import os, sys, subprocess
CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
mode = sys.argv[1]
prob = inputs.config2()
h = L.Landau.from_problem(prob, device=0)
o = Oracle(prob)
fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
nb = 16 if mode in ("vertex", "slots", "sym") else 1
if mode == "sym": h.set_mirror(False)
elif mode in ("vertex", "slots"): h.set_mirror(mode)
F = torch.tensor(np.stack([fg] * nb), device="cuda")
h.set_state_batched(F)
G = torch.empty((nb, 5, h.npoints), dtype=torch.float64, device="cuda")
h.point_coeffs_batched(G)
G = G[0].cpu().numpy()
Go, Ga = o.point_coeffs(fo)
e = np.abs(G - Go) / Ga
i = int(np.argmax(e.max(axis=0)))
print(mode, "path", h.stats()["inner_path"], "max %.2e" % e.max(), "at point", i, "comp", int(np.argmax(e[:, i])), "per-comp max", ["%.1e" % v for v in e.max(axis=1)], "point659", ["%.1e" % v for v in e[:, 659]])
'''
for mode, env in (("single", {}), ("vertex", {}), ("slots", {}), ("sym", {}), ("directed", {"LANDAU_MIRROR": "0", "LANDAU_SYM": "0"})):
    out = subprocess.run([sys.executable, "-c", CHILD, mode], capture_output=True, text=True, env=dict(os.environ, **env))
    print(out.stdout.strip() or out.stderr[-800:], flush=True)
