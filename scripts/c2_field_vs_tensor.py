"""Is C2's 8e-14 (G_D components, all inner kernels) from the point fields or the device tensor math?
G error vs the oracle for (a) the C2 state, (b) f = 1 on every DOF (T_D constant), (c) a single hot
Maxwellian, (d) the C2 state's e and D species separately."""
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
prob = inputs.config2()
h = L.Landau.from_problem(prob, device=0)
o = Oracle(prob)
def err(fg, fo, name):
    h.set_state(torch.tensor(fg, device="cuda"))
    G = torch.empty((5, h.npoints), dtype=torch.float64, device="cuda")
    h.point_coeffs(G)
    G = G.cpu().numpy()
    Go, Ga = o.point_coeffs(fo)
    e = np.abs(G - Go) / Ga
    print(name, "per-comp max", ["%.1e" % v for v in e.max(axis=1)], "worst point", int(np.argmax(e.max(axis=0))), flush=True)
fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
err(fg, fo, "C2 state      ")
err(np.ones_like(fg), np.ones_like(fo), "f = 1         ")
hot = inputs.Problem("hot", 3, prob.grids, prob.species, fmix=[[(1.0, 1.0, 0.0)], [(1.0, 1.0, 0.0)]], seed=1, noise=0.0)
err(inputs.coefficients(hot, h.all_nodes()), inputs.coefficients(hot, o.all_nodes()), "hot Maxwellian")
n = h.grid_ndof(0)
for a, name in ((0, "C2 e only     "), (1, "C2 D only     ")):
    g2, o2 = fg.copy(), fo.copy()
    g2[(1 - a) * n:(2 - a) * n] = 0.0
    o2[(1 - a) * n:(2 - a) * n] = 0.0
    err(g2, o2, name)
