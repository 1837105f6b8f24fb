"""Which side is off at C2's worst point-coefficient errors?  GPU G, oracle G, and an independent
reference at the worst target points: Eq. 3 integrated numerically over the azimuth for every source
(tests/_brute.tensors_quadrature, graded Gauss panels, no elliptic integrals), summed with math.fsum;
the 8 nearest sources additionally by 30-digit mpmath quadrature."""
import math
import json, os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import mpmath as mp
from oracle.oracle import Oracle
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
from tests._brute import tensor_mpmath, tensors_quadrature
prob = inputs.config2()
h = L.Landau.from_problem(prob, device=0)
o = Oracle(prob)
fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
h.set_state(torch.tensor(fg, device="cuda"))
G = torch.empty((5, h.npoints), dtype=torch.float64, device="cuda")
h.point_coeffs(G)
G = G.cpu().numpy()
Go, Ga = o.point_coeffs(fo)
err = np.abs(G - Go) / Ga
order = np.argsort(err.max(axis=0))[::-1][:3]
r, z, w = o.points()
TD, TKr, TKz = o.point_fields(fo)
out = []
for i in order:
    c = int(np.argmax(err[:, i]))
    js = np.array([j for j in range(r.size) if not (r[j] == r[i] and z[j] == z[i])])
    U = tensors_quadrature(np.full(js.size, r[i]), np.full(js.size, z[i]), r[js], z[js])
    near = js[np.argsort((r[js] - r[i]) ** 2 + (z[js] - z[i]) ** 2)[:8]]
    for jn in near:
        k = int(np.nonzero(js == jn)[0][0])
        U[:, k] = tensor_mpmath(r[i], z[i], r[jn], z[jn], dps=30)
    wd, wkr, wkz = w[js] * TD[js], w[js] * TKr[js], w[js] * TKz[js]
    vals = [wd * U[0], wd * U[1], wd * U[2], U[3] * wkr + U[1] * wkz, U[4] * wkr + U[2] * wkz]
    acc = [math.fsum(v) for v in vals]
    ref = np.array(acc)
    out.append({"point": int(i), "r": float(r[i]), "z": float(z[i]), "component": c,
                "gpu_minus_oracle_over_Gabs": float((G[c, i] - Go[c, i]) / Ga[c, i]),
                "gpu_minus_ref_over_Gabs": float((G[c, i] - ref[c]) / Ga[c, i]),
                "oracle_minus_ref_over_Gabs": float((Go[c, i] - ref[c]) / Ga[c, i])})
    print(out[-1], flush=True)
json.dump(out, open("gpurun_out/c2_worst_point.json", "w"), indent=1)
