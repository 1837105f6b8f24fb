#!/usr/bin/env python3
"""GPU-vs-oracle parity margins (the numbers behind tests/test_gpu_parity.py), as one JSON document.

For C1-C3 (full oracle), a C4 batch on the symmetric kernel (sampled vertices) and C5 (sampled
cells): max |G_gpu - G_ora| / G^abs, max |J_gpu - J_ora| / J^abs, max |dJ| / max |J|, and the
conservation residuals of the GPU Jacobian.  Runs on cuda:0; uses the oracle (test infrastructure).
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle.oracle import Oracle  # noqa: E402
from paper_conf_ipps_adamsbkw22_b200 import inputs  # noqa: E402
from paper_conf_ipps_adamsbkw22_b200 import landau as L  # noqa: E402
from tests.test_gpu_parity import _conservation  # noqa: E402

DEV = "cuda:0"


def run(h, f, fmt=L.LANDAU_CSR, G=False):
    h.set_state(torch.tensor(f, device=DEV))
    if G:
        out = torch.empty((5, h.npoints), dtype=torch.float64, device=DEV)
        h.point_coeffs(out)
    else:
        out = torch.empty(h.nnz if fmt == L.LANDAU_CSR else h.ncoo, dtype=torch.float64, device=DEV)
        h.jacobian(out, fmt)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def main():
    rep = {}
    for cfg in ("C1", "C2", "C3"):
        prob = inputs.CONFIGS[cfg]()
        h = L.Landau.from_problem(prob, device=0)
        o = Oracle(prob)
        fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
        G = run(h, fg, G=True)
        Go, Ga = o.point_coeffs(fo)
        J = run(h, fg)
        Jo, Ja = o.jacobian(fo)
        d, m, e = _conservation(prob, h, J, fg)
        eg = np.abs(G - Go) / Ga
        worst = np.unravel_index(int(np.argmax(eg)), eg.shape)
        r, z, _ = h.points()
        rep[cfg] = {"G_err_over_Gabs": float(eg.max()),
                    "G_worst_point": {"component": int(worst[0]), "r": float(r[worst[1]]), "z": float(z[worst[1]]),
                                      "r_over_R": float(r[worst[1]] / prob.grids[0][0])},
                    "J_err_over_Jabs": float(np.max(np.abs(J - Jo) / Ja)),
                    "J_maxerr_over_maxJ": float(np.abs(J - Jo).max() / np.abs(Jo).max()),
                    "conservation": {"density": d, "momentum": m, "energy": e},
                    "kernel": ["directed", "symmetric", "tensor cache", "mirror slot", "per-vertex",
                               "mirror-directed (single build: one cooperative kernel)"][h.stats()["inner_path"]]}
    # C4 batch on the mirror slot kernel and on the per-vertex kernel (the headline path)
    for mode, key in (("slots", "C4_batch64_mirror_slots"), ("vertex", "C4_batch64_vertex")):
        nb = 64
        prob0 = inputs.config4_vertex(0)
        h = L.Landau.from_problem(prob0, device=0)
        h.set_mirror(mode)
        nodes = h.all_nodes()
        verts = [int(round(k * 1023 / (nb - 1))) for k in range(nb)]
        probs = [inputs.config4_vertex(b) for b in verts]
        F = torch.tensor(np.stack([inputs.coefficients(p, nodes) for p in probs]), device=DEV)
        h.set_state_batched(F)
        out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
        h.jacobian_batched(out)
        Jb = out.cpu().numpy()
        worst = {"J_err_over_Jabs": 0.0, "J_maxerr_over_maxJ": 0.0, "conservation_max": 0.0,
                 "inner_path": h.stats()["inner_path"]}
        for k in (0, 21, 42, 63):
            o = Oracle(probs[k])
            Jo, Ja = o.jacobian(o.coefficients())
            worst["J_err_over_Jabs"] = max(worst["J_err_over_Jabs"], float(np.max(np.abs(Jb[k] - Jo) / Ja)))
            worst["J_maxerr_over_maxJ"] = max(worst["J_maxerr_over_maxJ"], float(np.abs(Jb[k] - Jo).max() / np.abs(Jo).max()))
            worst["conservation_max"] = max(worst["conservation_max"],
                                            max(_conservation(probs[k], h, Jb[k], inputs.coefficients(probs[k], nodes))))
        rep[key] = dict(worst, vertices_checked=[verts[k] for k in (0, 21, 42, 63)])
    # the headline batch: 1024 vertices in automatic mode (per-vertex kernel, stream-K)
    nb = 1024
    prob0 = inputs.config4_vertex(0, nb)
    h = L.Landau.from_problem(prob0, device=0)
    nodes = h.all_nodes()
    F = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b, nb), nodes) for b in range(nb)]), device=DEV)
    h.set_state_batched(F)
    out = torch.empty((nb, h.nnz), dtype=torch.float64, device=DEV)
    h.jacobian_batched(out)
    Jb = out.cpu().numpy()
    split = set(int(x) for x in h.vtx_split_vertices(nb))
    sample = [0, 148, 500, 1023] + sorted(split)[:2]
    worst = {"J_err_over_Jabs": 0.0, "conservation_max": 0.0, "inner_path": h.stats()["inner_path"]}
    for b in sample:
        o = Oracle(inputs.config4_vertex(b, nb))
        Jo, Ja = o.jacobian(o.coefficients())
        worst["J_err_over_Jabs"] = max(worst["J_err_over_Jabs"], float(np.max(np.abs(Jb[b] - Jo) / Ja)))
        worst["conservation_max"] = max(worst["conservation_max"],
                                        max(_conservation(inputs.config4_vertex(b, nb), h, Jb[b],
                                                          inputs.coefficients(inputs.config4_vertex(b, nb), nodes))))
    rep["C4_headline_1024"] = dict(worst, vertices_checked=sample, vertices_split_between_ctas=len(split))
    # C5 sampled cells
    prob = inputs.config5()
    h = L.Landau.from_problem(prob, device=0)
    o = Oracle(prob)
    fg, fo = inputs.coefficients(prob, h.all_nodes()), o.coefficients()
    rng = np.random.default_rng(2022)
    ncell = len(prob.grids[0][1])
    cells = np.sort(rng.choice(ncell, 32, replace=False))
    nqp = (prob.order + 1) ** 2
    targets = (cells[:, None] * nqp + np.arange(nqp)[None, :]).ravel()
    G = run(h, fg, G=True)
    Go, Ga = o.point_coeffs(fo, targets)
    Jc = run(h, fg, L.LANDAU_COO)
    mask = np.zeros(ncell, dtype=np.uint8)
    mask[cells] = 1
    Jo, Ja = o.jacobian_coo(fo, mask)
    sel = np.isfinite(Jo)
    rep["C5_sampled"] = {"cells": cells.tolist(), "G_err_over_Gabs": float(np.max(np.abs(G[:, targets] - Go) / Ga)),
                         "J_err_over_Jabs": float(np.max(np.abs(Jc[sel] - Jo[sel]) / Ja[sel]))}
    rep["tolerances"] = {"G": 1e-12, "J": 1e-11, "conservation": 1e-13}
    print(json.dumps(rep, indent=1))


if __name__ == "__main__":
    main()
