"""One per-vertex-kernel launch with the LANDAU_VTX_TRACE build: per-CTA timeline summary."""
import os, sys, subprocess
CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
B = int(sys.argv[1])
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
base = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 8)])
F = torch.tensor(np.concatenate([base] * (B // 128 + 1))[:B], device="cuda")
G = torch.empty((B, 5, h.npoints), dtype=torch.float64, device="cuda")
h.set_state_batched(F)
h.point_coeffs_batched(G); torch.cuda.synchronize()
print("=====", flush=True)
h.point_coeffs_batched(G); torch.cuda.synchronize()
'''
B = sys.argv[1] if len(sys.argv) > 1 else "128"
out = subprocess.run([sys.executable, "-c", CHILD, B], capture_output=True, text=True,
                     env=dict(os.environ, LANDAU_LIB=os.path.abspath("build_variants/liblandau_trace.so"))).stdout
lines = out.split("=====")[-1].strip().splitlines()
ev_of = {}
smid_of = {}
for l in lines:
    p = l.split()
    if len(p) != 6 or p[0] != "VTX":
        continue
    ev_of.setdefault(int(p[1]), []).append((int(p[2]), int(p[3]), int(p[4])))
    smid_of[int(p[1])] = int(p[5])
recs = [(c, [(tag, t) for _, tag, t in sorted(v)]) for c, v in ev_of.items()]
t0 = min(ev[0][1] for _, ev in recs)
ends = sorted((ev[-1][1] - t0) / 1e3 for _, ev in recs)
starts = sorted((ev[0][1] - t0) / 1e3 for _, ev in recs)
print("B", B, "ctas", len(recs), "start spread us: %.2f..%.2f" % (starts[0], starts[-1]), "end us: min %.1f median %.1f max %.1f" % (ends[0], ends[len(ends)//2], ends[-1]))
# per-CTA phase durations
import statistics
pro, stage, rounds, wr, comb = [], [], [], [], []
for c, ev in recs:
    d = dict()
    for i in range(1, len(ev)):
        tag, t = ev[i]; ptag, pt = ev[i-1]
        d.setdefault((ptag, tag), []).append((t - pt) / 1e3)
    pro += d.get((0, 1), [])
    stage += d.get((1, 2), []) + d.get((4, 2), [])
    rounds += d.get((2, 3), [])
    wr += d.get((3, 4), []) + d.get((3, 5), [])
    comb += d.get((5, 4), [])
for name, v in (("prologue", pro), ("stage", stage), ("rounds", rounds), ("write/partial(+combine)", wr), ("after combine", comb)):
    if v:
        print("%-26s n %4d  mean %7.2f  max %7.2f us" % (name, len(v), statistics.mean(v), max(v)))
worst = max(recs, key=lambda r: r[1][-1][1])
print("slowest CTA", worst[0], [(t, round((x - t0) / 1e3, 1)) for t, x in worst[1]])

# per-SM speed: mean duration of whole-vertex round blocks (the segments with all rounds) per SM
full = {}
for c, ev in recs:
    for i in range(1, len(ev)):
        if ev[i - 1][0] == 2 and ev[i][0] == 3:
            full.setdefault(smid_of[c], []).append((ev[i][1] - ev[i - 1][1]) / 1e3)
rows = sorted((statistics.mean(v), sm, len(v)) for sm, v in full.items())
print("segment-rounds time by SM (mean us, smid, n): fastest", rows[:6], "slowest", rows[-6:])
by_half = {}
for m, sm, n in rows:
    by_half.setdefault(sm // 74, []).append(m)
print({k: round(statistics.mean(v), 1) for k, v in by_half.items()})
