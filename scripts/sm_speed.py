"""Per-SM speed of the per-vertex kernel (LANDAU_VTX_TRACE build, build_variants/liblandau_trace.so):
each CTA's rounds phases (tags 2 -> 3) timed with %globaltimer and keyed by %smid; two launches in
each of two processes, to see whether the speed is a property of the SM.
Usage: python scripts/sm_speed.py [B]"""
import os, sys, subprocess
import numpy as np
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
if os.environ.get("SM_SPEED_DATA") == "zero": F.zero_()
if os.environ.get("SM_SPEED_DATA") == "same": F[:] = F[0]
if os.environ.get("SM_SPEED_DATA") == "reverse": F = F.flip(0).contiguous()
G = torch.empty((B, 5, h.npoints), dtype=torch.float64, device="cuda")
h.set_state_batched(F)
h.point_coeffs_batched(G); torch.cuda.synchronize()
for _ in range(2):
    print("=====", flush=True)
    h.point_coeffs_batched(G); torch.cuda.synchronize()
'''
B = sys.argv[1] if len(sys.argv) > 1 else "1024"
runs = []
for proc in range(2):
    r = subprocess.run([sys.executable, "-c", CHILD, B], capture_output=True, text=True,
                       env=dict(os.environ,
                                LANDAU_LIB=os.path.abspath("build_variants/liblandau_trace.so")))
    out = r.stdout
    calib = {}
    for l in r.stderr.splitlines():
        p = l.split()
        if len(p) == 5 and p[0] == "CALIB":
            calib[int(p[1])] = [int(x) / 1e3 for x in p[2:]]
    if calib:
        print("process %d calibration (us per CTA, 3 launches): min %.1f max %.1f" % (proc, min(min(v) for v in calib.values()), max(max(v) for v in calib.values())))
    for chunk in out.split("=====")[1:]:
        ev, sm = {}, {}
        for l in chunk.strip().splitlines():
            p = l.split()
            if len(p) == 6 and p[0] == "VTX":
                ev.setdefault(int(p[1]), []).append((int(p[2]), int(p[3]), int(p[4])))
                sm[int(p[1])] = int(p[5])
        if not ev:
            continue
        t0 = min(min(t for _, _, t in v) for v in ev.values())
        per_sm = {}
        for c, v in ev.items():
            v.sort()
            busy, last2 = 0.0, None
            for _, tag, t in v:
                if tag == 2:
                    last2 = t
                if tag == 3 and last2 is not None:
                    busy += (t - last2) / 1e3
                    last2 = None
            per_sm[sm[c]] = (busy, (v[-1][2] - t0) / 1e3, c)
        runs.append(per_sm)
sms = sorted(set.intersection(*[set(r) for r in runs]))
busy = np.array([[r[s][0] for s in sms] for r in runs])
ends = np.array([[r[s][1] for s in sms] for r in runs])
print("B", B, "CTAs", len(sms), "launches", len(runs))
for k in range(len(runs)):
    print("launch %d: rounds-busy per CTA us min %.1f median %.1f max %.1f | end us min %.1f mean %.1f max %.1f"
          % (k, busy[k].min(), np.median(busy[k]), busy[k].max(), ends[k].min(), ends[k].mean(), ends[k].max()))
for a in range(1, len(runs)):
    print("corr(busy launch0, launch%d) = %.3f" % (a, np.corrcoef(busy[0], busy[a])[0, 1]))
order = np.argsort(busy.mean(0))
print("fastest smid", [sms[i] for i in order[:8]], "slowest", [sms[i] for i in order[-8:]])
print("busy by smid (mean of launches):", " ".join("%d:%.0f" % (sms[i], busy[:, i].mean()) for i in range(len(sms))))
if calib:
    cal = np.array([np.median(calib[runs[0][s][2]]) for s in sms])
    print("corr(calibration time, production busy) by CTA = %.3f" % np.corrcoef(cal, busy.mean(0))[0, 1])
    print("calib/busy ratio min %.4f max %.4f" % ((cal / busy.mean(0)).min(), (cal / busy.mean(0)).max()))
print("CTA of smid per launch:", [[runs[k][s][2] for s in sms[:12]] for k in range(len(runs))])
Wv = int(os.environ.get("SM_SPEED_WV", "37"))
Bn = int(B)
S = len(sms)
byc = {runs[0][s][2]: busy[:, i].mean() for i, s in enumerate(sms)}
print("per CTA (c: busy us, first-weight offset in its vertex, weights):")
print(" ".join("%d:%.0f/%d" % (c, byc[c], ((c * Bn * Wv + S - 1) // S) % Wv) for c in sorted(byc)))
