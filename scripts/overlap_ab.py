"""A/B of a library knob (env var ENVVAR, default LANDAU_OVERLAP = K chunks): per-step time of the whole Jacobian
build (graph replay, median of per-step CUDA events, L2 flushed between steps) and the CSR values'
largest difference from the K = 1 build, relative to max |J|.  Each K runs in its own process (the
knob is read once).  Usage: python scripts/overlap_ab.py [B] K1 K2 ...   (first K is the reference)"""
import os, subprocess, sys
CHILD = r'''
import os, sys, statistics, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
B = int(sys.argv[2])
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
base = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 8)])
F = torch.tensor(np.concatenate([base] * (B // 128 + 1))[:B], device="cuda")
J = torch.empty((B, h.nnz), dtype=torch.float64, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
h.set_state_batched(F)
for _ in range(5): h.jacobian_batched(J)
torch.cuda.synchronize()
ts = []
for _ in range(int(os.environ.get("STEPS", "30"))):
    flush.zero_()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); h.jacobian_batched(J); b.record(); torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
np.save(sys.argv[1], J.cpu().numpy())
print("ms %.4f min %.4f launches %d" % (statistics.median(ts), min(ts), h.launch_count()))
'''
B = sys.argv[1]
ref = None
import numpy as np
for rep in range(int(os.environ.get("REPS", "2"))):
    for K in sys.argv[2:]:
        out = "/tmp/J_%d.npy" % sys.argv[2:].index(K)
        r = subprocess.run([sys.executable, "-c", CHILD, out, B], capture_output=True, text=True,
                           env=dict(os.environ, **{os.environ.get("ENVVAR", "LANDAU_OVERLAP"): K}))
        msg = r.stdout.strip() or r.stderr[-800:]
        if r.returncode == 0:
            Jv = np.load(out)
            if ref is None:
                ref = Jv
            msg += f" maxdiff/max|J| {np.max(np.abs(Jv - ref)) / np.abs(ref).max():.2e}" \
                   f" bitwise {np.array_equal(Jv.view(np.uint64), ref.view(np.uint64))}"
        print(f"B{B} K={K}", msg, flush=True)
