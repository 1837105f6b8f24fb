"""Inner-kernel time of library build variants (LANDAU_LIB) on the C4 batch; G must equal the default
build's bit for bit when the variant only reschedules (e.g. LANDAU_VTX_PIPE).  Usage:
python scripts/vtx_variants.py lib1.so [lib2.so ...]  (each in a child process)"""
import os, subprocess, sys
CHILD = r'''
import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L
B = int(os.environ.get("VB", "1024"))
h = L.Landau.from_problem(inputs.config4_vertex(0), device=0)
nodes = h.all_nodes()
base = np.stack([inputs.coefficients(inputs.config4_vertex(b), nodes) for b in range(0, 1024, 8)])
F = torch.tensor(np.concatenate([base] * (B // 128 + 1))[:B], device="cuda")
G = torch.empty((B, 5, h.npoints), dtype=torch.float64, device="cuda")
h.set_state_batched(F)
for _ in range(3): h.point_coeffs_batched(G)
h.set_timing(True)
for _ in range(10): h.point_coeffs_batched(G)
t = h.get_timing()
np.save(sys.argv[1], G.cpu().numpy())
print("inner_ms %.4f path %d" % (t["inner"][0] / t["inner"][1], h.stats()["inner_path"]))
'''
ref = None
for i, lib in enumerate(sys.argv[1:]):
    out = f"/tmp/G_{i}.npy"
    r = subprocess.run([sys.executable, "-c", CHILD, out], capture_output=True, text=True,
                       env=dict(os.environ, LANDAU_LIB=os.path.abspath(lib)))
    import numpy as np
    msg = r.stdout.strip() or r.stderr[-500:]
    if r.returncode == 0:
        G = np.load(out)
        if ref is None:
            ref = G
        same = np.array_equal(G.view(np.uint64), ref.view(np.uint64))
        msg += f" bitwise_equal_to_first {same} maxrel {np.max(np.abs(G - ref)) / np.abs(ref).max():.2e}"
    print(os.path.basename(lib), msg, flush=True)
