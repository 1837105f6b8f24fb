#!/usr/bin/env python3
"""Benchmark of the Landau Jacobian hot path on B200 (contract: see DESIGN.md §10 Measurement).

Headline workload = BASELINE.json configs[3] built on configs[1]: a FIXED job of 1024 independent
spatial-vertex velocity grids, each the e + D Q3 AMR C2 grid (68 cells, N = 1,088 points, 601 DOFs per
species) with its own thermal-quench-shaped f, sharded over the ranks with no communication
(1024/N vertices per GPU, "scaling": "strong" -- the driver's 1/2/4/8-GPU runs measure the
">= 7x at 8 GPUs" target of north_star directly).  --weak gives every GPU its own --batch vertices.

One step = the whole hot path (SURVEY.md §8(a) a-1 .. a-6) for the local batch:
    landau_set_state_batched -> landau_jacobian_batched (CSR) -> landau_mass (CSR)
with the inputs already resident in HBM.  L2 (126 MB) is flushed between timed steps by writing a
256 MiB buffer outside the timed events.  ms_per_step is the median of the per-step CUDA-event times
(max over ranks).  e2e repeats the step through landau_jacobian_host with pinned host buffers (H2D of f
and D2H of every Jacobian value inside the timed region).

Sub-lines of the same JSON line: "weak" (N > 1: 1024 vertices per GPU), "configs"
(C1, C2, C3 single builds with their full-oracle cpu_baseline; C5 = one Q4 mesh of 108,800 points with
the tile pairs of the mirror kernel split over the N GPUs and one NCCL all-reduce of the partial G per
build, its roofline, its 32-element / 800-target oracle spot check as cpu_baseline and parity), the
NEXT-3 Newton iterations and the NEXT-4 variants.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl landau|reference] [--workload C4|C1|C2|C3|C5]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Landau Jacobian builds/sec + pair-interactions/sec; FP64 % of peak, 1/2/4/8 B200"
UNIT = "builds/s"
# Per-stage library timers (CUDA events around every kernel) force direct launches; inside the timed
# region they would cost the C4 step its CUDA-graph replay (measured 2.92 vs 2.90 ms at 1024 vertices,
# 0.451 vs 0.425 ms at 128), so the headline times graph-replayed steps and the stage breakdown (and
# the dominant kernel's duration for the roofline) comes from a second pass of the same K steps.
# C5 (an NCCL collective inside the build) never replays graphs: its timers stay in the timed region.
TIMERS_IN_LOOP = ("C5",)


class StdoutToStderr:
    """Route fd 1 to fd 2 while libraries initialise (NCCL may print its version on stdout), so that
    rank 0's stdout carries exactly one JSON line."""

    def __enter__(self):
        sys.stdout.flush()
        self._saved = os.dup(1)
        os.dup2(2, 1)
        return self

    def __exit__(self, *a):
        sys.stdout.flush()
        os.dup2(self._saved, 1)
        os.close(self._saved)


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="landau", choices=["landau", "reference"])
    ap.add_argument("--workload", default="C4", choices=["C4", "C1", "C2", "C3", "C5", "C2ncu"])
    ap.add_argument("--batch", type=int, default=1024, help="C4 vertices in the whole job (--weak: per GPU)")
    ap.add_argument("--weak", action="store_true", help="C4: --batch vertices per GPU instead of in the whole job")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sublines", action="store_true", help="headline only (no configs/variants/newton)")
    ap.add_argument("--cpu-sample", type=int, default=16, help="oracle C4 vertices for cpu_baseline")
    ap.add_argument("--stage-timers", default="auto", choices=["auto", "loop", "separate"],
                    help="per-stage library timers inside the timed region (direct launches) or in a separate "
                         "pass after it (the timed steps replay CUDA graphs)")
    ap.add_argument("--c5-cells", type=int, default=32, help="C5 oracle spot check: seeded-random cells")
    ap.add_argument("--tensor-cache", action="store_true",
                    help="NEXT-4 variant: cached mesh tensors + FP64 GEMM inner integral (not the headline path)")
    return ap.parse_args(argv)


def job_vertices(args, world):
    """C4 vertices in the whole job: --batch in all (default, strong scaling) or per GPU (--weak)."""
    return args.batch * world if args.weak else args.batch


def workload(args, world, rank):
    """(description, problem for the mesh, list of per-item problems of this rank)."""
    from paper_conf_ipps_adamsbkw22_b200 import inputs
    if args.workload == "C4":
        B = job_vertices(args, world)
        lo, hi = rank * B // world, (rank + 1) * B // world
        items = [inputs.config4_vertex(b, B) for b in range(lo, hi)]
        desc = {"workload": f"C4: {B} x C2 vertex grids (e+D, Q3 AMR 68 cells, N=1088, thermal-quench f), "
                            f"{B // world} per GPU, no communication",
                "vertices": B, "vertices_per_gpu": B // world, "points_per_vertex": 1088, "order": 3, "species": 2,
                "l2": "flushed between timed steps (256 MiB write)"}
        return desc, items[0] if items else inputs.config4_vertex(0, B), items
    p = inputs.CONFIGS[args.workload]()
    desc = {"workload": f"{args.workload} single build", "points": p.npoints, "order": p.order,
            "species": len(p.species), "l2": "flushed between timed steps (256 MiB write)"}
    return desc, p, [p] if rank == 0 or world == 1 or args.workload == "C5" else []


class Clocks:
    """SM clock and clock-event reasons sampled in-process through NVML every 5 ms (nvidia-smi when NVML
    is unavailable) during the timed region (B200_PROFILING.md clocks line).  __enter__ returns only
    after the first sample is taken; mark_start/mark_end bracket the timed region and summary() keeps
    the samples inside it (all samples if the region saw none)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    # NVML clock-event reason bits (nvml.h nvmlClocksEventReason*)
    NVML_BITS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40}

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.times = []
        self.t0 = self.t1 = None
        self._stop = threading.Event()
        self._ready = threading.Event()
        self._t = None

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        idx = self.index
        vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
        parts = [p.strip() for p in vis.split(",") if p.strip()]
        if parts and all(p.isdigit() for p in parts) and idx < len(parts):
            idx = int(parts[idx])
        return pynvml, pynvml.nvmlDeviceGetHandleByIndex(idx)

    def _add(self, row):
        self.rows.append(row)
        self.times.append(time.perf_counter())
        self._ready.set()

    def _run(self):
        try:
            nv, h = self._nvml_handle()
            reasons_fn = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                nv.nvmlDeviceGetCurrentClocksThrottleReasons
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            self.source = "nvml"
            while True:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                bits = reasons_fn(h)
                self._add([str(self.index), str(sm), str(mx), "", hex(bits)] +
                          ["Active" if bits & self.NVML_BITS[k] else "Not Active"
                           for k in ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")])
                if self._stop.wait(0.005):
                    return
        except Exception:
            self.rows, self.times = [], []
        self.source = "nvidia-smi"
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5).stdout
                for line in out.strip().splitlines():
                    self._add([x.strip() for x in line.split(",")])
            except Exception:
                pass
            self._ready.set()
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        self._ready.wait(timeout=15)   # the first sample exists before the timed region starts
        return self

    def mark_start(self):
        self.t0 = time.perf_counter()

    def mark_end(self):
        self.t1 = time.perf_counter()
        time.sleep(0.006)               # one more sample at the region's end

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        rows = self.rows
        if self.t0 is not None and self.t1 is not None and self.times:
            inside = [r for r, t in zip(self.rows, self.times) if self.t0 - 0.006 <= t <= self.t1 + 0.006]
            rows = inside or self.rows
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if len(r) > 5 + k and r[5 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows), "source": getattr(self, "source", "nvidia-smi")}


def fp64_peak_tflops(props, sm_max_mhz):
    """Derived FP64 (DFMA) peak: SMs x 64 FP64 lanes per SM per clock (4 SMSPs x 16) x 2 FLOP x clock.
    See DESIGN.md 'Roofline'; tools/fp64_peak.cu measures the DFMA rate on the box."""
    return props.multi_processor_count * 64 * 2 * sm_max_mhz * 1e6 / 1e12


def load_profile_traffic(key):
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "inner_traffic.json"))).get(key)
    except Exception:
        return None


# FP64 FLOP (2*DFMA + DMUL + DADD) per pair evaluation, counted once from ncu
# sm__sass_thread_inst_executed_op_{dfma,dmul,dadd}_pred_on of each inner kernel on the C4 workload
# (profiles/r02_flops_*.csv with the degree-9 D fit):
FLOP_PER_PAIR_DIRECTED = 169.0   # inner_kernel, per ordered (target, source) pair
FLOP_PER_PAIR_SYMMETRIC = 185.2  # inner_sym_kernel, per unordered pair
FLOP_PER_EVAL_MIRROR = 190.1     # inner_mir_kernel (slot kernel), per U or V tensor evaluation
FLOP_PER_EVAL_VTX = 190.2        # inner_vtx_kernel (per-vertex kernel), per U or V tensor evaluation
FLOP_PER_PAIR_3D = 58.0          # inner3d_kernel, per ordered pair
FLOP_PER_EVAL_MDIR = 179.2       # inner_mdir_kernel (mirror directed), per padded U or V evaluation
INNER_PATHS = ["directed (ordered pairs)", "symmetric (unordered pairs)", "tensor cache + FP64 DGEMM (cuBLAS)",
               "mirror-symmetric slot kernel (one tensor per unordered pair and its z-mirror)",
               "mirror-symmetric per-vertex kernel (stream-K over vertex rounds, sums in shared memory)",
               "mirror-symmetric directed (U + V per target and source, forward sums)"]


def inner_flops(st, N):
    """(FLOP per evaluation, FLOP per inner launch) from the library's stats of the last build."""
    p = st["inner_path"]
    if p == 2:
        return 14.0, 14.0 * st["nbatch"] * N * N
    if p == 5:
        return FLOP_PER_EVAL_MDIR, FLOP_PER_EVAL_MDIR * st["nbatch"] * st["pair_evaluations"]
    if p in (3, 4):
        f = FLOP_PER_EVAL_VTX if p == 4 else FLOP_PER_EVAL_MIRROR
        return f, f * st["nbatch"] * st["pair_evaluations"]
    if p == 1:
        return FLOP_PER_PAIR_SYMMETRIC, FLOP_PER_PAIR_SYMMETRIC * st["nbatch"] * N * (N - 1) / 2
    return FLOP_PER_PAIR_DIRECTED, FLOP_PER_PAIR_DIRECTED * st["nbatch"] * st["targets"] * N


def timed_steps(torch, stream, step, steps, flush, clk=None):
    """Per-step CUDA-event times (ms) on the library's stream, L2 flushed before each step."""
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    torch.cuda.synchronize()
    if clk:
        clk.mark_start()
    for k in range(steps):
        flush.fill_(float(k))
        evs[k][0].record(stream)
        step()
        evs[k][1].record(stream)
    torch.cuda.synchronize()
    if clk:
        clk.mark_end()
    return [a.elapsed_time(b) for a, b in evs]


def max_over_ranks(torch, dist, world, x):
    t = torch.tensor([float(x)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def oracle_c4_baseline(B, nsample):
    """The oracle (full Jacobian incl. its |.| scale) on nsample C4 vertices b = 0, 68, ...,
    all host cores, plus a 1-core figure on two of them."""
    from oracle.oracle import Oracle, get_threads, set_threads
    from paper_conf_ipps_adamsbkw22_b200 import inputs
    step = max(1, (B - 1) // max(nsample - 1, 1)) if nsample > 1 else 1
    verts = [min(B - 1, k * step) for k in range(nsample)]
    t = 0.0
    for b in verts:
        o = Oracle(inputs.config4_vertex(b, B))
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        t += time.perf_counter() - t0
    cores = get_threads()
    set_threads(1)
    t1 = 0.0
    for b in verts[:2]:
        o = Oracle(inputs.config4_vertex(b, B))
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        t1 += time.perf_counter() - t0
    set_threads(cores)
    return {"value": len(verts) / t, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"full oracle Jacobian (incl. |.| scale) of {len(verts)} of the {B} C4 vertices (b = {verts})",
            "seconds": t, "value_1core": min(2, len(verts)) / t1, "omp_num_threads": os.environ.get("OMP_NUM_THREADS"),
            "nproc": os.cpu_count()}


def oracle_full_build(prob):
    """One full oracle Jacobian (with the |.| scale) of a single-build config: (J, Ja, seconds)."""
    from oracle.oracle import Oracle
    o = Oracle(prob)
    f = o.coefficients()
    t0 = time.perf_counter()
    J, Ja = o.jacobian(f)
    return o, J, Ja, time.perf_counter() - t0


def oracle_c5_sample(prob, ncells=16, seed=2022):
    """The oracle's C5 element blocks (all N sources, |.| scale) for ncells seeded-random cells, scaled to
    builds/s by the cell count (the oracle's cost is linear in the target cells): (builds/s, seconds, sample)."""
    from oracle.oracle import Oracle
    o = Oracle(prob)
    ncell = len(prob.grids[0][1])
    cells = np.sort(np.random.default_rng(seed).choice(ncell, ncells, replace=False))
    mask = np.zeros(ncell, dtype=np.uint8)
    mask[cells] = 1
    f = o.coefficients()
    t0 = time.perf_counter()
    o.jacobian_coo(f, mask)
    secs = time.perf_counter() - t0
    return (ncells / (ncell * secs), secs,
            f"oracle element blocks of {ncells} seeded-random C5 cells of {ncell} (all {prob.npoints} sources, incl. |.| "
            f"scale), scaled to whole builds by the cell count")


def run_reference(args, world, rank):
    """--impl reference: the oracle arm (the CPU program the paper's equations define), timed on host cores."""
    if rank != 0:
        return 0
    from oracle.oracle import Oracle, get_threads
    from paper_conf_ipps_adamsbkw22_b200 import inputs
    desc, prob0, _ = workload(args, world, 0)
    desc = dict(desc, parallelism=f"batch-shard x{world}" if world > 1 else "1 GPU")
    B = job_vertices(args, world)
    times = []
    sample = f"1 vertex Jacobian per step ({args.workload}), full oracle incl. |.| scale"
    for k in range(args.warmup + args.steps if args.workload != "C5" else 0):
        p = inputs.config4_vertex((k * 97) % B, B) if args.workload == "C4" else inputs.CONFIGS[args.workload]()
        o = Oracle(p)
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        dt = time.perf_counter() - t0
        if k >= args.warmup:
            times.append(dt)
    if args.workload == "C5":   # a whole C5 oracle build is hours: each step a bounded cell sample
        for k in range(args.warmup + args.steps):
            v, secs, sample = oracle_c5_sample(prob0, 8, seed=2022 + k)
            if k >= args.warmup:
                times.append(1.0 / v)
        sample = "per step: " + sample
    med = statistics.median(times)
    value = 1.0 / med
    N = 1088 if args.workload == "C4" else prob0.npoints
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * med,
            "higher_is_better": True, "scaling": "weak" if args.weak or args.workload != "C4" else "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": desc, "pairs_per_s": value * N * N,
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": get_threads(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def single_build_line(torch, L, inputs, name, local, stream, flush, steps, warmup, with_cpu):
    """One C1/C2/C3 build per step (set_state + jacobian (CSR) + mass, CUDA-graph replay), and the full
    oracle on the same config as its cpu_baseline."""
    p = inputs.CONFIGS[name]()
    h = L.Landau.from_problem(p, device=local, stream=stream)
    f = torch.tensor(inputs.coefficients(p, h.all_nodes()), device="cuda")
    v = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    m = torch.empty(h.nnz, dtype=torch.float64, device="cuda")

    def step():
        h.set_state(f)
        h.jacobian(v)
        h.mass(1.0e3, m)

    for _ in range(max(warmup, 3)):
        step()
    ts = timed_steps(torch, stream, step, steps, flush)
    ms = statistics.median(ts)
    st = h.stats()
    out = {"value": 1e3 / ms, "unit": UNIT, "ms_per_step": ms, "ms_mean": statistics.mean(ts),
           "points": p.npoints, "pairs_per_s": 1e3 / ms * p.npoints ** 2, "inner_path": INNER_PATHS[st["inner_path"]],
           "note": f"BASELINE configs ({name}): one build per step, set_state + jacobian (CSR) + mass, CUDA-graph replay"}
    if with_cpu:
        o, Jo, Ja, secs = oracle_full_build(p)
        from oracle.oracle import get_threads
        Jg = v.cpu().numpy()
        out["cpu_baseline"] = {"value": 1.0 / secs, "unit": UNIT, "cores": get_threads(), "kind": "oracle",
                               "sample": f"one full {name} oracle Jacobian (incl. |.| scale)"}
        out["parity_max_dJ_over_Jabs"] = float(np.max(np.abs(Jg - Jo) / Ja))
    h.close()
    return out


def c5_line(torch, dist, L, inputs, world, rank, local, stream, flush, steps, warmup, ncheck, with_cpu, peak):
    """C5: one e+D Q4 mesh (4,352 cells, N = 108,800).  LANDAU_DIST_ELEMENTS over the N ranks: the mirror
    slot kernel's tile pairs are split (landau_pair_partition), each rank reduces a partial G over all
    points and one ncclAllReduce sums them (the path's exchange step); element matrices and assembly
    then run for every cell.  Timed per build (max over ranks), with the all-reduce's own event time,
    the inner kernel's roofline, and (rank 0, outside the timed region) the oracle on every pair of the
    points of ncheck seeded-random cells: their COO element blocks against the GPU (parity) and the
    oracle time as cpu_baseline (SURVEY §8(d) spot check: 32 cells, 800 targets)."""
    p = inputs.config5()
    with StdoutToStderr():
        if world > 1:
            dd = L.make_dist(L.LANDAU_DIST_ELEMENTS)
        else:
            dd = {"rank": 0, "world": 1, "mode": L.LANDAU_DIST_ELEMENTS, "nccl_unique_id": L.landau_nccl_unique_id()}
        h = L.Landau.from_problem(p, device=local, stream=stream, dist=dd)
    F = torch.tensor(inputs.coefficients(p, h.all_nodes()), device="cuda")
    v = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    m = torch.empty(h.nnz, dtype=torch.float64, device="cuda")

    def step():
        h.set_state(F)
        h.jacobian(v)
        h.mass(1.0e3, m)

    for _ in range(max(warmup, 2)):
        step()
    if world > 1:
        dist.barrier()
    h.set_timing(True)
    ts = timed_steps(torch, stream, step, steps, flush)
    tim = h.get_timing()
    h.set_timing(False)
    st = h.stats()
    ms = max_over_ranks(torch, dist, world, statistics.median(ts))
    N = h.npoints
    fpe, fpl = inner_flops(st, N)
    inner_s = tim["inner"][0] / max(tim["inner"][1], 1) / 1e3
    ach = fpl / inner_s / 1e12 if tim["inner"][1] else None
    out = {"value": 1e3 / ms, "unit": UNIT, "ms_per_step": ms, "points": N, "pairs_per_s": 1e3 / ms * N * N,
           "parallelism": f"pair split x{world} + ncclAllReduce of G ({5 * N * 8 / 1e6:.2f} MB)" if world > 1
           else "1 GPU (LANDAU_DIST_ELEMENTS handle at world 1: no exchange)",
           "inner_path": INNER_PATHS[st["inner_path"]],
           "stage_ms_per_step": {k: v_[0] / steps for k, v_ in tim.items() if v_[0]},
           "allreduce_ms_per_step": tim["allgather"][0] / steps if tim["allgather"][1] else 0.0,
           "roofline": {"bound": "alu", "kernel": "inner_mir_kernel (a-2, this rank's share of the tile pairs)",
                        "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak if ach else None,
                        "flop_per_eval": fpe, "flops_per_launch": fpl, "inner_ms_per_launch": inner_s * 1e3}}
    if rank == 0 and ncheck > 0:
        from oracle.oracle import Oracle, get_threads
        Jc = torch.empty(h.ncoo, dtype=torch.float64, device="cuda")
        h.jacobian(Jc, L.LANDAU_COO)
        Jg = Jc.cpu().numpy()
        o = Oracle(p)
        ncell = len(p.grids[0][1])
        cells = np.sort(np.random.default_rng(2022).choice(ncell, ncheck, replace=False))
        mask = np.zeros(ncell, dtype=np.uint8)
        mask[cells] = 1
        t0 = time.perf_counter()
        Jo, Ja = o.jacobian_coo(o.coefficients(), mask)
        secs = time.perf_counter() - t0
        sel = np.isfinite(Jo)
        targets = ncheck * (p.order + 1) ** 2
        out["parity"] = {"cells": int(ncheck), "targets": int(targets), "entries": int(sel.sum()),
                         "max_dJ_over_Jabs": float(np.max(np.abs(Jg[sel] - Jo[sel]) / Ja[sel])),
                         "bar": 1e-11}
        if with_cpu:
            out["cpu_baseline"] = {"value": targets / secs, "unit": "target points/s (all N sources each)",
                                   "cores": get_threads(), "kind": "oracle",
                                   "sample": f"oracle element blocks of {ncheck} seeded-random cells ({targets} targets x "
                                             f"{N} sources, incl. |.| scale)", "seconds": secs,
                                   "gpu_same_unit": N * 1e3 / ms}
    h.close()
    return out


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, world, rank)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_adamsbkw22_b200 import inputs
    from paper_conf_ipps_adamsbkw22_b200 import landau as L

    torch.cuda.set_device(local)
    if world > 1:
        with StdoutToStderr():
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    stream = torch.cuda.current_stream()
    desc, prob0, items = workload(args, world, rank)
    dist_desc = None
    if args.workload == "C5":
        with StdoutToStderr():
            dist_desc = L.make_dist(L.LANDAU_DIST_ELEMENTS) if world > 1 else \
                {"rank": 0, "world": 1, "mode": L.LANDAU_DIST_ELEMENTS, "nccl_unique_id": L.landau_nccl_unique_id()}
        items = [prob0]
        desc = dict(desc, workload="C5: one e+D Q4 mesh (4352 cells, N=108800), LANDAU_DIST_ELEMENTS: the mirror "
                                   "kernel's tile pairs split over the GPUs, NCCL all-reduce of the partial G")
    with StdoutToStderr():
        h = L.Landau.from_problem(prob0, device=local, stream=stream, dist=dist_desc)
    if args.tensor_cache:
        h.set_tensor_cache(True)
        desc = dict(desc, variant="NEXT-4 tensor cache: inner integral as FP64 GEMMs over cached tensors")
    nodes = h.all_nodes()
    nloc = len(items)
    N = h.npoints
    F_host = np.stack([inputs.coefficients(p, nodes) for p in items]) if nloc else np.zeros((1, h.ndof))
    F = torch.tensor(F_host, device="cuda")
    vals = torch.empty((max(nloc, 1), h.nnz), dtype=torch.float64, device="cuda")
    mvals = torch.empty(h.nnz, dtype=torch.float64, device="cuda")
    flush = torch.empty(256 * 1024 * 1024 // 8, dtype=torch.float64, device="cuda")
    shift = 1.0e3
    props = torch.cuda.get_device_properties(local)

    def step():
        if nloc:
            h.set_state_batched(F)
            h.jacobian_batched(vals)
            h.mass(shift, mvals)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    # stage timers: see TIMERS_IN_LOOP
    in_loop_timers = args.workload in TIMERS_IN_LOOP if args.stage_timers == "auto" else args.stage_timers == "loop"
    h.set_timing(in_loop_timers)
    n0 = h.launch_count()
    with Clocks(local) as clk:
        ts = timed_steps(torch, stream, step, args.steps, flush, clk)
    launches = h.launch_count() - n0
    st = h.stats()   # how the timed builds ran (read before the e2e pass changes the batch layout)
    if not in_loop_timers:
        h.set_timing(True)
        for k in range(args.steps):
            flush.fill_(float(k))
            step()
    tim = h.get_timing()
    h.set_timing(False)
    local_med, local_mean = statistics.median(ts), statistics.mean(ts)
    if world > 1:
        dist.barrier()
    ms_per_step = max_over_ranks(torch, dist, world, local_med)
    ms_mean = max_over_ranks(torch, dist, world, local_mean)
    total_builds = job_vertices(args, world) if args.workload == "C4" else 1
    scaling = "weak" if (args.weak or args.workload != "C4") else "strong"
    value = total_builds / (ms_per_step / 1e3)
    pairs_per_build = N * N

    # ---- e2e through the host-pointer C-ABI entry point --------------------------------------
    f_pin = torch.tensor(F_host).pin_memory()
    v_pin = torch.empty((max(nloc, 1), h.nnz), dtype=torch.float64).pin_memory()
    for _ in range(min(args.warmup, 2)):
        if nloc:
            h.jacobian_host(f_pin, v_pin)
    ets = []
    for k in range(args.steps):
        flush.fill_(float(k))
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        if nloc:
            h.jacobian_host(f_pin, v_pin)
        b.record(stream)
        torch.cuda.synchronize()
        ets.append(a.elapsed_time(b))
    e_ms = max_over_ranks(torch, dist, world, statistics.median(ets))
    e2e_value = total_builds / (e_ms / 1e3)

    # ---- roofline of the dominant kernel (inner integral, FP64 pipe) --------------------------
    inner_ms, inner_n = tim["inner"]
    inner_avg_s = inner_ms / max(inner_n, 1) / 1e3
    flop_per_pair, flops_per_launch = inner_flops(st, N)
    achieved = flops_per_launch / inner_avg_s / 1e12 if inner_n else None
    clocks = clk.summary()
    sm_max = clocks["sm_max_mhz"] or 1965.0
    peak = fp64_peak_tflops(props, sm_max)
    roof = {"bound": "alu", "kernel": "inner_vtx_kernel (a-2, FP64 pipe; inner_path says which kernel ran)",
            "timing": ("CUDA events around the kernel on the library stream, " +
                       ("inside the timed region" if in_loop_timers else
                        "over a second pass of the same K steps right after the timed region")),
            "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": (achieved / peak) if achieved else None,
            "traffic": load_profile_traffic(args.workload),
            "fp64_pipe_active_ncu": load_profile_traffic(args.workload + "_fp64_pipe_active"),
            "peak_note": f"derived FP64 DFMA peak: {props.multi_processor_count} SMs x 64 lanes x 2 FLOP x {sm_max:.0f} MHz "
                         "(MEASURED_PEAKS.json has no FP64 figure; tools/fp64_peak.cu measured 36.96 TFLOP/s)",
            "inner_path": INNER_PATHS[st["inner_path"]],
            "flop_per_pair": flop_per_pair, "flops_per_launch": flops_per_launch,
            "inner_ms_per_launch": inner_avg_s * 1e3,
            "inner_share_of_step": (inner_ms / args.steps) / local_mean if local_mean else None,
            "pairs_per_s_inner": pairs_per_build * max(nloc, 1) / inner_avg_s * world if inner_n else None}
    stage_ms = {k: v[0] / args.steps for k, v in tim.items()}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "ms_per_step_mean": ms_mean,
            "timing": "median of per-step CUDA-event times on the library stream, max over ranks",
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(desc, parallelism=(f"pair split x{world}" if args.workload == "C5" else
                                              f"batch-shard x{world}") if world > 1 else "1 GPU"),
            "pairs_per_s": value * pairs_per_build, "roofline": roof, "stage_ms_per_step": stage_ms,
            "stage_timers": "in timed region" if in_loop_timers else
                            "separate pass of the same K steps right after the timed region (direct launches; "
                            "the timed region replays CUDA graphs)",
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(F_host.nbytes) * world,
                    "d2h_bytes_per_step": int(v_pin.numel() * 8) * world, "api": "landau_jacobian_host",
                    "ms_per_step": e_ms},
            "gpu_launches": int(launches), "clocks": clocks}
    extras = args.workload == "C4" and not args.tensor_cache and not args.no_sublines

    # ---- weak scaling sub-line (N > 1): every GPU its own 1024 vertices ---------------------------
    if extras and world > 1:
        try:
            Bw = args.batch
            hw = L.Landau.from_problem(prob0, device=local, stream=stream)
            Fw = torch.tensor(np.stack([inputs.coefficients(inputs.config4_vertex(b, Bw * world), nodes)
                                        for b in range(rank * Bw, (rank + 1) * Bw)]), device="cuda")
            vw = torch.empty((Bw, hw.nnz), dtype=torch.float64, device="cuda")

            def wstep():
                hw.set_state_batched(Fw)
                hw.jacobian_batched(vw)
                hw.mass(shift, mvals)
            for _ in range(args.warmup):
                wstep()
            dist.barrier()
            wms = max_over_ranks(torch, dist, world, statistics.median(timed_steps(torch, stream, wstep, args.steps, flush)))
            line["weak"] = {"value": Bw * world / (wms / 1e3), "unit": UNIT, "ms_per_step": wms,
                            "vertices_per_gpu": Bw, "vertices": Bw * world, "scaling": "weak"}
            hw.close()
            del Fw, vw
        except Exception as e:
            line["weak"] = {"unavailable": str(e)[:200]}

    # ---- configs: C1-C3 single builds (rank 0) and C5 across all ranks ----------------------------
    if extras:
        cfgs = {}
        if rank == 0:
            for name in ("C1", "C2", "C3"):
                try:
                    cfgs[name] = single_build_line(torch, L, inputs, name, local, stream, flush, args.steps, args.warmup,
                                                   world == 1 and not args.no_cpu_baseline)
                except Exception as e:
                    cfgs[name] = {"unavailable": str(e)[:200]}
        try:
            cfgs["C5"] = c5_line(torch, dist, L, inputs, world, rank, local, stream, flush, max(5, args.steps // 2),
                                 args.warmup, args.c5_cells, world == 1 and not args.no_cpu_baseline, peak)
        except Exception as e:
            cfgs["C5"] = {"unavailable": str(e)[:200]}
        line["configs"] = cfgs
        if "C2" in cfgs:
            line["c2_single_build"] = cfgs["C2"]

    # ---- NEXT-4 variants on the same job (informational; the headline is the pairwise path) -------
    if extras and nloc:
        try:
            h.set_tensor_cache(True)
            step()
            h.set_timing(True)
            vts = timed_steps(torch, stream, step, args.steps, flush)
            vt = h.get_timing()
            h.set_timing(False)
            h.set_tensor_cache("recompute")
            step()
            rts = timed_steps(torch, stream, step, args.steps, flush)
            h.set_tensor_cache(False)
            vstep = max_over_ranks(torch, dist, world, statistics.median(vts))
            rstep = max_over_ranks(torch, dist, world, statistics.median(rts))
            gemm_s = vt["inner"][0] / max(vt["inner"][1], 1) / 1e3
            line["variants"] = {"tensor_cache_gemm": {
                "value": total_builds / (vstep / 1e3), "unit": UNIT, "ms_per_step": vstep,
                "inner_ms_per_launch": gemm_s * 1e3, "inner_tflops": 14.0 * nloc * N * N / gemm_s / 1e12,
                "note": "SURVEY NEXT-4: mesh tensors cached once (7 N^2 doubles), inner integral as three FP64 "
                        "DGEMMs (cuBLAS, FP64 tensor cores); same sums up to order, parity-tested"},
                "tensor_gemm_recompute": {
                "value": total_builds / (rstep / 1e3), "unit": UNIT, "ms_per_step": rstep,
                "note": "the GEMM formulation with all N^2 tensors re-evaluated inside every timed build "
                        "(the batch shares one mesh): no state carried across builds"}}
        except Exception as e:
            line["variants"] = {"tensor_cache_gemm": {"unavailable": str(e)[:200]}}
        try:
            xyz3, w3 = inputs.points3d(8, 3)
            wTD3, wTK3 = inputs.fields3d(xyz3, w3)
            n3 = int(w3.size)
            X3, D3, K3 = (torch.tensor(a, device="cuda") for a in (xyz3, wTD3, wTK3))
            G3 = torch.empty((9, n3), dtype=torch.float64, device="cuda")
            for _ in range(2):
                L.landau3d_inner(X3, D3, K3, G3, stream)
            ms3 = statistics.median(timed_steps(torch, stream, lambda: L.landau3d_inner(X3, D3, K3, G3, stream),
                                                args.steps, flush))
            line.setdefault("variants", {})["inner3d_cartesian"] = {
                "value": n3 * n3 / (ms3 * 1e-3), "unit": "pairs/s", "points": n3, "ms_per_launch": ms3,
                "tflops": FLOP_PER_PAIR_3D * n3 * n3 / (ms3 * 1e-3) / 1e12,
                "frac_of_fp64_peak": FLOP_PER_PAIR_3D * n3 * n3 / (ms3 * 1e-3) / 1e12 / peak,
                "note": "SURVEY NEXT-4: G_D, G_K with U = (|u|^2 I - u u^T)/|u|^3 directly (no elliptic integrals), "
                        "ordered pairs, parity-tested against oracle O12"}
        except Exception as e:
            line.setdefault("variants", {})["inner3d_cartesian"] = {"unavailable": str(e)[:200]}
        try:   # the whole 3D Jacobian (a-1, inner, a-4, a-3 + a-5) on the same 8^3 Q3 grid, two species
            p3 = inputs.config3d(8, 3)
            with torch.cuda.stream(stream):
                h3 = L.Landau3D(p3.ncell, p3.order, p3.R, p3.species, p3.nu, device=local, stream=stream)
            F3 = torch.tensor(inputs.coefficients3d(p3, h3.nodes()), device="cuda")
            J3 = torch.empty((len(p3.species), h3.nnz), dtype=torch.float64, device="cuda")
            for _ in range(2):
                h3.jacobian(F3, J3)
            ms3j = statistics.median(timed_steps(torch, stream, lambda: h3.jacobian(F3, J3), args.steps, flush))
            h3.set_timing(True)
            for _ in range(2):   # the second timed build (the first pays the partials pool's growth)
                h3.jacobian(F3, J3)
            st3 = h3.get_timing()
            h3.set_timing(False)
            line["variants"]["jacobian3d"] = {
                "value": 1e3 / ms3j, "unit": "builds/s", "ms_per_step": ms3j, "points": h3.npoints, "ndof": h3.ndof,
                "nnz_per_species": h3.nnz, "species": len(p3.species), "stage_ms": st3,
                "note": "SURVEY NEXT-4 completed: 3D Cartesian Jacobian (field3d, inner3d, element3d, assembly) on "
                        "8^3 Q3 cubes, e + a light ion; parity-tested against oracle O13 on 2^3/3^3 grids"}
            h3.close()
        except Exception as e:
            line.setdefault("variants", {})["jacobian3d"] = {"unavailable": str(e)[:200]}

    # ---- NEXT-3: quasi-Newton backward-Euler iterations on the same batch --------------------------
    if extras and nloc:
        try:
            it_per_call, dt_n = 2, 0.002
            Fn = torch.empty_like(F)
            # the thermal-quench source of Eq. 4 (a cold pulse injecting 5x the initial density over 10
            # steps, reading R-7): the first step's rate x each vertex's cold-Maxwellian shape
            rate = 5.0 * inputs.quench_pulse_fraction(0.0, dt_n, 10 * dt_n) / dt_n
            Src = torch.tensor(np.stack([rate * inputs.quench_source_shape(p, nodes) for p in items]), device="cuda")
            for _ in range(2):
                h.implicit_step_batched(dt_n, F, Fn, max_iter=it_per_call, rtol=0.0, src=Src)
            h.set_timing(True)
            nts = timed_steps(torch, stream,
                              lambda: h.implicit_step_batched(dt_n, F, Fn, max_iter=it_per_call, rtol=0.0, src=Src),
                              args.steps, flush)
            nt = h.get_timing()
            h.set_timing(False)
            ms_it = max_over_ranks(torch, dist, world, statistics.median(nts)) / it_per_call
            line["newton"] = {
                "value": total_builds / (ms_it / 1e3), "unit": "vertex Newton iterations/s", "ms_per_iteration": ms_it,
                "stage_ms_per_iteration": {k: v[0] / (args.steps * it_per_call) for k, v in nt.items()},
                "note": "SURVEY NEXT-3: backward-Euler step by quasi-Newton (Jacobian about each iterate, A = M/dt - J "
                        "factored by the RCM band LU, solve) with the thermal-quench source of Eq. 4 (cold pulse, "
                        "R-7), all vertices of the job per iteration, dt = 0.002, "
                        f"{it_per_call} iterations per landau_implicit_step_batched call; context: the paper's V100 "
                        "node figure is a different problem (10 species, 80 cells, CPU LU)"}
        except Exception as e:
            line["newton"] = {"unavailable": str(e)[:200]}

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        if args.workload == "C4":
            line["cpu_baseline"] = oracle_c4_baseline(job_vertices(args, world), args.cpu_sample)
        elif args.workload == "C5":
            v, secs, sample = oracle_c5_sample(prob0, 16)
            from oracle.oracle import get_threads
            line["cpu_baseline"] = {"value": v, "unit": UNIT, "cores": get_threads(), "kind": "oracle",
                                    "sample": sample, "seconds": secs}
        elif args.workload in ("C1", "C2", "C3", "C2ncu"):
            _, _, _, secs = oracle_full_build(prob0)
            from oracle.oracle import get_threads
            line["cpu_baseline"] = {"value": 1.0 / secs, "unit": UNIT, "cores": get_threads(), "kind": "oracle",
                                    "sample": f"one full {args.workload} oracle Jacobian (incl. |.| scale)"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
