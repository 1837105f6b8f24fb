#!/usr/bin/env python3
"""Benchmark of the Landau Jacobian hot path on B200 (contract: see DESIGN.md §Measurement).

Workload (default, BASELINE.json configs[3] built on configs[1]): a batch of 1024 independent
spatial-vertex velocity grids, each the e + D Q3 AMR C2 grid (68 cells, N = 1,088 points, 601 DOFs
per species) with its own thermal-quench-shaped f.  The vertices are independent problems, so they are
sharded over the ranks with no communication: --batch vertices per GPU (default 1024), a job of
--batch x world vertices ("scaling": "weak"); --strong splits a fixed job of --batch vertices instead.

One step = the whole hot path (SURVEY.md §8(a) a-1 .. a-6) for the local batch:
    landau_set_state_batched -> landau_jacobian_batched (CSR) -> landau_mass (CSR)
with the inputs already resident in HBM.  L2 (126 MB) is flushed between timed steps by writing a
256 MiB buffer outside the timed events.  e2e repeats the step through landau_jacobian_host with
pinned host buffers (H2D of f and D2H of every Jacobian value inside the timed region).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl landau|reference] [--workload C4|C2|C3|C5]
"""
import argparse
import json
import math
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


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="landau", choices=["landau", "reference"])
    ap.add_argument("--workload", default="C4", choices=["C4", "C1", "C2", "C3", "C5"])
    ap.add_argument("--batch", type=int, default=1024, help="C4 vertices per GPU (--strong: in the whole job)")
    ap.add_argument("--strong", action="store_true", help="C4: split a fixed job of --batch vertices over the GPUs")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle vertices for cpu_baseline (0 = auto)")
    ap.add_argument("--tensor-cache", action="store_true",
                    help="NEXT-4 variant: cached mesh tensors + FP64 GEMM inner integral (not the headline path)")
    return ap.parse_args()


def job_vertices(args, world):
    """C4 vertices in the whole job: --batch per GPU (weak scaling), or --batch in all (--strong)."""
    return args.batch if args.strong else args.batch * world


def workload(args, world, rank):
    """(name, problem for the mesh, list of per-item problems of this rank, pairs per build)."""
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
    return desc, p, [p] if rank == 0 or world == 1 else []


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    # NVML clock-event reason bits (nvml.h nvmlClocksEventReason*)
    NVML_BITS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40}

    def _nvml_handle(self):
        import pynvml
        pynvml.nvmlInit()
        idx = self.index
        vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
        parts = [p.strip() for p in vis.split(",") if p.strip()]
        if parts and all(p.isdigit() for p in parts) and idx < len(parts):
            idx = int(parts[idx])
        return pynvml, pynvml.nvmlDeviceGetHandleByIndex(idx)

    def _run(self):
        # In-process NVML sampling every 5 ms, so that a timed region of a few tens of ms still gets
        # several samples; nvidia-smi (one process per sample, ~50 ms) only when NVML is unavailable.
        try:
            nv, h = self._nvml_handle()
            reasons_fn = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                nv.nvmlDeviceGetCurrentClocksThrottleReasons
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            while True:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                bits = reasons_fn(h)
                self.rows.append([str(self.index), str(sm), str(mx), "", hex(bits)] +
                                 ["Active" if bits & self.NVML_BITS[k] else "Not Active"
                                  for k in ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown",
                                            "sw_power_cap")])
                if self._stop.wait(0.005):
                    break
            self.source = "nvml"
            return
        except Exception:
            self.rows = []
        self.source = "nvidia-smi"
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=5).stdout
                for line in out.strip().splitlines():
                    self.rows.append([x.strip() for x in line.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if len(r) > 5 + k and r[5 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows), "source": getattr(self, "source", "nvidia-smi")}


def fp64_peak_tflops(props, sm_max_mhz):
    """Derived FP64 (DFMA) peak: SMs x 64 FP64 lanes per SM per clock (4 SMSPs x 16) x 2 FLOP x clock.
    See DESIGN.md 'Roofline'; tools/fp64_peak.cu measures the DFMA rate on the box."""
    return props.multi_processor_count * 64 * 2 * sm_max_mhz * 1e6 / 1e12


def load_profile_traffic(workload):
    path = os.path.join(ROOT, "profiles", "inner_traffic.json")
    try:
        d = json.load(open(path))
        return d.get(workload)
    except Exception:
        return None


# FP64 FLOP (2*DFMA + DMUL + DADD) per pair evaluation, counted once from ncu
# sm__sass_thread_inst_executed_op_{dfma,dmul,dadd}_pred_on of each inner kernel on the C4 workload
# (profiles/r01_inner_ncu.txt):
#   directed kernel:  173 FLOP per ordered (target, source) pair, N^2 per batch item
#   symmetric kernel: 189 FLOP per unordered pair, N (N - 1) / 2 per batch item (both targets updated)
FLOP_PER_PAIR_DIRECTED = 173.0
FLOP_PER_PAIR_SYMMETRIC = 189.2
# mirror-symmetric kernel: FP64 FLOP (2 DFMA + DMUL + DADD, ncu SASS counts on C4) per tensor
# evaluation, (N/2)^2 evaluations per batch item (profiles/r01_flops_mirror.csv)
FLOP_PER_EVAL_MIRROR = 194.7   # inner_mir_kernel (slot kernel; profiles/r01_flops_mirror.csv)
FLOP_PER_EVAL_VTX = 195.0      # inner_vtx_kernel (per-vertex kernel; profiles/r01_flops_vtx.csv)
FLOP_PER_PAIR_3D = 58.0        # inner3d_kernel, per ordered pair (profiles/r01_flops_3d.csv)
FLOP_PER_EVAL_MDIR = 183.2     # inner_mdir_kernel (mirror directed, per padded U or V evaluation; profiles/r01_flops_mdir.csv)


def cpu_baseline(args, desc, nsample):
    from oracle.oracle import Oracle, get_threads
    from paper_conf_ipps_adamsbkw22_b200 import inputs
    B = args.batch
    if args.workload == "C4":
        verts = [int(round(k * (B - 1) / max(nsample - 1, 1))) for k in range(nsample)]
        probs = [inputs.config4_vertex(b, B) for b in verts]
        sample = f"full oracle Jacobian (incl. |.| scale) of {nsample} of the {B} C4 vertices (b = {verts})"
    else:
        probs = [inputs.CONFIGS[args.workload]()]
        sample = f"full oracle Jacobian of one {args.workload} build"
    from oracle.oracle import set_threads
    t = 0.0
    for p in probs:
        o = Oracle(p)
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        t += time.perf_counter() - t0
    cores = get_threads()
    # the single-core figure of SURVEY §8(d), on the first two vertices of the sample
    set_threads(1)
    t1 = 0.0
    for p in probs[:2]:
        o = Oracle(p)
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        t1 += time.perf_counter() - t0
    set_threads(cores)
    return {"value": len(probs) / t, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
            "seconds": t, "value_1core": min(2, len(probs)) / t1}


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
    n_per_step = 1
    for k in range(args.warmup + args.steps):
        if args.workload == "C4":
            p = inputs.config4_vertex((k * 97) % B, B)
        else:
            p = inputs.CONFIGS[args.workload]()
        o = Oracle(p)
        f = o.coefficients()
        t0 = time.perf_counter()
        o.jacobian(f)
        dt = time.perf_counter() - t0
        if k >= args.warmup:
            times.append(dt)
    T = sum(times)
    value = n_per_step * len(times) / T
    N = 1088 if args.workload == "C4" else prob0.npoints
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * T / len(times),
            "higher_is_better": True, "scaling": "strong" if args.strong else "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic", "config": desc, "pairs_per_s": value * N * N,
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": get_threads(), "kind": "oracle",
                             "sample": f"1 vertex Jacobian per step ({args.workload}), full oracle"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


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
        # one large mesh: the mirror kernel's tile pairs split over the ranks, one NCCL all-reduce of
        # the partial G per build (the pair split; the element split + all-gather on non-mirror meshes)
        if world > 1:
            dist_desc = L.make_dist(L.LANDAU_DIST_ELEMENTS)
        else:
            dist_desc = {"rank": 0, "world": 1, "mode": L.LANDAU_DIST_ELEMENTS,
                         "nccl_unique_id": L.landau_nccl_unique_id()}
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
    # Per-stage library timers (CUDA events on the library stream) run inside the timed region for
    # large batches; small single builds replay as CUDA graphs, so their stage breakdown is taken in
    # a separate pass right after the timed region.
    in_loop_timers = args.workload in ("C4", "C5")
    h.set_timing(in_loop_timers)
    n0 = h.launch_count()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        for k in range(args.steps):
            flush.fill_(float(k))
            evs[k][0].record(stream)
            step()
            evs[k][1].record(stream)
        torch.cuda.synchronize()
    launches = h.launch_count() - n0
    st = h.stats()   # how the timed builds ran (read before the e2e pass changes the batch layout)
    if not in_loop_timers:
        h.set_timing(True)
        for k in range(args.steps):
            flush.fill_(float(k))
            step()
    tim = h.get_timing()
    h.set_timing(False)
    local_ms = sum(a.elapsed_time(b) for a, b in evs)
    t = torch.tensor([local_ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.barrier()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_ms = float(t.item())
    total_builds = job_vertices(args, world) if args.workload == "C4" else 1
    scaling = "strong" if (args.strong or args.workload != "C4") else "weak"
    ms_per_step = total_ms / args.steps
    value = total_builds / (ms_per_step / 1e3)
    pairs_per_build = N * N

    # ---- e2e through the host-pointer C-ABI entry point --------------------------------------
    f_pin = torch.tensor(F_host).pin_memory()
    v_pin = torch.empty((max(nloc, 1), h.nnz), dtype=torch.float64).pin_memory()
    for _ in range(min(args.warmup, 2)):
        if nloc:
            h.jacobian_host(f_pin, v_pin)
    e_ms = 0.0
    for k in range(args.steps):
        flush.fill_(float(k))
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        if nloc:
            h.jacobian_host(f_pin, v_pin)
        b.record(stream)
        torch.cuda.synchronize()
        e_ms += a.elapsed_time(b)
    et = torch.tensor([e_ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
    e2e_value = total_builds / (float(et.item()) / args.steps / 1e3)

    # ---- roofline of the dominant kernel (inner integral, FP64 pipe) --------------------------
    inner_ms, inner_n = tim["inner"]
    inner_avg_s = inner_ms / max(inner_n, 1) / 1e3
    if st["inner_path"] == 2:   # GEMMs: 2 FLOP per multiply-add, 7 N^2 per batch item (three DGEMMs)
        flop_per_pair = 14.0
        flops_per_launch = 14.0 * st["nbatch"] * N * N
    elif st["inner_path"] == 5:
        flop_per_pair = FLOP_PER_EVAL_MDIR
        flops_per_launch = flop_per_pair * st["nbatch"] * st["pair_evaluations"]
    elif st["inner_path"] in (3, 4):
        flop_per_pair = FLOP_PER_EVAL_VTX if st["inner_path"] == 4 else FLOP_PER_EVAL_MIRROR
        # (N/2)^2 U + V evaluations per batch item (+ the N/2 self-mirror pairs and tile padding); with
        # the pair split, this rank's share
        flops_per_launch = flop_per_pair * st["nbatch"] * st["pair_evaluations"]
    elif st["inner_path"] == 1:
        flop_per_pair = FLOP_PER_PAIR_SYMMETRIC
        flops_per_launch = flop_per_pair * st["nbatch"] * N * (N - 1) / 2
    else:
        flop_per_pair = FLOP_PER_PAIR_DIRECTED
        flops_per_launch = flop_per_pair * st["nbatch"] * st["targets"] * N
    achieved = flops_per_launch / inner_avg_s / 1e12 if inner_n else None
    clocks = clk.summary()
    props = torch.cuda.get_device_properties(local)
    sm_max = clocks["sm_max_mhz"] or 1965.0
    peak = fp64_peak_tflops(props, sm_max)
    step_ms_lib = sum(v[0] for v in tim.values()) / args.steps
    roof = {"bound": "alu", "kernel": "inner_vtx_kernel / inner_mir_kernel / inner_sym_kernel / inner_kernel (a-2, FP64 pipe)", "achieved": achieved, "peak": peak,
            "unit": "TFLOP/s", "frac": (achieved / peak) if achieved else None,
            "traffic": load_profile_traffic(args.workload),
            "fp64_pipe_active_ncu": load_profile_traffic(args.workload + "_fp64_pipe_active"),
            "peak_note": f"derived FP64 DFMA peak: {props.multi_processor_count} SMs x 64 lanes x 2 FLOP x {sm_max:.0f} MHz",
            "inner_path": ["directed (ordered pairs)", "symmetric (unordered pairs)",
                           "tensor cache + FP64 DGEMM (cuBLAS)",
                           "mirror-symmetric (one tensor per unordered pair and its z-mirror)",
                           "mirror-symmetric, one CTA per vertex (sums in shared memory)",
                           "mirror-symmetric directed (U + V per target and source, forward sums)"][st["inner_path"]],
            "flop_per_pair": flop_per_pair, "flops_per_launch": flops_per_launch,
            "inner_ms_per_launch": inner_avg_s * 1e3,
            "inner_share_of_step": (inner_ms / args.steps) / ms_per_step if ms_per_step else None,
            "pairs_per_s_inner": pairs_per_build * max(nloc, 1) / inner_avg_s * world if inner_n else None}
    stage_ms = {k: v[0] / args.steps for k, v in tim.items()}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(desc, parallelism=(f"element-split x{world}" if args.workload == "C5" else
                                              f"batch-shard x{world}") if world > 1 else "1 GPU"),
            "pairs_per_s": value * pairs_per_build, "roofline": roof, "stage_ms_per_step": stage_ms,
            "stage_timers": "in timed region" if in_loop_timers else "separate pass (graphs off)",
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(F_host.nbytes) * world,
                    "d2h_bytes_per_step": int(v_pin.numel() * 8) * world, "api": "landau_jacobian_host"},
            "gpu_launches": int(launches), "clocks": clocks}
    # NEXT-4 variant on the same job (informational; the headline above is the pairwise path)
    if args.workload == "C4" and not args.tensor_cache and nloc:
        try:
            h.set_tensor_cache(True)
            step()
            torch.cuda.synchronize()
            h.set_timing(True)
            vev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for k in range(args.steps):
                flush.fill_(float(k))
                vev[k][0].record(stream)
                step()
                vev[k][1].record(stream)
            torch.cuda.synchronize()
            vt = h.get_timing()
            h.set_timing(False)
            # the same GEMM formulation with the tensors re-evaluated inside every timed build
            h.set_tensor_cache("recompute")
            step()
            torch.cuda.synchronize()
            rev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for k in range(args.steps):
                flush.fill_(float(k))
                rev[k][0].record(stream)
                step()
                rev[k][1].record(stream)
            torch.cuda.synchronize()
            rms = torch.tensor([sum(a.elapsed_time(b) for a, b in rev)], dtype=torch.float64, device="cuda")
            h.set_tensor_cache(False)
            vms = torch.tensor([sum(a.elapsed_time(b) for a, b in vev)], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(vms, op=dist.ReduceOp.MAX)
            vstep = float(vms.item()) / args.steps
            if world > 1:
                dist.all_reduce(rms, op=dist.ReduceOp.MAX)
            rstep = float(rms.item()) / args.steps
            gemm_s = vt["inner"][0] / max(vt["inner"][1], 1) / 1e3
            line["variants"] = {"tensor_cache_gemm": {
                "value": total_builds / (vstep / 1e3), "unit": UNIT, "ms_per_step": vstep,
                "inner_ms_per_launch": gemm_s * 1e3,
                "inner_tflops": 14.0 * nloc * N * N / gemm_s / 1e12,
                "note": "SURVEY NEXT-4: mesh tensors cached once (7 N^2 doubles), inner integral as three FP64 "
                        "DGEMMs (cuBLAS, FP64 tensor cores); same sums up to order, parity-tested"},
                "tensor_gemm_recompute": {
                "value": total_builds / (rstep / 1e3), "unit": UNIT, "ms_per_step": rstep,
                "note": "the GEMM formulation with all N^2 tensors re-evaluated inside every timed build "
                        "(the batch shares one mesh): no state carried across builds"}}
        except Exception as e:   # the variant is optional: report why it did not run
            line["variants"] = {"tensor_cache_gemm": {"unavailable": str(e)[:200]}}
        # NEXT-4, the other variant: the inner integral with the 3D Cartesian tensor of Eq. 3
        # (landau3d_inner) on a 3D point set of the thermal-quench shape, 8^3 Q3 cubes (N = 32768)
        try:
            xyz3, w3 = inputs.points3d(8, 3)
            wTD3, wTK3 = inputs.fields3d(xyz3, w3)
            n3 = int(w3.size)
            X3, D3, K3 = (torch.tensor(a, device="cuda") for a in (xyz3, wTD3, wTK3))
            G3 = torch.empty((9, n3), dtype=torch.float64, device="cuda")
            for _ in range(2):
                L.landau3d_inner(X3, D3, K3, G3, stream)
            ev3 = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for k in range(args.steps):
                ev3[k][0].record(stream)
                L.landau3d_inner(X3, D3, K3, G3, stream)
                ev3[k][1].record(stream)
            torch.cuda.synchronize()
            ms3 = sum(a.elapsed_time(b) for a, b in ev3) / args.steps
            line.setdefault("variants", {})["inner3d_cartesian"] = {
                "value": n3 * n3 / (ms3 * 1e-3), "unit": "pairs/s",
                "points": n3, "ms_per_launch": ms3,
                "tflops": FLOP_PER_PAIR_3D * n3 * n3 / (ms3 * 1e-3) / 1e12,
                "frac_of_fp64_peak": FLOP_PER_PAIR_3D * n3 * n3 / (ms3 * 1e-3) / 1e12 / peak,
                "note": "SURVEY NEXT-4: G_D, G_K with U = (|u|^2 I - u u^T)/|u|^3 directly (no elliptic integrals), "
                        "ordered pairs, parity-tested against oracle O12"}
        except Exception as e:
            line.setdefault("variants", {})["inner3d_cartesian"] = {"unavailable": str(e)[:200]}
    # NEXT-3: quasi-Newton backward-Euler iterations on the same batch (the paper's figure of merit,
    # "Newton iterations per second", @37187): per iteration set_state + Jacobian + band LU + solve
    if args.workload == "C4" and not args.tensor_cache and nloc:
        try:
            it_per_call = 2
            Fn = torch.empty_like(F)
            for _ in range(2):
                h.implicit_step_batched(0.002, F, Fn, max_iter=it_per_call, rtol=0.0)
            torch.cuda.synchronize()
            h.set_timing(True)
            nev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for k in range(args.steps):
                flush.fill_(float(k))
                nev[k][0].record(stream)
                h.implicit_step_batched(0.002, F, Fn, max_iter=it_per_call, rtol=0.0)
                nev[k][1].record(stream)
            torch.cuda.synchronize()
            nt = h.get_timing()
            h.set_timing(False)
            nms = torch.tensor([sum(a.elapsed_time(b) for a, b in nev)], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(nms, op=dist.ReduceOp.MAX)
            ms_it = float(nms.item()) / (args.steps * it_per_call)
            line["newton"] = {
                "value": total_builds / (ms_it / 1e3), "unit": "vertex Newton iterations/s", "ms_per_iteration": ms_it,
                "stage_ms_per_iteration": {k: v[0] / (args.steps * it_per_call) for k, v in nt.items()},
                "note": "SURVEY NEXT-3: backward-Euler step by quasi-Newton (Jacobian about each iterate, A = M/dt - J "
                        "factored by the RCM band LU, solve), all vertices of the job per iteration, dt = 0.002, "
                        f"{it_per_call} iterations per landau_implicit_step_batched call; context: the paper's V100 "
                        "node figure is a different problem (10 species, 80 cells, CPU LU)"}
        except Exception as e:
            line["newton"] = {"unavailable": str(e)[:200]}
    # configs[1] itself (one C2 grid, one build per step; launch-latency regime, CUDA-graph replay)
    if args.workload == "C4" and rank == 0:
        try:
            p2 = inputs.config2()
            h2 = L.Landau.from_problem(p2, device=local, stream=stream)
            f2 = torch.tensor(inputs.coefficients(p2, h2.all_nodes()), device="cuda")
            v2 = torch.empty(h2.nnz, dtype=torch.float64, device="cuda")
            m2 = torch.empty(h2.nnz, dtype=torch.float64, device="cuda")
            for _ in range(max(args.warmup, 3)):
                h2.set_state(f2)
                h2.jacobian(v2)
                h2.mass(shift, m2)
            torch.cuda.synchronize()
            ev2 = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
            for k in range(args.steps):
                flush.fill_(float(k))
                ev2[k][0].record(stream)
                h2.set_state(f2)
                h2.jacobian(v2)
                h2.mass(shift, m2)
                ev2[k][1].record(stream)
            torch.cuda.synchronize()
            ms2 = sum(a.elapsed_time(b) for a, b in ev2) / args.steps
            line["c2_single_build"] = {"value": 1e3 / ms2, "unit": UNIT, "ms_per_step": ms2,
                                       "pairs_per_s": 1e3 / ms2 * p2.npoints ** 2,
                                       "inner_path": ["directed", "symmetric", "tensor cache", "mirror", "mirror per-vertex", "mirror directed"][h2.stats()["inner_path"]],
                                       "note": "BASELINE configs[1]: one e+D Q3 AMR grid (N=1088) per step, "
                                               "set_state + jacobian (CSR) + mass, CUDA-graph replay"}
            h2.close()
        except Exception as e:
            line["c2_single_build"] = {"unavailable": str(e)[:200]}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        ns = args.cpu_sample or (8 if args.workload == "C4" else 1)
        line["cpu_baseline"] = cpu_baseline(args, desc, ns)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
