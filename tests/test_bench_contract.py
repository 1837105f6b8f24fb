"""bench.py contract checks that need no GPU: the reference arm (the oracle, this tier's reference)
prints one JSON line with the driver's keys on the same metric/config as the GPU arm."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "0"], capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "builds/s" and d["dtype"] == "f64"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"].startswith("C4")


def test_reference_arm_other_ranks_exit_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2", LOCAL_RANK="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "0"], capture_output=True, text=True, timeout=120, cwd=ROOT, env=env)
    assert out.returncode == 0 and out.stdout.strip() == ""


def test_c4_sharding_strong_and_weak():
    """C4 vertices are independent problems: by default a fixed job of --batch vertices (BASELINE
    configs[3]: 1024) is split over the ranks (strong scaling); --weak gives every rank its own --batch
    vertices.  The ranks' vertex ranges are disjoint and cover the job, and world 1 is the same batch
    either way."""
    sys.path.insert(0, ROOT)
    import bench
    for weak, world, job in ((False, 1, 16), (False, 2, 16), (False, 4, 16), (True, 1, 16), (True, 2, 32)):
        args = bench.parse(["--batch", "16"] + (["--weak"] if weak else []))
        assert bench.job_vertices(args, world) == job
        seen = []
        for rank in range(world):
            desc, _, items = bench.workload(args, world, rank)
            assert desc["vertices"] == job and len(items) == job // world
            seen += [it.seed for it in items]
        assert sorted(seen) == [20220 + b for b in range(job)]
    assert bench.parse([]).batch == 1024 and not bench.parse([]).weak


def test_clock_region_filter_and_handshake():
    """Clocks keeps only the samples taken inside the timed region (mark_start/mark_end) and falls
    back to all samples when the region saw none."""
    sys.path.insert(0, ROOT)
    import bench
    c = bench.Clocks(0)
    c.source = "nvml"
    row = lambda sm: ["0", str(sm), "1965", "", "0x0", "Not Active", "Not Active", "Not Active", "Not Active"]
    c.rows = [row(1000), row(1965), row(1965), row(1200)]
    c.times = [0.0, 10.0, 10.5, 20.0]
    c.t0, c.t1 = 9.9, 10.6
    s = c.summary()
    assert s["samples"] == 2 and s["sm_mhz"] == 1965.0
    c.t0, c.t1 = 30.0, 31.0
    assert c.summary()["samples"] == 4


def test_clock_summary_decodes_nvml_reason_bits():
    """The clocks key: NVML clock-event reason bits (nvml.h: sw_power_cap 0x4, hw_slowdown 0x8,
    sw_thermal_slowdown 0x20, hw_thermal_slowdown 0x40) become the reasons the driver rejects or notes;
    the SM clock is the median over samples, the max clock the largest reported."""
    sys.path.insert(0, ROOT)
    import bench
    c = bench.Clocks(0)
    B = bench.Clocks.NVML_BITS

    def row(sm, bits):
        return ["0", str(sm), "1965", "", hex(bits)] + [
            "Active" if bits & B[k] else "Not Active"
            for k in ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")]

    c.rows = [row(1965, 0), row(1900, B["sw_power_cap"]), row(1965, 0x1)]   # 0x1 = GPU idle: not a reason
    c.source = "nvml"
    s = c.summary()
    assert s == {"sm_mhz": 1965.0, "sm_max_mhz": 1965.0, "reasons": ["sw_power_cap"], "samples": 3,
                 "source": "nvml"}
    c.rows = [row(1200, B["hw_thermal_slowdown"] | B["hw_slowdown"]), row(1300, B["sw_thermal_slowdown"])]
    assert c.summary()["reasons"] == ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"]
    assert c.summary()["sm_mhz"] == 1250.0
