#!/usr/bin/env python3
"""Key metrics of one kernel from an ncu report (ncu -i REP --page raw --csv)."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__issue_active.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "sm__sass_thread_inst_executed_op_dfma_pred_on.sum", "sm__sass_thread_inst_executed_op_dmul_pred_on.sum",
        "sm__sass_thread_inst_executed_op_dadd_pred_on.sum", "sm__sass_thread_inst_executed_op_fp64_pred_on.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]
STALL = "smsp__average_warps_issue_stalled_"


def main(rep, pairs=None):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        name = vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"
        print(f"# kernel: {name}")
        for k in KEYS:
            if k in hdr:
                print(f"{k:75s} {vals[hdr.index(k)]:>22s} {units[hdr.index(k)]}")
        st = [(h, float(vals[i])) for i, h in enumerate(hdr)
              if h.startswith(STALL) and h.endswith("_per_issue_active.ratio") and vals[i] not in ("", "n/a")]
        st.sort(key=lambda t: -t[1])
        print("# top stall reasons (warps per issue-active cycle)")
        for h, v in st[:8]:
            print(f"  {h[len(STALL):-len('_per_issue_active.ratio')]:30s} {v:8.3f}")
        if pairs:
            i = hdr.index("sm__sass_thread_inst_executed_op_dfma_pred_on.sum") if "sm__sass_thread_inst_executed_op_dfma_pred_on.sum" in hdr else None
            if i is not None:
                f = lambda k: float(vals[hdr.index(k)].replace(",", ""))
                dfma, dmul, dadd = (f(f"sm__sass_thread_inst_executed_op_{o}_pred_on.sum") for o in ("dfma", "dmul", "dadd"))
                print(f"# per pair ({pairs:.4g} pairs): DFMA {dfma/pairs:.2f} DMUL {dmul/pairs:.2f} DADD {dadd/pairs:.2f} "
                      f"FLOP {(2*dfma+dmul+dadd)/pairs:.2f} FP64 instr {(dfma+dmul+dadd)/pairs:.2f}")


if __name__ == "__main__":
    main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else None)
