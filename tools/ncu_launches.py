#!/usr/bin/env python3
"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list per kernel (share of time)."""
import collections
import csv
import sys


def main(path, step_kernels=None, nstep=3):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr, data = rows[hi], rows[hi + 1:]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in data:
        if len(r) <= vi:
            continue
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}.get(r[ui], 1.0)
        name = r[ki].split("(")[0].replace("(anonymous namespace)::", "")
        agg.setdefault(name, []).append(float(r[vi].replace(",", "")) * scale)
    if step_kernels:   # the headline step: the first nstep launches of each of its kernels (it runs first)
        print(f"{'kernel':48s} {'launches':>8s} {'mean_us':>10s} {'share of step':>14s}")
        sel = {k: v[:nstep] for k, v in agg.items() if any(s in k for s in step_kernels)}
        step = sum(sum(v) / len(v) for v in sel.values())
        for k, v in sorted(sel.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
            print(f"{k:48s} {len(v):8d} {sum(v)/len(v):10.2f} {100*sum(v)/len(v)/step:13.1f}%")
        print(f"{'step (sum of means)':48s} {'':8s} {step:10.2f}\n")
    tot = sum(sum(v) for v in agg.values())
    print(f"{'kernel':48s} {'launches':>8s} {'total_us':>12s} {'mean_us':>10s} {'share':>7s}")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"{k:48s} {len(v):8d} {sum(v):12.1f} {sum(v)/len(v):10.2f} {100*sum(v)/tot:6.1f}%")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2].split(",") if len(sys.argv) > 2 else None)
