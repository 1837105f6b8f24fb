#!/usr/bin/env python3
"""Per-CUDA-source-line warp-stall samples of one kernel from an ncu report (compile with -lineinfo,
capture with --import-source on):  python tools/ncu_source_hot.py REP KERNEL_REGEX [TOP]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def main(rep, kernel, top=25):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kernel}", "--print-source",
                          "cuda,sass"], capture_output=True, text=True).stdout
    acc = defaultdict(float)
    src = {}
    fname = "?"
    hdr = None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] in ("File Path", "File Name"):
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < 5 or not r[0].isdigit():
            continue
        key = (fname, int(r[0]))
        src[key] = r[1]
        try:
            acc[key] += float(r[4] or 0)
        except ValueError:
            pass
    tot = sum(acc.values()) or 1.0
    for key, v in sorted(acc.items(), key=lambda t: -t[1])[:top]:
        print(f"{v / tot * 100:6.2f}%  {key[0]}:{key[1]:<5d} {src[key].strip()[:130]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 25)
