#!/usr/bin/env python
"""Per-CUDA-source-line warp instructions executed and stall samples from an ncu report
(--import-source on, -lineinfo).  Usage: ncu_lines.py rep.ncu-rep [n_top] [units]
`units` (e.g. packets/32 = warp chunks) normalises instruction counts per unit."""
import csv
import io
import subprocess
import sys


def main(rep, ntop=40, units=0.0):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = None
    lines = []
    fname = ""
    for r in rows:
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr) or not r[0]:
            continue
        x = dict(zip(hdr, r))
        try:
            lines.append((fname, int(r[0]), r[1].strip()[:90], int(x["Instructions Executed"] or 0),
                          int(x["Warp Stall Sampling (All Samples)"] or 0)))
        except (ValueError, KeyError):
            pass
    tot_i = sum(l[3] for l in lines) or 1
    tot_s = sum(l[4] for l in lines) or 1
    print(f"total warp instructions {tot_i}" + (f"  = {tot_i / units:.1f} per unit" if units else ""))
    for f, ln, src, ie, st in sorted(lines, key=lambda l: -l[3])[:ntop]:
        per = f"{ie / units:8.1f}" if units else ""
        print(f"{100 * ie / tot_i:5.1f}% {per} stall {100 * st / tot_s:5.1f}%  {f}:{ln:<5d} {src}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40, float(sys.argv[3]) if len(sys.argv) > 3 else 0.0)
