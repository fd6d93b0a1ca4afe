#!/usr/bin/env python
"""Per-source-line samples of one stall reason (default long_sb) from an ncu report.
Usage: ncu_stalls.py rep.ncu-rep [reason] [n_top]"""
import csv
import io
import subprocess
import sys


def main(rep, reason="stall_long_sb", ntop=25):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    hdr, fname, rows = None, "", []
    for r in csv.reader(io.StringIO(out)):
        if len(r) == 2 and r[0] == "File Path":
            fname = r[1].split("/")[-1]
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr) or not r[0]:
            continue
        x = dict(zip(hdr, r))
        try:
            rows.append((int(x[reason] or 0), fname, int(r[0]), r[1].strip()[:100]))
        except (ValueError, KeyError):
            pass
    tot = sum(r[0] for r in rows) or 1
    print(f"{reason}: total samples {tot}")
    for v, f, ln, src in sorted(rows, reverse=True)[:ntop]:
        print(f"{100 * v / tot:5.1f}%  {f}:{ln:<5d} {src}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "stall_long_sb", int(sys.argv[3]) if len(sys.argv) > 3 else 25)
