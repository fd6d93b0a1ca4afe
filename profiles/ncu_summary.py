#!/usr/bin/env python
"""Summarise an ncu --set full capture of sfc_kernel: SOL, occupancy, stalls, DRAM bytes,
and the top SASS lines by warp-stall samples.  Usage: ncu_summary.py rep.ncu-rep [n_top]"""
import csv
import io
import subprocess
import sys


def ncu(*args):
    return subprocess.run(["ncu", "-i", *args], capture_output=True, text=True).stdout


def main(rep, ntop=25):
    raw = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    hdr, units, vals = raw[0], raw[1], raw[2]
    d = dict(zip(hdr, vals))
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
            "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "launch__grid_size", "launch__block_size", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__inst_executed.sum", "smsp__inst_executed.avg.per_cycle_active",
            "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
            "l1tex__t_sector_hit_rate.pct", "launch__shared_mem_per_block_dynamic"]
    out = []
    for k in keys:
        if k in d:
            u = units[hdr.index(k)]
            out.append(f"{k:70s} {d[k]:>16s} {u}")
    st = [(h.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""), float(v or 0))
          for h, v in zip(hdr, vals) if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio")]
    st.sort(key=lambda x: -x[1])
    out.append("warp stall reasons (cycles per issued instruction):")
    out += [f"  {n:40s} {v:8.3f}" for n, v in st[:10]]
    src = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source", "sass"))))
    h2 = src[1]
    rows = []
    for r in src[2:]:
        if len(r) < len(h2):
            continue
        x = dict(zip(h2, r))
        try:
            rows.append((int(x["Warp Stall Sampling (All Samples)"]), int(x["Instructions Executed"] or 0),
                         x["Address"][-5:], x["Source"].strip()[:70]))
        except ValueError:
            pass
    tot = sum(r[0] for r in rows) or 1
    out.append(f"top SASS by stall samples (total {tot}):")
    for s, ie, a, src_ in sorted(rows, key=lambda r: -r[0])[:ntop]:
        out.append(f"  {100 * s / tot:5.1f}%  exec={ie:11d}  {a}  {src_}")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
