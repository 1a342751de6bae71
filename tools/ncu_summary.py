#!/usr/bin/env python
"""Summarise an ncu --set full report of the update kernel: key section metrics and the
source lines with the most warp-stall samples.  Usage: tools/ncu_summary.py report.ncu-rep [N]"""
import csv
import io
import subprocess
import sys

KEYS = [
    "Duration", "Elapsed Cycles", "SM Active Cycles", "Memory Throughput", "DRAM Throughput",
    "L1/TEX Cache Throughput", "L2 Cache Throughput", "Compute (SM) Throughput",
    "Executed Ipc Active", "Issue Slots Busy", "Registers Per Thread", "Grid Size", "Block Size",
    "Dynamic Shared Memory Per Block", "Achieved Active Warps Per SM", "Eligible Warps Per Scheduler",
    "Warp Cycles Per Issued Instruction", "Executed Instructions", "L2 Hit Rate", "L1/TEX Hit Rate",
]


def ncu(args):
    return subprocess.run(["ncu"] + args, capture_output=True, text=True).stdout


def main():
    rep = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    det = list(csv.reader(io.StringIO(ncu(["-i", rep, "--page", "details", "--csv"]))))
    hdr = det[0]
    im, iu, iv = hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
    ik = hdr.index("Kernel Name")
    print("kernel:", det[1][ik][:100])
    for r in det[1:]:
        if r[im] in KEYS:
            print(f"  {r[im]:40s} {r[iv]:>16s} {r[iu]}")
    raw = list(csv.reader(io.StringIO(ncu(["-i", rep, "--page", "raw", "--csv"]))))
    h, u, v = raw[0], raw[1], raw[2]
    for name in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
                 "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
                 "smsp__inst_executed.sum", "sm__cycles_elapsed.avg"):
        if name in h:
            i = h.index(name)
            print(f"  {name:40s} {v[i]:>16s} {u[i]}")
    src = list(csv.reader(io.StringIO(ncu(["-i", rep, "--page", "source", "--csv",
                                           "--print-source", "cuda,sass"]))))
    hh = src[2]
    i_s = hh.index("Warp Stall Sampling (All Samples)")
    i_i = hh.index("Instructions Executed")
    stalls = [x for x in hh if x.startswith("stall_") and "Not Issued" not in x]
    agg, ts, ti = [], 0, 0
    for r in src[3:]:
        if len(r) <= max(i_s, i_i) or not r[0]:
            continue
        try:
            s = int(r[i_s]) if r[i_s] not in ("-", "") else 0
            n = int(r[i_i]) if r[i_i] not in ("-", "") else 0
        except ValueError:
            continue
        st = {x: int(r[hh.index(x)]) for x in stalls if r[hh.index(x)] not in ("-", "")}
        agg.append((s, n, r[0], r[1][:80], st))
        ts += s
        ti += n
    print(f"  stall samples {ts}, instructions {ti}")
    for s, n, ln, code, st in sorted(agg, reverse=True)[:top]:
        t3 = ", ".join(f"{k[6:]}={v}" for k, v in sorted(st.items(), key=lambda x: -x[1])[:3])
        print(f"  {100 * s / max(ts, 1):5.1f}% inst {n:11d} L{ln:>4} {code:80s} {t3}")


if __name__ == "__main__":
    main()
