"""Summarise an ncu report: key SOL metrics + top stall source lines (CUDA source view)."""
import csv
import io
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Memory Throughput",
        "Eligible Warps Per Scheduler", "Issued Warp Per Scheduler", "Achieved Occupancy",
        "Registers Per Thread", "L2 Cache Throughput", "L1/TEX Cache Throughput",
        "Executed Instructions", "Avg. Active Threads Per Warp"]


KFILTER = []


def run(args):
    return subprocess.run(["ncu", "-i"] + args + KFILTER, capture_output=True, text=True).stdout


def main(rep, top=25):
    det = list(csv.reader(io.StringIO(run([rep, "--page", "details", "--csv"]))))
    hdr = det[0]
    ki = hdr.index("Kernel Name")
    ni, ui, vi = hdr.index("Metric Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
    for r in det[1:]:
        if r[ni] in KEYS:
            print(f"{r[ki][:40]:40s} {r[ni]:32s} {r[vi]:>14s} {r[ui]}")
    raw = list(csv.reader(io.StringIO(run([rep, "--page", "raw", "--csv"]))))
    h, units, vals = raw[0], raw[1], raw[2:]
    for want in ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors.sum",
                 "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_read.sum",
                 "lts__t_sectors_op_write.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
                 "l1tex__t_sector_hit_rate.pct", "gpu__time_duration.sum"]:
        if want in h:
            i = h.index(want)
            for v in vals:
                print(f"  {want:50s} {v[i]:>16s} {units[i]}")
    src = list(csv.reader(io.StringIO(run([rep, "--page", "source", "--csv", "--print-source",
                                           "cuda,sass"]))))
    # rows after the header: "Line No","Source"(cuda),"Address","Source"(sass), metrics...
    # a CUDA line row carries the line's code; following sass rows have an empty line no.
    hdr2 = None
    agg = {}
    code = {}
    cur = None
    for r in src:
        if len(r) > 4 and r[0] == "Line No":
            hdr2 = r
            si = hdr2.index("Warp Stall Sampling (All Samples)")
            ei = hdr2.index("Instructions Executed")
            continue
        if hdr2 is None or len(r) < len(hdr2):
            continue
        if r[0]:
            cur = int(r[0])
            code[cur] = r[1]
        try:
            s = float(r[si] or 0)
            e = float(r[ei] or 0)
        except ValueError:
            continue
        if r[2] and cur is not None:   # sass row
            a = agg.setdefault(cur, [0.0, 0.0])
            a[0] += s
            a[1] += e
    tot = sum(a[0] for a in agg.values()) or 1
    for ln, (s, e) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{100*s/tot:5.1f}%  inst={e:12.0f}  L{ln:>4}  {code.get(ln, '').strip()[:90]}")

if __name__ == "__main__":
    # python tools/ncu_summary.py REPORT [TOP] [KERNEL_REGEX]
    if len(sys.argv) > 3:
        KFILTER[:] = ["-k", "regex:" + sys.argv[3]]
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
