"""Per-source-line instruction counts and stall samples of one kernel in an ncu report.
    python tools/ncu_lines.py REPORT.ncu-rep [kernel-name-substring] [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
want = sys.argv[2] if len(sys.argv) > 2 else ""
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, keep = [], True
for r in csv.reader(io.StringIO(txt)):       # one section per kernel: keep the wanted one
    if r and r[0] == "Function Name":
        keep = want in r[1]
        print("#", r[1], "(selected)" if keep else "")
    if keep:
        rows.append(r)
hdr = next(r for r in rows if r and r[0] == "Line No")
ie = hdr.index("Instructions Executed")
ss = hdr.index("Warp Stall Sampling (All Samples)")
per, tot, tots = [], 0, 0
for r in rows:
    if len(r) > ie and r[0] and r[0] != "Line No" and r[ie] not in ("-", ""):
        try:
            n, s = int(r[ie]), int(r[ss])
        except ValueError:
            continue
        tot += n
        tots += s
        per.append((n, s, r[0], r[1][:95]))
print(f"total instructions {tot/1e6:.1f}M  stall samples {tots}")
for n, s, line, src in sorted(per, reverse=True)[:top]:
    print(f"{n/1e6:9.1f}M {100*s/max(tots,1):5.1f}% L{line:>5} {src}")
