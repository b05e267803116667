"""Table 3 analogue: whole-run L2 read / write accesses of the four
pointer-jumping variants, relative to Jump4 (ECL-CC's intermediate pointer jumping), and
Jump4's read:write ratio (the paper: 8.82).

Collect (one ncu process per config and variant, all of our kernels of one run):
    ncu --metrics lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,\
lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,lts__t_requests_op_read.sum,\
lts__t_requests_op_write.sum --clock-control none --csv --log-file OUT/l2rw_<C>_J<j>.csv \
        python tools/prof.py --config <C> --reps 1 --jump <j>
then summarise:
    python tools/table3.py OUT
"""
import csv
import glob
import json
import os
import re
import sys
from collections import defaultdict


def load(path):
    tot = defaultdict(float)
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for row in csv.DictReader(lines):
        try:
            tot[row["Metric Name"]] += float(row["Metric Value"].replace(",", ""))
        except (KeyError, ValueError):
            pass
    return tot


def main():
    d = sys.argv[1]
    data = defaultdict(dict)
    for p in glob.glob(os.path.join(d, "l2rw_*_J*.csv")):
        m = re.search(r"l2rw_(C\d)_J(\d|p)\.csv$", p)
        if m:
            j = m.group(2)
            data[m.group(1)][0 if j == "p" else int(j)] = load(p)
    out = {}
    for c in sorted(data):
        j4 = data[c].get(4)
        if not j4:
            continue
        rd = lambda t: t["lts__t_sectors_op_read.sum"]  # noqa: E731
        wr = lambda t: t["lts__t_sectors_op_write.sum"]  # noqa: E731
        row = {"jump4_read_sectors": rd(j4), "jump4_write_sectors": wr(j4),
               "jump4_atom_sectors": j4.get("lts__t_sectors_op_atom.sum", 0.0),
               "jump4_read_per_write": round(rd(j4) / max(wr(j4), 1), 2)}
        for j in (1, 2, 3):
            if j in data[c]:
                row[f"Jump{j}_read_rel"] = round(rd(data[c][j]) / rd(j4), 3)
                row[f"Jump{j}_write_rel"] = round(wr(data[c][j]) / max(wr(j4), 1), 3)
        jp = data[c].get(0)      # Jump4 on the plain path (batch 0): Jump1-3's own path
        if jp:
            row["jump4_plain_read_per_write"] = round(rd(jp) / max(wr(jp), 1), 2)
            for j in (1, 2, 3):
                if j in data[c]:
                    row[f"Jump{j}_read_rel_plain"] = round(rd(data[c][j]) / rd(jp), 3)
                    row[f"Jump{j}_write_rel_plain"] = round(wr(data[c][j]) / max(wr(jp), 1), 3)
        out[c] = row
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
