"""Key ncu metrics per kernel from a `--page details --csv` export, plus the instruction mix
and top stall reasons from the matching `--page source --csv` export (if present).
  python profiles/ncu_summary.py gpurun_out/ncu_<tag>_details.csv [gpurun_out/ncu_<tag>_source.csv.gz]"""
import collections
import csv
import gzip
import sys

WANT = ["Duration", "DRAM Throughput", "L2 Cache Throughput", "L1/TEX Cache Throughput", "L2 Hit Rate",
        "Achieved Active Warps Per SM", "Issued Warp Per Scheduler", "Warp Cycles Per Issued Instruction",
        "Registers Per Thread", "Dynamic Shared Memory Per Block", "Grid Size"]
rows = list(csv.reader(open(sys.argv[1])))
h = rows[0]
ki, mn, mv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
seen = collections.OrderedDict()
for r in rows[1:]:
    if r[mn] in WANT:
        seen.setdefault(r[ki][:60], {})[r[mn]] = r[mv]
for k, d in seen.items():
    print(k)
    print("   " + ", ".join(f"{m}={d[m]}" for m in WANT if m in d))
if len(sys.argv) > 2:
    p = sys.argv[2]
    f = gzip.open(p, "rt") if p.endswith(".gz") else open(p)
    rows = list(csv.reader(f))
    i = 0
    while i < len(rows):
        r = rows[i]
        if r and r[0] == "Kernel Name":
            name, hdr, j, body = r[1], rows[i + 1], i + 2, []
            while j < len(rows) and rows[j] and rows[j][0] != "Kernel Name":
                body.append(rows[j])
                j += 1
            ie, src = hdr.index("Instructions Executed"), hdr.index("Source")
            c, tot = collections.Counter(), 0
            for b in body:
                n = int(b[ie]) if b[ie].isdigit() else 0
                t = b[src].split()
                op = (t[1] if t and t[0].startswith("@") and len(t) > 1 else (t[0] if t else "")).split(".")[0]
                c[op] += n
                tot += n
            print(name[:70], "warp instrs", tot, "sass", len(body))
            print("   " + ", ".join(f"{k}:{v / tot * 100:.1f}%" for k, v in c.most_common(14)))
            i = j
        else:
            i += 1
