"""Top SASS instructions by warp-stall samples from an `ncu --page source --csv` export."""
import csv, gzip, sys
path = sys.argv[1]
want = sys.argv[2] if len(sys.argv) > 2 else ""
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
f = gzip.open(path, "rt") if path.endswith(".gz") else open(path)
rows = list(csv.reader(f))
i = 0
while i < len(rows):
    r = rows[i]
    if r and r[0] == "Kernel Name":
        name = r[1]
        hdr = rows[i + 1]
        j = i + 2
        body = []
        while j < len(rows) and rows[j] and rows[j][0] != "Kernel Name":
            body.append(rows[j]); j += 1
        if want in name:
            si = hdr.index("Warp Stall Sampling (All Samples)")
            tot = sum(int(b[si]) for b in body if b[si].isdigit())
            print("=====", name[:110], "total samples", tot)
            idx = sorted(range(len(body)), key=lambda k: -int(body[k][si]) if body[k][si].isdigit() else 0)
            for k in idx[:top]:
                b = body[k]
                print(f"{int(b[si]) / max(tot, 1) * 100:5.1f}%  {k:5d} {b[1].strip()[:90]}")
        i = j
    else:
        i += 1
