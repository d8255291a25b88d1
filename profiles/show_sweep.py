"""Print one summary line per bench JSON: python profiles/show_sweep.py gpurun_out/<tag>_*.json"""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "unreadable", e)
        continue
    ks = {k.replace("_tiles", "").replace("_rows", ""): round(v["avg_ms"], 3) for k, v in d.get("kernels", {}).items()}
    r = d.get("roofline", {})
    print(f"{f.split('/')[-1]:45s} step {d['ms_per_step']:.3f} ms {d['value']:8.0f} {d['unit']} {ks} "
          f"roof {r.get('kernel')} {r.get('frac', 0):.3f}")
