"""Extract per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) of libsr's
kernels from an `ncu --set full ... --page raw --csv` export and merge it into
profiles/ncu_traffic.json, keyed "<config>_K<K>_<kernel kind>" (bench.py reads it into the
roofline `traffic` field).

  python profiles/ncu_traffic.py <raw.csv> <config> <K> [source-tag] [kernel-sig]

kernel-sig is bench.kernel_source_sig() of the sources the capture ran (write it on the GPU box
next to the capture); bench.py uses a record only when it matches the current sources.
"""
import csv
import json
import os
import sys

KINDS = {"spmm_dense_kernel": "spmm_dense_tiles", "spmm_sparse_kernel": "spmm_sparse_rows",
         "spmm_task_kernel": "spmm_sparse_rows", "sddmm_dense_kernel": "sddmm_dense_tiles",
         "sddmm_sparse_kernel": "sddmm_sparse_rows", "sddmm_task_kernel": "sddmm_sparse_rows",
         "spmm_rtile_kernel": "spmm_register_tiles", "sddmm_rtile_kernel": "sddmm_register_tiles"}
UNIT = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def main(path, config, K, tag="", sig=None):
    rows = list(csv.reader(open(path)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ix = {h: i for i, h in enumerate(hdr)}
    out_path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "ncu_traffic.json")
    table = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for d in data:
        name = d[ix["Kernel Name"]]
        kind = next((v for k, v in KINDS.items() if k in name), None)
        if kind is None:
            continue
        total = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            total += float(d[ix[m]]) * UNIT[units[ix[m]]]
        t = float(d[ix["gpu__time_duration.sum"]]) * {"nsecond": 1e-9, "ns": 1e-9, "usecond": 1e-6, "us": 1e-6,
                                                       "msecond": 1e-3, "ms": 1e-3}[units[ix["gpu__time_duration.sum"]]]
        rec = {"bytes": total, "ncu_duration_s": t, "source": tag or os.path.basename(path)}
        if sig:
            rec["kernel_sig"] = sig
        for m, key in (("lts__t_sector_hit_rate.pct", "l2_hit_pct"), ("l1tex__t_sector_hit_rate.pct", "l1_hit_pct")):
            if m in ix and d[ix[m]] not in ("", "n/a"):
                rec[key] = float(d[ix[m]])
        table[f"{config}_K{K}_{kind}"] = rec
    json.dump(table, open(out_path, "w"), indent=1, sort_keys=True)
    print(json.dumps(table, indent=1))


if __name__ == "__main__":
    main(*sys.argv[1:])
