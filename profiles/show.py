import json, sys
for tag in sys.argv[1:]:
    d = json.loads(open(f"/root/repo/gpurun_out/{tag}.json").read().strip().splitlines()[-1])
    print(tag, "value", round(d["value"], 1), "ms/step", round(d["ms_per_step"], 3), json.dumps(d["per_op_gflops"]))
    for k, v in d["kernels"].items():
        print("  ", k, round(v["avg_ms"], 3), "ms", round(v["achieved_gbs"], 1), "GB/s")
