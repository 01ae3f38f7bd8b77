import json, glob, os
for f in sorted(glob.glob("gpurun_out/qp_*.json")):
    c = os.path.basename(f)[3:-5]
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        r = d.get("roofline", {})
        print(c, "GFLOP/s", d["value"], "ms", d["ms_per_step"], "frac", r.get("frac"), "units", d["config"].get("num_units"), "U", d["config"].get("unit_blocks"))
    except Exception as e:
        print(c, "ERR", open(f.replace(".json", ".err")).read()[-1500:])
