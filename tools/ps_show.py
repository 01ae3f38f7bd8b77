import json, glob, os, collections, sys
pre = sys.argv[1] if len(sys.argv) > 1 else "ps"
res = collections.defaultdict(dict)
for f in sorted(glob.glob(f"gpurun_out/{pre}_*.json")):
    b = os.path.basename(f)[len(pre) + 1:-5]
    v, c = b.rsplit("_", 1)
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        res[v][c] = d["value"]
    except Exception:
        res[v][c] = "ERR"
cfgs = sorted({c for r in res.values() for c in r})
print("variant".ljust(22), *[c.rjust(9) for c in cfgs])
for v, r in res.items():
    print(v.ljust(22), *[str(r.get(c, "-")).rjust(9) for c in cfgs])
