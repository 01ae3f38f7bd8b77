import json, glob, os, collections
res = collections.defaultdict(dict)
par = {}
for f in sorted(glob.glob("gpurun_out/vs_*_parity.txt")):
    v = os.path.basename(f)[3:-len("_parity.txt")]
    par[v] = open(f).read().strip()
for f in sorted(glob.glob("gpurun_out/vs_*.json")):
    b = os.path.basename(f)[3:-5]
    v, c = b.rsplit("_", 1)
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        res[v][c] = d["value"]
    except Exception:
        res[v][c] = "ERR"
cfgs = sorted({c for r in res.values() for c in r})
print("variant".ljust(22), *[c.rjust(9) for c in cfgs], "  parity")
for v, r in res.items():
    print(v.ljust(22), *[str(r.get(c, "-")).rjust(9) for c in cfgs], "  ", par.get(v, "?"))
