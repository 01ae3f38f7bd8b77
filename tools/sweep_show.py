"""Print value (GFLOP/s) of bench JSON lines matching a glob: python tools/sweep_show.py 'gpurun_out/pp*_c2.json'"""
import glob
import json
import sys

for pat in sys.argv[1:]:
    for f in sorted(glob.glob(pat)):
        try:
            d = json.loads(open(f).read().strip().splitlines()[-1])
            print(f"{f:50s} {d['value']:10.1f} GFLOP/s  frac {d.get('roofline', {}).get('frac')}  "
                  f"units {d['config'].get('num_units')} U {d['config'].get('unit_blocks')}")
        except Exception as e:  # noqa: BLE001
            print(f"{f:50s} -- {e}")
