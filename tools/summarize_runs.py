"""One line per bench JSON file in a directory: ms/step steady and cold, roofline, parity."""
import glob
import json
import os
import sys

for f in sorted(glob.glob(os.path.join(sys.argv[1], "*.json"))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f"{os.path.basename(f):40s} {d['ms_per_step']:.4f} cold {d['cold_l2']['ms_per_step']:.4f} "
              f"{d['roofline']['bound']} {d['roofline']['frac']:.3f} {d.get('parity')}")
    except Exception as e:  # noqa: BLE001 - a diagnostics table
        print(f"{os.path.basename(f):40s} ERR {e}")
