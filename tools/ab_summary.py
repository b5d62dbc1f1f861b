"""Summarise tools/ab.sh output: per (config, dist, build) the median ms and SM clocks."""
import collections
import json
import sys

import numpy as np

agg = collections.defaultdict(list)
for line in open(sys.argv[1]):
    try:
        lib, cfg, js = line.split(" ", 2)
        d = json.loads(js)
    except ValueError:
        continue
    agg[(cfg, d["dist"], lib)].append((d["ms"], d.get("sm_mhz")))
base = {}
for k in sorted(agg):
    ms = [m for m, _ in agg[k]]
    med = float(np.median(ms))
    key = k[:2]
    base.setdefault(key, med)
    print(f"{k[0]:12s} {k[1]:8s} {k[2]:24s} median {med:.4f} ms  ({med / base[key]:.3f}x of first)  "
          f"runs {[round(m, 4) for m in ms]}  mhz {[c for _, c in agg[k]]}")
