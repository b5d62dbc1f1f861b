"""Per-kernel share of an ncu launch list (ncu --metrics gpu__time_duration.sum ... --csv):
cold-cache, serialised times, so compare SHARES, not absolutes."""
import collections
import csv
import sys

for f in sys.argv[1:]:
    rows = [r for r in csv.reader(open(f)) if r and (r[0] == "ID" or r[0].isdigit())]
    h = rows[0]
    ik, im, iv, iu = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot = collections.defaultdict(float)
    n = collections.Counter()
    for r in rows[1:]:
        if r[im] != "gpu__time_duration.sum":
            continue
        scale = {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(r[iu], 1e-3)
        k = r[ik].split("(")[0][:60]
        tot[k] += float(r[iv].replace(",", "")) * scale
        n[k] += 1
    s = sum(tot.values()) or 1.0
    print(f)
    for k, t in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"  {k:60s} launches {n[k]:4d}  {t / n[k]:9.1f} us/launch  share {100 * t / s:5.1f} %")
