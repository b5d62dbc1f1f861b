"""Refresh profiles/traffic.json (per-launch DRAM and L2->SM bytes that bench.py reports as
roofline.traffic / roofline.l2) from committed ncu summaries.

    python tools/update_traffic.py weak:zipf:G1=profiles/r01/full_weak_zipf.summary.json ...
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    path = os.path.join(ROOT, "profiles", "traffic.json")
    tj = json.load(open(path)) if os.path.exists(path) else {}
    for arg in sys.argv[1:]:
        key, summ = arg.split("=", 1)
        m = json.load(open(os.path.join(ROOT, summ) if not os.path.isabs(summ) else summ))["metrics"][0]
        tj[key] = {"dram_bytes_per_launch": m["dram_read"] + m["dram_write"], "dram_read": m["dram_read"],
                   "dram_write": m["dram_write"], "l2_read_bytes_per_launch": m.get("l2_read_bytes"),
                   "duration_s_ncu": m["duration"], "kernel": m["kernel"],
                   "source": f"{summ} (ncu --set full --clock-control none)"}
        print(key, tj[key]["dram_bytes_per_launch"], tj[key]["duration_s_ncu"])
    with open(path, "w") as f:
        json.dump(tj, f, indent=1)


if __name__ == "__main__":
    main()
