"""Write committed summaries of ncu reports: profiles/<tag>/<name>.summary.json with the
tracked metrics, the warp-stall breakdown and the top SASS lines by stall samples."""
import csv
import io
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summary  # noqa: E402


def stalls(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, vals = rows[0], rows[2]
    res = {}
    for i, h in enumerate(hdr):
        if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued"):
            try:
                res[h.replace("smsp__pcsamp_warps_issue_stalled_", "")] = float(vals[i].replace(",", ""))
            except ValueError:
                pass
    tot = sum(res.values()) or 1.0
    return {k: round(100 * v / tot, 1) for k, v in sorted(res.items(), key=lambda kv: -kv[1]) if v / tot > 0.005}


def hot_sass(path, n=15):
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    isrc, iss = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
    data = []
    for r in rows[2:]:
        try:
            data.append((int(r[iss] or 0), r[isrc].strip()))
        except (ValueError, IndexError):
            pass
    tot = sum(d[0] for d in data) or 1
    return [f"{100 * c / tot:5.1f}%  {src}" for c, src in sorted(data, reverse=True)[:n]]


if __name__ == "__main__":
    tag = sys.argv[1]
    for p in sys.argv[2:]:
        name = os.path.basename(p).replace(".ncu-rep", "")
        d = {"report": name, "metrics": summary(p), "stall_pct": stalls(p), "hot_sass": hot_sass(p)}
        os.makedirs(f"profiles/{tag}", exist_ok=True)
        with open(f"profiles/{tag}/{name}.summary.json", "w") as f:
            json.dump(d, f, indent=1)
        print(name, json.dumps(d["stall_pct"]))
