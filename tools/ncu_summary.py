"""Summarise an ncu --set full report (raw page) into the metrics we track."""
import csv
import io
import json
import subprocess
import sys

WANT = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "l1tex__t_sector_hit_rate.pct": "l1_hit_pct",
    "l1tex__throughput.avg.pct_of_peak_sustained_active": "l1_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_pct",
    "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed": "l1_data_pipe_pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum": "l1_shared_wavefronts",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "smsp__inst_executed.sum": "inst",
    "sm__cycles_elapsed.avg.per_second": "sm_hz",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_read_sectors",
    "lts__t_sectors_srcunit_tex_lookup_miss.sum": "l2_miss_sectors",
}


def summary(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {"kernel": vals[hdr.index("Kernel Name")][:90]}
        for k, name in WANT.items():
            if k in hdr:
                i = hdr.index(k)
                try:
                    v = float(vals[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                if u == "Gbyte":
                    v *= 1e9
                elif u == "Mbyte":
                    v *= 1e6
                elif u == "Kbyte":
                    v *= 1e3
                elif u == "ms":
                    v *= 1e-3
                elif u == "us":
                    v *= 1e-6
                elif u == "ns":
                    v *= 1e-9
                d[name] = v
        if "l2_read_sectors" in d:
            d["l2_read_bytes"] = d["l2_read_sectors"] * 32
            if "duration" in d:
                d["l2_read_gbs"] = d["l2_read_bytes"] / d["duration"] / 1e9
        if "dram_read" in d and "duration" in d:
            d["dram_gbs"] = (d["dram_read"] + d.get("dram_write", 0)) / d["duration"] / 1e9
        res.append(d)
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        for d in summary(p):
            print(json.dumps({"report": p.split("/")[-1], **d}))
