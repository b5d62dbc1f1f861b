"""Option sweep for the fused kernel on one GPU (tables generated once per config).

    python tools/sweep.py --config weak --dist zipf --opts 'kernel=1' 'chunk_rows=256' ...
Prints one line per option set: ms/step, samples/s, lookup-counted GB/s.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import synth
import synth.gpu as SG
from paper_conf_sc_chenbyo24_b200 import emb as E
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="weak")
    ap.add_argument("--dists", default="zipf,uniform")
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--opts", nargs="*", default=[""])
    ap.add_argument("--baseline", action="store_true")
    ap.add_argument("--repeat", type=int, default=1)
    ap.add_argument("--gap", type=float, default=0.0, help="idle seconds before each measurement (clock recovery)")
    ap.add_argument("--rows", type=int, default=None, help="override rows per table (e.g. an L2-resident table)")
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    over = {"rows": a.rows} if a.rows else {}
    w = synth.make_workload(a.config, G=1, **over)
    tables, _ = SG.local_tables(w, 0, dev)
    layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tables, w.B, w.wdtype, w.odtype)
    s = torch.cuda.Stream()
    agg = {}
    for dist in a.dists.split(","):
        wd = synth.make_workload(a.config, G=1, dist=dist, **over)
        bs = [SG.rank_csr(wd, wd.batch_seed(i), 0, dev) for i in range(3)]
        nnz = np.mean([int(b[0][-1]) for b in bs])
        byt = nnz * (w.dim * w.elem_bytes() + 8) + w.T * w.B * (8 + w.dim * w.out_elem_bytes())
        for o in [o for _ in range(a.repeat) for o in a.opts]:
            defaults = {"chunk_rows": 0, "ctas_per_sm": 0, "stagger": 1, "carveout": 0, "fwd_interleave": 0,
                        "tma_store": 0, "tail_div": 4}
            kv = dict(defaults)
            for item in o.split(",") if o else []:
                k, v = item.split("=")
                kv[k] = int(v)
            for k, v in kv.items():
                E.emb_set_option(layer.ctx, k, v)
            fn = (lambda i: layer.forward_baseline(bs[i % 3][0], bs[i % 3][1], None, 0, s)) if a.baseline else \
                 (lambda i: layer.forward(bs[i % 3][0], bs[i % 3][1], 0, s))
            for i in range(5):
                fn(i)
            torch.cuda.synchronize()
            if a.gap > 0:
                import time
                time.sleep(a.gap)
                for i in range(2):
                    fn(i)
                torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(s)
            for i in range(a.steps):
                fn(i)
            e1.record(s)
            try:
                import pynvml
                pynvml.nvmlInit()
                h = pynvml.nvmlDeviceGetHandleByIndex(0)
                clk = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                pw = pynvml.nvmlDeviceGetPowerUsage(h) / 1000
            except Exception:
                clk = pw = None
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / a.steps
            agg.setdefault((dist, o), []).append(ms)
            print(json.dumps({"config": a.config, "rows": int(w.rows[0]), "dist": dist, "opts": o, "ms": round(ms, 4),
                              "Msamples_s": round(w.B / ms / 1e3, 3), "GBs": round(byt / ms / 1e6, 1),
                              "sm_mhz": clk, "power_w": pw}), flush=True)
            assert layer.device_error() == 0
    for (dist, o), v in agg.items():
        print(json.dumps({"summary": True, "config": a.config, "dist": dist, "opts": o, "median_ms": round(float(np.median(v)), 4),
                          "min_ms": round(min(v), 4), "n": len(v)}), flush=True)
    layer.close()


if __name__ == "__main__":
    main()
