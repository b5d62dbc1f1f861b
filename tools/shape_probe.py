"""Lookup-counted gather rate of the fused forward on workload shapes derived from a BASELINE
config (one GPU), to separate what the kernel pays per row from what the workload shape
costs (table switches, bag length, index width).

    python tools/shape_probe.py --config weak --shape T=1,B=425984 --shape pmin=128,pmax=128
Prints one JSON line per shape: ms/step, lookups, lookup-counted TB/s of row bytes.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

import synth
import synth.gpu as SG
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="weak")
    ap.add_argument("--shape", action="append", default=[], help="make_workload overrides k=v,k=v ('' = the config)")
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--idx32", action="store_true")
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    for sh in a.shape or [""]:
        over = {}
        for item in sh.split(",") if sh else []:
            k, v = item.split("=")
            over[k] = v if k == "dist" else int(v)
        w = synth.make_workload(a.config, G=1, **over)
        tables, _ = SG.local_tables(w, 0, dev)
        layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tables, w.B, w.wdtype, w.odtype)
        bs = [SG.rank_csr(w, w.batch_seed(i), 0, dev) for i in range(3)]
        if a.idx32:
            bs = [(o.to(torch.int32), x.to(torch.int32)) for o, x in bs]
        torch.cuda.synchronize()                          # tables / CSR are generated on the default stream
        s = torch.cuda.Stream()
        fn = lambda i: layer.forward(bs[i % 3][0], bs[i % 3][1], 0, s)
        for i in range(5):
            fn(i)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(s)
        for i in range(a.steps):
            fn(i)
        e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.steps
        nnz = sum(int(b[0][-1]) for b in bs) / 3
        rb = w.dim * w.elem_bytes()
        print(json.dumps({"config": a.config, "shape": sh, "T": w.T, "B": w.B, "ms": round(ms, 4), "lookups": int(nnz),
                          "lookup_TBps": round(nnz * rb / ms / 1e9, 2)}), flush=True)
        assert layer.device_error() == 0
        layer.close()
        del tables, bs
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
