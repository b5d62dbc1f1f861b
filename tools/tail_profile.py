"""Kernel tail from the f1 in-kernel trace: every warp appends {globaltimer, bytes} after each
claimed chunk, so the completion times of the chunks show when work runs out.  Prints the
span from the first to the last chunk completion and how long the last 1 % / 5 % of the
chunks took (the tail a programmatic dependent launch could overlap).

    python tools/tail_profile.py --config weak|single
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
    ap.add_argument("--dist", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    w = synth.make_workload(a.config, G=1, dist=a.dist)
    tables, _ = SG.local_tables(w, 0, dev)
    layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tables, w.B, w.wdtype, w.odtype,
                          options={"trace_capacity": 1 << 21})
    off, idx = SG.rank_csr(w, w.batch_seed(0), 0, dev)
    for _ in range(3):
        layer.forward(off, idx)
    torch.cuda.synchronize()
    E.emb_trace_read(layer.ctx, 1 << 21)                  # drop warm-up records
    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(s)
    layer.forward(off, idx, 0, s)
    e1.record(s)
    torch.cuda.synchronize()
    rec = E.emb_trace_read(layer.ctx, 1 << 21)
    t = np.sort(np.asarray(rec)[:, 0].astype(np.int64))
    t = (t - t[0]) / 1e3                                  # us after the first chunk completion
    n = len(t)
    out = {"config": a.config, "chunks": n, "kernel_us": e0.elapsed_time(e1) * 1e3,
           "span_first_to_last_chunk_us": float(t[-1]),
           "last_1pct_chunks_us": float(t[-1] - t[int(0.99 * n)]),
           "last_5pct_chunks_us": float(t[-1] - t[int(0.95 * n)]),
           "first_chunk_after_start_us_est": float(e0.elapsed_time(e1) * 1e3 - t[-1])}
    print(json.dumps(out))
    layer.close()


if __name__ == "__main__":
    main()
