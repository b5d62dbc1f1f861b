"""f1 claim evidence (Figs. 7/10): communication volume over time of the
fused PGAS kernel, from the in-kernel trace (emb_set_option("trace_capacity")).

G ranks are simulated in ONE process on one GPU (their kernels run concurrently on
separate streams and store into each other's symmetric buffers).  For every rank the
records {t, remote bytes, local bytes} of each claimed chunk are binned over the
kernel's span; the output shows whether remote traffic is spread across the whole
computation (paper claim 2, "smooth network usage") or bunched at the end (the
bulk-synchronous baseline, whose exchange starts only after its pool kernel ends).

    python tools/comm_timeline.py --G 2 --config weak --bins 40 > profiles/r01/comm_timeline_weak_G2.json
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
from paper_conf_sc_chenbyo24_b200.comm import LocalGroup, run_ranks
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--G", type=int, default=2)
    ap.add_argument("--config", default="weak")
    ap.add_argument("--tables-per-rank", type=int, default=8)
    ap.add_argument("--bins", type=int, default=40)
    ap.add_argument("--dist", default="zipf")
    a = ap.parse_args()
    G = a.G
    dev = torch.device("cuda", 0)
    base = synth.make_workload(a.config, G=G, dist=a.dist)
    T = a.tables_per_rank * G
    w = synth.make_workload(a.config, G=G, dist=a.dist, T=T)
    tabs = [SG.local_tables(w, r, dev)[0] for r in range(G)]
    grp = LocalGroup(G)
    layers = run_ranks(G, lambda r: PgasEmbedding(r, G, 0, w.rows, w.owner, w.dim, tabs[r], w.B, w.wdtype, w.odtype,
                                                  grp.allgather_for(r), {"trace_capacity": 1 << 20}))
    csr = [SG.rank_csr(w, w.batch_seed(0), r, dev) for r in range(G)]
    streams = [torch.cuda.Stream() for _ in range(G)]
    for it in range(3):  # warm-up, then the traced forward
        torch.cuda.synchronize()
        for r in range(G):
            E.emb_trace_read(layers[r].ctx, 0)
        evs = []
        for r in range(G):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(streams[r])
            layers[r].forward(csr[r][0], csr[r][1], 0, streams[r])
            e1.record(streams[r])
            evs.append((e0, e1))
        torch.cuda.synchronize()
    traces = [E.emb_trace_read(layers[r].ctx, 1 << 20) for r in range(G)]
    t0 = min(int(tr[:, 0].min()) for tr in traces)
    t1 = max(int(tr[:, 0].max()) for tr in traces)
    edges = np.linspace(t0, t1 + 1, a.bins + 1)
    out = {"config": a.config, "dist": a.dist, "G": G, "tables_per_rank": a.tables_per_rank, "global_batch": w.B,
           "dim": w.dim, "span_us": (t1 - t0) / 1e3, "bins": a.bins, "ranks": []}
    for r in range(G):
        tr = traces[r]
        t = tr[:, 0].astype(np.int64)
        rem = (tr[:, 1] >> np.uint64(32)).astype(np.int64)
        loc = (tr[:, 1] & np.uint64(0xFFFFFFFF)).astype(np.int64)
        # bins over THIS rank's own active span (simulated ranks share one GPU and largely
        # run one after another, so a global time axis would mix their spans)
        r0, r1 = int(t.min()), int(t.max())
        e = np.linspace(r0, r1 + 1, a.bins + 1)
        hr, _ = np.histogram(t, bins=e, weights=rem)
        hl, _ = np.histogram(t, bins=e, weights=loc)
        active = hr[hr > 0]
        cum = np.cumsum(hr) / max(hr.sum(), 1)
        out["ranks"].append({
            "rank": r, "records": int(tr.shape[0]), "remote_bytes": int(rem.sum()), "local_bytes": int(loc.sum()),
            "kernel_ms": evs[r][0].elapsed_time(evs[r][1]), "active_span_us": (r1 - r0) / 1e3,
            "start_offset_us": (r0 - t0) / 1e3,
            "remote_bytes_per_bin": hr.astype(int).tolist(), "local_bytes_per_bin": hl.astype(int).tolist(),
            "remote_frac_by_quarter": [float(cum[int(a.bins * q) - 1]) for q in (0.25, 0.5, 0.75, 1.0)],
            "remote_bins_nonzero_frac": float((hr > 0).mean()),
            "remote_cv_over_bins": float(hr.std() / hr.mean()) if hr.mean() > 0 else None,
        })
    print(json.dumps(out))
    run_ranks(G, lambda r: layers[r].close())


if __name__ == "__main__":
    main()
