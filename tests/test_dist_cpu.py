"""world_size-2 gloo tests of the multi-rank host plumbing (CPU, no GPU):
the IPC-handle all-gather callback, and the MP->DP exchange of the comparison path
(pool per owner -> all_to_all_single -> unpack) against the oracle's layout step (P11)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, G, port, q):
    import sys
    sys.path.insert(0, ROOT)
    try:
        import torch.distributed as dist

        import synth
        from oracle import emb_oracle as O
        from paper_conf_sc_chenbyo24_b200.comm import torch_allgather

        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=G)
        # 1. the all-gather callback used for IPC handles: rank order, exact bytes
        ag = torch_allgather()
        blob = bytes([rank]) * 64 + b"handle-of-rank-%d" % rank
        allb = ag(blob)
        ok1 = allb == b"".join(bytes([r]) * 64 + b"handle-of-rank-%d" % r for r in range(G))
        # 2. conventional exchange over a real process group vs the oracle's layout
        w = synth.make_workload("tiny", G=G, pmin=0, pmax=9, B=23, T=5, dim=8,
                                owner=np.array([1, 0, 1, 1, 0][:5]) % G)
        tabs = [synth.table_rows(w.table_seed, t, int(w.rows[t]), w.dim) for t in range(w.T)]
        off, idx = synth.rank_csr(w, 77, rank)
        local = list(w.local_tables(rank))
        starts, counts = O.split_batch(w.B, G)
        Z = [O.pool_table_f32(tabs[t], *(lambda o, lo, hi: (o, idx[lo:hi]))(*O.rank_table_csr(off, i, w.B)))
             for i, t in enumerate(local)]
        send = np.concatenate([np.stack([z[starts[d]:starts[d] + counts[d]] for z in Z], 1).reshape(-1)
                               if Z else np.zeros(0, np.float32) for d in range(G)])
        T_of = [int((w.owner == s).sum()) for s in range(G)]
        in_splits = [counts[d] * len(local) * w.dim for d in range(G)]
        out_splits = [counts[rank] * T_of[s] * w.dim for s in range(G)]
        recv = torch.empty(sum(out_splits))
        dist.all_to_all_single(recv, torch.from_numpy(send.astype(np.float32)), out_splits, in_splits)
        recv = recv.numpy()
        Y = np.empty((counts[rank], w.T, w.dim), np.float32)
        pos = 0
        for s in range(G):  # unpack: recv[src][b][t_l][:] -> Y[b][t][:]
            ts = [t for t in range(w.T) if w.owner[t] == s]
            blk = recv[pos:pos + out_splits[s]].reshape(counts[rank], len(ts), w.dim)
            for j, t in enumerate(ts):
                Y[:, t] = blk[:, j]
            pos += out_splits[s]
        offs, idxs = zip(*[synth.rank_csr(w, 77, r) for r in range(G)])
        ref = O.emb_forward(tabs, w.owner, offs, idxs, w.B, G)[rank]
        ok2 = np.array_equal(Y.view(np.uint32), ref.view(np.uint32))
        dist.destroy_process_group()
        q.put((rank, ok1, ok2, ""))
    except Exception:
        import traceback
        q.put((rank, False, False, traceback.format_exc()))


@pytest.mark.parametrize("G", [2])
def test_gloo_world2_allgather_and_exchange(G):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, G, port, q)) for r in range(G)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=180) for _ in range(G))
    for p in ps:
        p.join(timeout=60)
    for rank, ok1, ok2, tb in res:
        assert tb == "", tb
        assert ok1, f"rank {rank}: all-gather bytes wrong"
        assert ok2, f"rank {rank}: gloo exchange != oracle layout"
