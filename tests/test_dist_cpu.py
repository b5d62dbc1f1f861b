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


def _bench_worker(rank, G, port, q):
    """bench.py's multi-rank host logic over a real gloo world of 2: per-rank roofline dicts
    all-gathered, combined into max_r t_roof / max_r t_measured; the f1 trace summary of
    synthetic records; the f3 shard placement of --shards."""
    import sys
    sys.path.insert(0, ROOT)
    try:
        import torch.distributed as dist

        import bench
        import synth

        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=G)
        peak = 6553.6
        hbm = [3.0e9, 2.0e9][rank]
        egress, ingress = [(1.0e8, 2.0e8), (4.0e9, 1.0e8)][rank]
        t_r = bench.rank_roof(hbm, egress, ingress, peak)
        mine = {"rank": rank, "t_roof_ms": t_r * 1e3, "hbm_compulsory_bytes": hbm, "nvlink_egress_bytes": egress,
                "nvlink_ingress_bytes": ingress}
        allr = [None] * G
        dist.all_gather_object(allr, mine)
        ms_r = [0.9, 1.3][rank]
        t = torch.tensor([ms_r], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        rc = bench.combine_roofline(allr, float(t.item()), peak)
        # rank 1 binds: 4e9 B of NVLink egress at 770 GB/s (5.19 ms) > every HBM term
        exp_t = 4.0e9 / 770e9 * 1e3
        ok = (rc["binding"]["rank"] == 1 and rc["bound"] == "nvlink" and abs(rc["t_roof_ms"] - exp_t) < 1e-12 and
              abs(rc["frac"] - exp_t / 1.3) < 1e-12 and rc["bytes"] == 4.0e9)
        # f1 summary: 100 chunks spread evenly over 1 ms, rank r's remote share r/2
        ts = np.arange(100, dtype=np.uint64) * np.uint64(10000) + np.uint64(5)
        rem = np.full(100, 512 * rank, dtype=np.uint64)
        loc = np.full(100, 512, dtype=np.uint64)
        s = bench.trace_summary(np.stack([ts, (rem << np.uint64(32)) | loc], 1))
        ok = ok and s["records"] == 100 and s["local_bytes"] == 51200 and s["remote_bytes"] == 51200 * rank
        if rank == 1:
            ok = ok and s["remote_frac_by_quarter"] == [0.25, 0.5, 0.75, 1.0] and s["remote_bins_nonzero_frac"] == 1.0
        # --shards placement: shard s of table t on rank (owner[t] + s) % G, contiguous row cuts
        w = synth.make_workload("tiny", G=G, T=4, rows=1000)
        shards = bench.shard_layout(w, 3, G)
        for tt in range(w.T):                       # contiguous cover of [0, M_t), owners rotate
            mine_t = sorted((s_, lo, hi, o) for (t2, s_, lo, hi, o) in shards if t2 == tt)
            ok = ok and mine_t[0][1] == 0 and mine_t[-1][2] == 1000
            ok = ok and all(a[2] == b[1] for a, b in zip(mine_t, mine_t[1:]))
            ok = ok and [o for (_, _, _, o) in mine_t] == [(int(w.owner[tt]) + k) % G for k in range(3)]
        dist.destroy_process_group()
        q.put((rank, bool(ok), True, ""))
    except Exception:
        import traceback
        q.put((rank, False, False, traceback.format_exc()))


def test_gloo_world2_bench_multirank_host_logic():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_bench_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=180) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
    for rank, ok, _, tb in res:
        assert tb == "", tb
        assert ok, f"rank {rank}: bench multi-rank host logic wrong"
