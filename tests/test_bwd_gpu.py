"""GPU parity of the f2 backward (emb_backward_grad_slot / emb_backward) against the
oracle's transpose: exact on integer-valued gradients (any atomic order is exact), and
within the order-independent recursive-summation bound |err| <= n * 2^-24 * S (n =
contributions to the row, S = sum |g|) on float gradients."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import emb_test_helpers as H
import synth
from oracle import emb_oracle as O
from paper_conf_sc_chenbyo24_b200.comm import LocalGroup, run_ranks
from paper_conf_sc_chenbyo24_b200 import emb as E
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

DEV = torch.device("cuda", 0)


def _dY(w, seed, integer):
    rng = np.random.default_rng(seed)
    _, counts = O.split_batch(w.B, w.G)
    if integer:
        return [rng.integers(-8, 9, size=(counts[r], w.T, w.dim)).astype(np.float32) for r in range(w.G)]
    return [rng.standard_normal((counts[r], w.T, w.dim)).astype(np.float32) for r in range(w.G)]


def _run_bwd(w, dY, seed, epochs=1, flags=0, opts=None):
    tabs = H.np_tables(w)
    offs, idxs = H.np_csrs(w, seed)
    tdev = [[torch.from_numpy(tabs[int(w.phys[t])]).to(DEV) for t in w.local_tables(r)] for r in range(w.G)]
    if w.G == 1:
        layers = [PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tdev[0], w.B, backward=True)]
    else:
        grp = LocalGroup(w.G)
        layers = run_ranks(w.G, lambda r: PgasEmbedding(r, w.G, 0, w.rows, w.owner, w.dim, tdev[r], w.B,
                                                        allgather=grp.allgather_for(r), backward=True))
    try:
        for k, v in (opts or {}).items():
            for L in layers:
                E.emb_set_option(L.ctx, k, v)
        dW = [[torch.zeros((int(w.rows[t]), w.dim), device=DEV) for t in w.local_tables(r)] for r in range(w.G)]
        streams = [torch.cuda.Stream() for _ in range(w.G)]
        ins = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(w.G)]
        for ep in range(epochs):
            for r in range(w.G):
                with torch.cuda.stream(streams[r]):
                    g = layers[r].grad_slot(streams[r])
                    g.copy_(torch.from_numpy(dY[r]).to(DEV, non_blocking=False))
            for r in range(w.G):                          # ranks share one GPU: publish all first
                layers[r].grad_ready(streams[r])
            torch.cuda.synchronize()
            for r in range(w.G):
                layers[r].backward(ins[r][0], ins[r][1], dW[r], flags, streams[r], publish=False)
            torch.cuda.synchronize()
        for r in range(w.G):
            assert layers[r].device_error() == 0
        out = {}
        for r in range(w.G):
            for tl, t in enumerate(w.local_tables(r)):
                out[int(t)] = dW[r][tl].cpu().numpy()
        return out, offs, idxs
    finally:
        if w.G == 1:
            layers[0].close()
        else:
            run_ranks(w.G, lambda r: layers[r].close())


@pytest.mark.parametrize("G,dim,dist", [(1, 16, "uniform"), (1, 128, "zipf"), (2, 64, "zipf"), (3, 32, "uniform"),
                                        (2, 256, "zipf")])
def test_bwd_integer_exact(G, dim, dist):
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=40, B=97, T=5, dim=dim, rows=300, dist=dist)
    dY = _dY(w, 3, integer=True)
    got, offs, idxs = _run_bwd(w, dY, 12)
    ref, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        assert np.array_equal(got[t].astype(np.float64), ref[t]), t


def test_bwd_float_within_bound_and_accumulates_over_epochs():
    w = synth.make_workload("tiny", G=2, pmin=1, pmax=64, B=200, T=4, dim=128, rows=500, dist="zipf")
    dY = _dY(w, 4, integer=False)
    got, offs, idxs = _run_bwd(w, dY, 13, epochs=3)          # dW accumulates 3 identical steps
    ref, S, cnt = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        n = 3 * cnt[t][:, None]
        err = np.abs(got[t].astype(np.float64) - 3 * ref[t])
        assert np.all(err <= n * 2.0 ** -24 * 3 * S[t] + 1e-30), t


def test_bwd_placement_invariance():
    outs = []
    for own in ([0, 0, 1, 1, 1], [1, 0, 1, 0, 1], [1, 1, 1, 1, 1]):
        w = synth.make_workload("tiny", G=2, pmin=0, pmax=9, B=61, T=5, dim=32, rows=100, owner=np.array(own))
        got, _, _ = _run_bwd(w, _dY(w, 9, integer=True), 6)
        outs.append(got)
    for d in outs[1:]:
        for t in d:
            assert np.array_equal(d[t], outs[0][t])


@pytest.mark.parametrize("opts", [{"bwd_interleave": 0}, {"bwd_group": 2}, {"bwd_group": 3}, {"bwd_group": 4},
                                  {"bwd_group": 7}, {"bwd_group": 1}, {"bwd_cache": 0}, {"bwd_cache": 0, "bwd_group": 3},
                                  {"bwd_cache": 0, "bwd_interleave": 0},
                                  {"bwd_cache": 16, "bwd_chunk_rows": 1024},
                                  {"bwd_cache": 16, "bwd_interleave": 0}, {"bwd_algo": 1},
                                  {"bwd_algo": 1, "bwd_chunk_rows": 7}])
def test_bwd_chunk_orders_integer_exact(opts):
    """every chunk order (table-major, groups of g tables incl. a ragged last group, all
    tables interleaved) visits every bag exactly once: exact on integer gradients"""
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=40, B=97, T=7, dim=64, rows=300, dist="zipf")
    dY = _dY(w, 5, integer=True)
    got, offs, idxs = _run_bwd(w, dY, 14, opts=opts)
    ref, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        assert np.array_equal(got[t].astype(np.float64), ref[t]), t


@pytest.mark.parametrize("dim,cache", [(16, 16), (64, 16), (128, 16), (256, 16), (16, 0), (128, 0), (512, 0),
                                       (16, -1), (64, -1), (128, -1), (256, -1), (512, -1)])
def test_bwd_row_cache_exact_and_float_bound(dim, cache):
    """f2 per-warp dW row cache (bwd_cache) and the sorted algorithm (cache -1 = bwd_algo 1):
    integer gradients exact, float gradients within the order-independent summation bound
    (cached rows are summed in shared memory first)"""
    opts = {"bwd_cache": cache, "bwd_chunk_rows": 512} if cache >= 0 else {"bwd_algo": -cache}
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=60, B=150, T=3, dim=dim, rows=200, dist="zipf")
    got, offs, idxs = _run_bwd(w, _dY(w, 21, integer=True), 22, opts=opts)
    ref, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, _dY(w, 21, integer=True), w.B, w.G)
    for t in range(w.T):
        assert np.array_equal(got[t].astype(np.float64), ref[t]), t
    dY = _dY(w, 23, integer=False)
    got, offs, idxs = _run_bwd(w, dY, 24, epochs=2, opts=opts)
    ref, S, cnt = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        n = 2 * cnt[t][:, None]
        err = np.abs(got[t].astype(np.float64) - 2 * ref[t])
        assert np.all(err <= n * 2.0 ** -24 * 2 * S[t] + 1e-30), t


@pytest.mark.parametrize("G,dist,algo", [(1, "zipf", 1), (2, "uniform", 1), (3, "zipf", 1)])
def test_bwd_sorted_algo_integer_exact_multi_epoch(G, dist, algo):
    """bwd_algo 1 (radix sort + segmented sum): exact on integer gradients over 3 epochs
    (workspace reuse), incl. empty bags and G > 1 one-sided dY loads"""
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=70, B=131, T=5, dim=128, rows=400, dist=dist)
    dY = _dY(w, 31, integer=True)
    got, offs, idxs = _run_bwd(w, dY, 32, epochs=3, opts={"bwd_algo": algo})
    ref, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        assert np.array_equal(got[t].astype(np.float64), 3 * ref[t]), t


def test_bwd_sorted_capacity_error():
    """a CSR with more lookups than the preset workspace sets EMB_DEVERR_CAPACITY (0x4)"""
    w = synth.make_workload("tiny", G=1, pmin=1, pmax=20, B=64, T=2, dim=32, rows=100)
    tabs = H.np_tables(w)
    offs, idxs = H.np_csrs(w, 5)
    L = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, [torch.from_numpy(tabs[int(w.phys[t])]).to(DEV) for t in range(w.T)],
                      w.B, backward=True)
    try:
        E.emb_set_option(L.ctx, "bwd_algo", 1)
        E.emb_set_option(L.ctx, "bwd_max_nnz", 10)
        dW = [torch.zeros((int(w.rows[t]), w.dim), device=DEV) for t in range(w.T)]
        g = L.grad_slot()
        g.zero_()
        L.backward(torch.from_numpy(offs[0]).to(DEV), torch.from_numpy(idxs[0]).to(DEV), dW)
        torch.cuda.synchronize()
        assert L.device_error(clear=True) & 0x4
    finally:
        L.close()


@pytest.mark.parametrize("G,dim,algo", [(1, 128, 1), (2, 128, 1), (1, 64, 1), (1, 128, 0)])
def test_bwd_medium_many_tasks_integer_exact(G, dim, algo):
    """a size where bwd_algo 1's sorted list spans hundreds of 512-entry reduce tasks, zipf-hot
    rows' runs cross task boundaries (one partial red.add per task) and the last task is ragged;
    also the radix passes' multi-tile histograms and the atomic default at the same size: exact
    on integer gradients against the oracle's transpose"""
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=90, B=3001, T=6, dim=dim, rows=20000, dist="zipf")
    dY = _dY(w, 41, integer=True)
    got, offs, idxs = _run_bwd(w, dY, 42, opts={"bwd_algo": algo})
    assert sum(int(o[-1]) for o in offs) > 100 * 512
    ref, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    for t in range(w.T):
        assert np.array_equal(got[t].astype(np.float64), ref[t]), t
