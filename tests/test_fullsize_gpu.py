"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(PgasEmbedding defaults, device-generated inputs): EVERY bag of at least four whole tables
(the first, the last -- which the guided tail claims in small chunks --, and two more) is
recomputed by the oracle from the counter generators (never from the CUDA path) and must
be bit-exact, and within the north star's S-normalised tolerance of the fp64 sum."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import synth
import synth.gpu as SG
from oracle import emb_oracle as O
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

DEV = torch.device("cuda", 0)


def _oracle_table(w, seed, t):
    """Oracle pooling of logical table t over the whole batch.  Only the rows the batch
    touches are regenerated (table_values of the distinct ids) and the ids are renumbered
    into that compact table -- a re-indexing of the input, not of the arithmetic."""
    o, x = synth.table_csr(w, seed, t)
    uniq, inv = np.unique(x, return_inverse=True)
    Wu = synth.table_values(w.table_seed, int(w.phys[t]), uniq, w.dim, w.mode, w.wdtype)
    Z = O.pool_table_f32(Wu, o, inv.astype(np.int64))
    Z64, S = O.pool_table_f64(Wu, o, inv.astype(np.int64))
    return Z, Z64, S


def _whole_table_parity(name, tables, dist=None, i32=False, **over):
    w = synth.make_workload(name, G=1, dist=dist, **over)
    dev_tables, _ = SG.local_tables(w, 0, DEV)
    seed = w.batch_seed(0)
    off, idx = SG.rank_csr(w, seed, 0, DEV)
    if i32:
        off, idx = off.to(torch.int32), idx.to(torch.int32)
    layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, dev_tables, w.B, w.wdtype, w.odtype)
    try:
        y = layer.forward(off, idx)
        torch.cuda.synchronize()
        assert layer.device_error() == 0
        bf16_out = y.dtype == torch.bfloat16
        cols = {}
        for t in tables:
            c = y[:, t, :]
            # bf16 output: the raw 16-bit patterns vs the oracle's RNE of the fp32 sum (C6)
            cols[t] = c.contiguous().view(torch.int16).cpu().numpy().view(np.uint16) if bf16_out else c.cpu().numpy()
        y1 = y.clone()
        layer.forward(off, idx)
        y2 = layer.forward(off, idx)                     # same slot again after a full ring turn
        torch.cuda.synchronize()
        assert torch.equal(y1.view(torch.int16), y2.view(torch.int16)), "forward is not deterministic"
    finally:
        layer.close()
        del dev_tables
        torch.cuda.empty_cache()
    del off, idx
    for t in tables:
        Z, Z64, S = _oracle_table(w, seed, t)
        got = cols[t]
        if bf16_out:
            exp = O.rne_bf16(Z)
            bad = np.argwhere(got != exp)
            assert bad.size == 0, (t, len(bad), bad[0].tolist())
            assert O.s_normalized_error(O.bf16_to_f32(got), Z64, S) <= 1e-2, t
        else:
            gb, eb = got.view(np.uint32), Z.view(np.uint32)
            bad = np.argwhere(gb != eb)
            assert bad.size == 0, (t, len(bad), bad[0].tolist())
            assert O.s_normalized_error(got, Z64, S) <= 1e-6, t


def test_single_config_whole_tables():
    _whole_table_parity("single", [0, 1, 13, 25])


def test_weak_config_whole_tables():
    _whole_table_parity("weak", [0, 1, 13, 25])


def test_weak_config_whole_tables_int32_indices():
    _whole_table_parity("weak", [0, 7, 25], i32=True)


def test_weak_config_uniform_whole_tables():
    _whole_table_parity("weak", [0, 12, 25], dist="uniform")


@pytest.mark.slow
def test_strong_config_g1_aliased_whole_tables():
    """208 logical tables over 104 physical ones (C27): tables 0 and 1 share rows"""
    _whole_table_parity("strong", [0, 1, 104, 207])


@pytest.mark.slow
def test_large_shard_bf16_whole_tables():
    """one rank's LPT share of the 8-GPU `large` config (64 mixed tables, 150 GB of bf16
    rows, d = 256, bf16 output): the first, the last, the largest and the smallest table"""
    rows = synth.make_workload("large_shard", G=1).rows
    ts = sorted({0, len(rows) - 1, int(np.argmax(rows)), int(np.argmin(rows))})
    _whole_table_parity("large_shard", ts)


def test_weak_config_backward_sampled_rows():
    """f2 at the weak config's full size: integer dY, sampled dW rows of two tables
    recomputed by the oracle's definition from the regenerated CSR (exact)."""
    w = synth.make_workload("weak", G=1)
    seed = w.batch_seed(0)
    tables, _ = SG.local_tables(w, 0, DEV)
    off, idx = SG.rank_csr(w, seed, 0, DEV)
    layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tables, w.B, w.wdtype, w.odtype, backward=True)
    check_t = [0, w.T - 1]
    try:
        dW = [torch.zeros((int(w.rows[t]), w.dim), device=DEV) if t in check_t else
              torch.zeros((1, w.dim), device=DEV) for t in range(w.T)]
        # tables not checked still need a full-size dW: reuse one scratch buffer for them
        scratch = torch.zeros((int(w.rows[1]), w.dim), device=DEV)
        dW = [d if t in check_t else scratch for t, d in enumerate(dW)]
        rng = np.random.default_rng(3)
        dY = rng.integers(-8, 9, size=(w.B, w.T, w.dim)).astype(np.float32)
        g = layer.grad_slot()
        g.copy_(torch.from_numpy(dY).to(DEV))
        layer.backward(off, idx, dW)
        torch.cuda.synchronize()
        assert layer.device_error() == 0
        for t in check_t:
            o, x = synth.table_csr(w, seed, t)
            bag_of = np.repeat(np.arange(w.B), np.diff(o))
            rows = np.unique(np.concatenate([x[:50], rng.integers(0, int(w.rows[t]), 50)]))
            got = dW[t][torch.from_numpy(rows).to(DEV)].cpu().numpy()
            for i, r in enumerate(rows):
                sel = bag_of[x == r]
                ref = dY[sel, t].astype(np.float64).sum(axis=0) if sel.size else np.zeros(w.dim)
                assert np.array_equal(got[i].astype(np.float64), ref), (t, r)
    finally:
        layer.close()
        del tables
        torch.cuda.empty_cache()
