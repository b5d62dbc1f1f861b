"""f3 row-wise sharding with in-kernel sparse-input partitioning (§V) on the
GPU vs the oracle's sharded definition (canonical partial per shard, shard-order combine):
bit-exact, including bf16 output, mixed table-wise/sharded tables, several ranks."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import emb_test_helpers as H
import synth
from oracle import emb_oracle as O
from paper_conf_sc_chenbyo24_b200 import emb as E
from paper_conf_sc_chenbyo24_b200.comm import LocalGroup, run_ranks
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

DEV = torch.device("cuda", 0)


def _shards(w, nshard_of, owner_of):
    out = []
    for t in range(w.T):
        S = nshard_of(t)
        cuts = np.linspace(0, int(w.rows[t]), S + 1).astype(int)
        for s in range(S):
            out.append((t, s, int(cuts[s]), int(cuts[s + 1]), owner_of(t, s)))
    return out


def _inputs(w, seed, shards):
    offs, idxs = [], []
    for r in range(w.G):
        local = sorted((t, s) for (t, s, lo, hi, o) in shards if o == r)
        oo, xx, base = [np.zeros(1, np.int64)], [], 0
        for (t, s) in local:
            o, x = synth.table_csr(w, seed, t)
            oo.append(o[1:] + base)
            xx.append(x)
            base += int(o[-1])
        offs.append(np.concatenate(oo))
        idxs.append(np.concatenate(xx) if xx else np.zeros(0, np.int64))
    return offs, idxs


def _run(w, shards, seeds, flags=0):
    tabs = H.np_tables(w)
    full = [tabs[int(w.phys[t])] for t in range(w.T)]
    if w.wdtype == "bf16":
        dev_full = [torch.from_numpy(synth.to_bf16_bits(a).view(np.int16)).to(DEV).view(torch.bfloat16) for a in full]
    else:
        dev_full = [torch.from_numpy(a).to(DEV) for a in full]
    local_w = [[dev_full[t][lo:hi] for (t, s, lo, hi, o) in sorted(shards) if o == r] for r in range(w.G)]
    grp = LocalGroup(w.G) if w.G > 1 else None
    layers = run_ranks(w.G, lambda r: PgasEmbedding(r, w.G, 0, w.rows, None, w.dim, local_w[r], w.B, w.wdtype,
                                                    w.odtype, grp.allgather_for(r) if grp else None,
                                                    {"timeout_ms": 20000}, shards=shards))
    try:
        streams = [torch.cuda.Stream() for _ in range(w.G)]
        for seed in seeds:
            offs, idxs = _inputs(w, seed, shards)
            ins = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(w.G)]
            torch.cuda.synchronize()
            ys = [layers[r].forward(ins[r][0], ins[r][1], flags, streams[r]) for r in range(w.G)]
            if flags & E.EMB_FWD_SEPARATE_WAIT:
                for r in range(w.G):
                    layers[r].wait(streams[r])
            torch.cuda.synchronize()
            got = [H.dev_out_to_np(y.clone()) for y in ys]
            tb = [synth.to_bf16_bits(a) for a in full] if w.wdtype == "bf16" else full
            if w.wdtype == "bf16":
                tb = [synth.bf16_bits_to_f32(a) for a in tb]
            ref = O.emb_forward_sharded(tb, shards, offs, idxs, w.B, w.G, out_dtype=w.odtype)
            for r in range(w.G):
                assert np.array_equal(H.bits(got[r]), H.bits(ref[r])), (seed, r)
                assert layers[r].device_error() == 0
            torch.cuda.synchronize()
            for y in ys:  # poison: the next-but-one epoch must rewrite everything
                y.fill_(float("nan"))
    finally:
        run_ranks(w.G, lambda r: layers[r].close())


@pytest.mark.parametrize("G,flags", [(1, 0), (2, 0), (3, 0), (2, 2)])
def test_sharded_bitexact(G, flags):
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=40, B=73, T=5, dim=64, rows=900, dist="zipf")
    shards = _shards(w, lambda t: [1, 2, 3, 1, 4][t], lambda t, s: (t + 2 * s) % G)
    _run(w, shards, [11, 12, 13], flags)


def test_sharded_bf16_out_and_small_rows():
    w = synth.make_workload("tiny", G=2, pmin=1, pmax=30, B=41, T=3, dim=16, rows=300, wdtype="bf16", odtype="bf16")
    shards = _shards(w, lambda t: 2, lambda t, s: s)
    _run(w, shards, [5, 6])


def test_sharded_all_shards_on_one_rank_and_rank_without_shards():
    w = synth.make_workload("tiny", G=3, pmin=0, pmax=25, B=50, T=3, dim=128, rows=500)
    shards = _shards(w, lambda t: 3, lambda t, s: 1)  # everything on rank 1, ranks 0/2 only consume
    _run(w, shards, [7])


def _run_plain(w, shards, seed, flags=0, bad=None):
    """Sharded forward on the GPU; returns (outputs, device errors, offs, idxs)."""
    tabs = H.np_tables(w)
    full = [tabs[int(w.phys[t])] for t in range(w.T)]
    dev_full = [torch.from_numpy(a).to(DEV) for a in full]
    local_w = [[dev_full[t][lo:hi] for (t, s, lo, hi, o) in sorted(shards) if o == r] for r in range(w.G)]
    grp = LocalGroup(w.G) if w.G > 1 else None
    layers = run_ranks(w.G, lambda r: PgasEmbedding(r, w.G, 0, w.rows, None, w.dim, local_w[r], w.B, w.wdtype,
                                                    w.odtype, grp.allgather_for(r) if grp else None,
                                                    {"timeout_ms": 20000}, shards=shards))
    try:
        offs, idxs = _inputs(w, seed, shards)
        if bad is not None:
            idxs = [bad(r, x.copy()) for r, x in enumerate(idxs)]
        ins = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(w.G)]
        streams = [torch.cuda.Stream() for _ in range(w.G)]
        torch.cuda.synchronize()
        ys = [layers[r].forward(ins[r][0], ins[r][1], flags, streams[r]) for r in range(w.G)]
        torch.cuda.synchronize()
        got = [H.dev_out_to_np(y.clone()) for y in ys]
        errs = [layers[r].device_error(clear=True) for r in range(w.G)]
    finally:
        run_ranks(w.G, lambda r: layers[r].close())
    return got, errs, full


@pytest.mark.parametrize("G", [1, 2, 3])
def test_sharded_equals_plain_unsharded_definition(G):
    """f3 against the PLAIN definition of the forward (no shards: Y_r[i, t] = sum over the
    bag in CSR order, O.emb_forward with a table-wise placement), not the sharded oracle:
    integer-valued tables make every summation order exact, so the sharded GPU output must
    equal it bit for bit; float tables stay within the north star's 1e-6 S-normalised bound."""
    for mode in ("int", "float"):
        w = synth.make_workload("tiny", G=G, pmin=0, pmax=60, B=67, T=4, dim=32, rows=800, dist="zipf", mode=mode)
        shards = _shards(w, lambda t: [3, 1, 2, 4][t], lambda t, s: (t + s) % G)
        got, errs, full = _run_plain(w, shards, 41)
        assert errs == [0] * G
        wt = synth.make_workload("tiny", G=1, pmin=0, pmax=60, B=67, T=4, dim=32, rows=800, dist="zipf", mode=mode)
        o1, x1 = synth.rank_csr(wt, 41, 0)                # table-wise, one rank: the plain definition
        plain = O.emb_forward(full, wt.owner, [o1], [x1], w.B, 1)[0]
        cat = np.concatenate(got, axis=0)
        if mode == "int":
            assert np.array_equal(cat.view(np.uint32), plain.view(np.uint32))
        else:
            for t in range(w.T):
                lo, hi = O.rank_table_csr(o1, t, w.B)[1:]
                z64, S = O.pool_table_f64(full[t], O.rank_table_csr(o1, t, w.B)[0], x1[lo:hi])
                assert O.s_normalized_error(cat[:, t], z64, S) <= 1e-6


def test_sharded_check_bounds():
    """EMB_FWD_CHECK_BOUNDS with row-sharded tables: ids outside the whole table's [0, M_t)
    are flagged on the rank that scans them and contribute nothing; ids of another shard
    are skipped silently."""
    G = 2
    w = synth.make_workload("tiny", G=G, pmin=1, pmax=20, B=40, T=2, dim=32, rows=300, mode="int")
    shards = _shards(w, lambda t: 2, lambda t, s: s)

    def bad(r, x):
        x[2] = 300 if r == 0 else -1
        return x
    got, errs, full = _run_plain(w, shards, 9, E.EMB_FWD_CHECK_BOUNDS, bad=bad)
    assert all(e & E.EMB_DEVERR_BOUNDS for e in errs)
    # expected: the plain definition over the ids that are in range (integer tables: exact)
    offs, idxs = _inputs(w, 9, shards)
    idxs = [bad(r, x.copy()) for r, x in enumerate(idxs)]
    exp = np.zeros((w.B, w.T, w.dim), np.float32)
    for r in range(G):                                    # rank r holds shard r of every table
        for k, t in enumerate(range(w.T)):
            o, lo, hi = O.rank_table_csr(offs[r], k, w.B)
            for b in range(w.B):
                xs = [int(v) for v in idxs[r][lo + o[b]: lo + o[b + 1]]]
                lo_r, hi_r = [(s_lo, s_hi) for (tt, s, s_lo, s_hi, own) in shards if tt == t and own == r][0]
                for v in xs:
                    if lo_r <= v < hi_r:
                        exp[b, t] += full[t][v]
    cat = np.concatenate(got, axis=0)
    assert np.array_equal(cat, exp)


@pytest.mark.parametrize("G", [1, 2, 3])
def test_sharded_backward_integer_exact(G):
    """f2 on f3 row-sharded tables: every shard owner pulls the DP ranks' dY of its table's
    bags and scatters into ITS rows only; the expected dW of shard (t, s) is rows [lo, hi)
    of the table-wise transpose (the oracle's emb_backward on a one-rank placement of the
    same bags), exact on integer gradients over 2 epochs."""
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=40, B=61, T=4, dim=64, rows=500, dist="zipf")
    shards = _shards(w, lambda t: [2, 1, 3, 2][t], lambda t, s: (t + s) % G)
    tabs = H.np_tables(w)
    full = [tabs[int(w.phys[t])] for t in range(w.T)]
    dev_full = [torch.from_numpy(a).to(DEV) for a in full]
    mine = [sorted((t, s, lo, hi) for (t, s, lo, hi, o) in shards if o == r) for r in range(G)]
    local_w = [[dev_full[t][lo:hi] for (t, s, lo, hi) in mine[r]] for r in range(G)]
    grp = LocalGroup(G) if G > 1 else None
    layers = run_ranks(G, lambda r: PgasEmbedding(r, G, 0, w.rows, None, w.dim, local_w[r], w.B, w.wdtype, w.odtype,
                                                  grp.allgather_for(r) if grp else None, {"timeout_ms": 20000},
                                                  backward=True, shards=shards))
    try:
        offs, idxs = _inputs(w, 17, shards)
        ins = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(G)]
        starts, counts = O.split_batch(w.B, G)
        rng = np.random.default_rng(5)
        dW = [[torch.zeros((hi - lo, w.dim), device=DEV) for (t, s, lo, hi) in mine[r]] for r in range(G)]
        streams = [torch.cuda.Stream() for _ in range(G)]
        dYs = []
        for ep in range(2):
            dY = [rng.integers(-8, 9, size=(counts[r], w.T, w.dim)).astype(np.float32) for r in range(G)]
            dYs.append(dY)
            for r in range(G):
                with torch.cuda.stream(streams[r]):
                    layers[r].grad_slot(streams[r]).copy_(torch.from_numpy(dY[r]).to(DEV))
                layers[r].grad_ready(streams[r])
            for r in range(G):
                layers[r].backward(ins[r][0], ins[r][1], dW[r], 0, streams[r], publish=False)
            torch.cuda.synchronize()
        errs = [layers[r].device_error() for r in range(G)]
    finally:
        run_ranks(G, lambda r: layers[r].close())
    assert errs == [0] * G
    wt = synth.make_workload("tiny", G=1, pmin=0, pmax=40, B=61, T=4, dim=64, rows=500, dist="zipf")
    o1, x1 = synth.rank_csr(wt, 17, 0)
    ref = None
    for dY in dYs:
        r_ep, _, _ = O.emb_backward(w.rows, w.dim, wt.owner, [o1], [x1], [np.concatenate(dY, 0)], w.B, 1)
        ref = r_ep if ref is None else [a + b for a, b in zip(ref, r_ep)]
    for r in range(G):
        for k, (t, s, lo, hi) in enumerate(mine[r]):
            assert np.array_equal(dW[r][k].cpu().numpy().astype(np.float64), ref[t][lo:hi]), (r, t, s)


@pytest.mark.parametrize("G,odt", [(1, "f32"), (2, "f32"), (3, "f32"), (2, "bf16")])
def test_sharded_comparison_path_matches_fused_bitwise(G, odt):
    """f3 comparison path (pool every local shard's fp32 partial destination-major ->
    all-to-all, done with copies here -> unpack summing each table's partials in shard
    order) equals the fused PGAS path bit for bit, and both equal the sharded oracle."""
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=40, B=73, T=5, dim=64, rows=900, dist="zipf", odtype=odt)
    shards = _shards(w, lambda t: [1, 2, 3, 1, 4][t], lambda t, s: (t + 2 * s) % G)
    tabs = H.np_tables(w)
    full = [tabs[int(w.phys[t])] for t in range(w.T)]
    dev_full = [torch.from_numpy(a).to(DEV) for a in full]
    local_w = [[dev_full[t][lo:hi] for (t, s, lo, hi, o) in sorted(shards) if o == r] for r in range(G)]
    grp = LocalGroup(G) if G > 1 else None
    layers = run_ranks(G, lambda r: PgasEmbedding(r, G, 0, w.rows, None, w.dim, local_w[r], w.B, w.wdtype, w.odtype,
                                                  grp.allgather_for(r) if grp else None, {"timeout_ms": 20000},
                                                  shards=shards))
    try:
        offs, idxs = _inputs(w, 29, shards)
        ins = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(G)]
        streams = [torch.cuda.Stream() for _ in range(G)]
        torch.cuda.synchronize()
        yd = [layers[r].forward(ins[r][0], ins[r][1], 0, streams[r]) for r in range(G)]
        torch.cuda.synchronize()
        ys = [H.dev_out_to_np(y) for y in yd]
        sends, splits = [], []
        for r in range(G):
            sc, rc = E.emb_baseline_splits(layers[r].ctx)
            snd = torch.full((max(sum(sc), 1),), float("nan"), device=DEV)
            E.emb_baseline_pool(layers[r].ctx, ins[r][0], ins[r][1], snd)
            sends.append(snd)
            splits.append((sc, rc))
        torch.cuda.synchronize()
        outs = []
        for r in range(G):                                # all_to_all_single semantics, with copies
            recv = torch.cat([sends[src][sum(splits[src][0][:r]): sum(splits[src][0][:r]) + splits[src][0][r]]
                              for src in range(G)])
            assert recv.numel() == sum(splits[r][1])
            out = torch.full((layers[r].B_r, w.T, w.dim), float("nan"), device=DEV).to(layers[r].out_dtype)
            E.emb_baseline_unpack(layers[r].ctx, recv, out)
            torch.cuda.synchronize()
            outs.append(H.dev_out_to_np(out))
        errs = [layers[r].device_error() for r in range(G)]
    finally:
        run_ranks(G, lambda r: layers[r].close())
    assert errs == [0] * G
    ref = O.emb_forward_sharded(full, shards, offs, idxs, w.B, w.G, out_dtype=w.odtype)
    for r in range(G):
        assert np.array_equal(H.bits(outs[r]), H.bits(ys[r])), r
        assert np.array_equal(H.bits(outs[r]), H.bits(ref[r])), r
