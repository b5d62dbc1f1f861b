"""Pins for the CPU oracle.  CPU only: -m "not gpu".

Every test checks the oracle against something other than itself: pure-Python
brute force, a closed form, an invariant, a library routine (torch embedding_bag,
torch bf16 conversion) or the paper's worked-example structure (tests/golden/).
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import emb_oracle as O

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _tables(w, mode=None):
    mode = mode or w.mode
    return [synth.table_rows(w.table_seed, int(w.phys[t]), int(w.rows[t]), w.dim, mode, w.wdtype) for t in range(w.T)]


def _csrs(w, seed):
    offs, idxs = [], []
    for r in range(w.G):
        o, x = synth.rank_csr(w, seed, r)
        offs.append(o)
        idxs.append(x)
    return offs, idxs


def _brute(tables, owner, offs, idxs, B, G, acc="f32"):
    """P1: pure-Python triple loop straight from L91-95 + L111-113 (no numpy arithmetic)."""
    T = len(tables)
    d = tables[0].shape[1]
    q, rem = divmod(B, G)
    counts = [q + (1 if r < rem else 0) for r in range(G)]
    starts = [sum(counts[:r]) for r in range(G)]
    outs = []
    for r in range(G):
        Y = [[[0.0] * d for _ in range(T)] for _ in range(counts[r])]
        for i in range(counts[r]):
            b = starts[r] + i
            for t in range(T):
                o = int(owner[t])
                tl = [u for u in range(T) if int(owner[u]) == o].index(t)
                lo = int(offs[o][tl * B + b])
                hi = int(offs[o][tl * B + b + 1])
                for k in range(d):
                    if acc == "f64":
                        s = 0.0
                        for j in range(lo, hi):
                            s += float(tables[t][int(idxs[o][j]), k])
                    else:
                        s = np.float32(0.0)
                        for j in range(lo, hi):
                            v = np.float32(tables[t][int(idxs[o][j]), k])
                            s = v if j == lo else np.float32(s + v)
                    Y[i][t][k] = s
        outs.append(np.array(Y, dtype=np.float64 if acc == "f64" else np.float32))
    return outs


@pytest.mark.parametrize("pmin,pmax,G", [(4, 4, 2), (0, 6, 2), (0, 5, 3), (1, 3, 1)])
def test_p1_bruteforce_tiny(pmin, pmax, G):
    w = synth.make_workload("tiny", G=G, pmin=pmin, pmax=pmax)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 11)
    got = O.emb_forward(tabs, w.owner, offs, idxs, w.B, G)
    ref = _brute(tabs, w.owner, offs, idxs, w.B, G, "f32")
    ref64 = _brute(tabs, w.owner, offs, idxs, w.B, G, "f64")
    for r in range(G):
        assert got[r].shape == (synth.batch_split(w.B, G)[1][r], w.T, w.dim)
        assert np.array_equal(got[r].view(np.uint32), ref[r].view(np.uint32))  # bit-exact canonical order
        # float-mode values are multiples of 2^-23 with |sum| <= 128: fp64 is exact, fp32 close
        assert np.max(np.abs(got[r] - ref64[r])) <= 8 * 2.0 ** -23 * max(pmax, 1)


def test_p1_pool_table_matches_sequential_loop():
    rng = np.random.default_rng(0)
    W = rng.standard_normal((50, 8)).astype(np.float32)
    L = rng.integers(0, 40, size=30)
    off = np.concatenate([[0], np.cumsum(L)])
    idx = rng.integers(0, 50, size=off[-1])
    Z = O.pool_table_f32(W, off, idx)
    for b in range(30):
        ref = O.pool_bag_f32(W[idx[off[b]:off[b + 1]]])
        assert np.array_equal(Z[b].view(np.uint32), ref.view(np.uint32))
        # and the plain-Python loop, not numpy vector adds
        acc = None
        for j in range(off[b], off[b + 1]):
            acc = W[idx[j]].copy() if acc is None else np.array([np.float32(a + c) for a, c in zip(acc, W[idx[j]])], dtype=np.float32)
        if acc is None:
            acc = np.zeros(8, np.float32)
        assert np.array_equal(Z[b].view(np.uint32), acc.view(np.uint32))


def test_p2_one_hot_returns_row_bits_including_negative_zero():
    W = np.array([[1.5, -0.0, 3.0e-38, -2.25], [0.0, 1.0, -1.0, 7.0]], dtype=np.float32)
    off = np.array([0, 1, 2])
    idx = np.array([0, 1])
    Z = O.pool_table_f32(W, off, idx)
    assert np.array_equal(Z.view(np.uint32), W.view(np.uint32))
    assert np.signbit(Z[0, 1])  # -0.0 survives: accumulator starts at the first row (C4)


def test_p3_empty_bag_is_positive_zero():
    W = -np.ones((5, 4), dtype=np.float32)
    off = np.array([0, 0, 2, 2, 2])
    idx = np.array([1, 3])
    Z = O.pool_table_f32(W, off, idx)
    for b in (0, 2, 3):
        assert np.all(Z[b] == 0) and not np.any(np.signbit(Z[b]))
    assert np.all(Z[1] == -2)


@pytest.mark.parametrize("k", [1, 2, 7, 128])
def test_p4_duplicate_rows_scale(k):
    W = synth.table_rows(3, 0, 20, 16, "int")
    off = np.array([0, k])
    idx = np.full(k, 13)
    Z = O.pool_table_f32(W, off, idx)
    assert np.array_equal(Z[0], k * W[13])


def test_p5_integer_tables_exact_any_order():
    w = synth.make_workload("tiny", G=2, mode="int", pmin=1, pmax=128, B=64)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 5)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G)
    # fp64 per table, reversed order: must equal exactly (|sum| <= 8*128 << 2^24)
    for r in range(w.G):
        for tl, t in enumerate(w.local_tables(r)):
            o, lo, hi = O.rank_table_csr(offs[r], tl, w.B)
            x = idxs[r][lo:hi]
            for b in range(w.B):
                rows = tabs[t][x[o[b]:o[b + 1]]][::-1].astype(np.float64)
                ref = rows.sum(axis=0) if rows.size else np.zeros(w.dim)
                dst = int(np.searchsorted(np.array(O.split_batch(w.B, w.G)[0]), b, side="right") - 1)
                i = b - O.split_batch(w.B, w.G)[0][dst]
                assert np.array_equal(Y[dst][i, t].astype(np.float64), ref)


def test_p6_identity_routing():
    """Identity-encoded rows + one-hot bags: every output slot decodes to (t, row)."""
    G = 3
    w = synth.make_workload("tiny", G=G, mode="identity", pmin=1, pmax=1, B=30, T=7)
    w.owner = np.array([2, 0, 1, 1, 0, 2, 2], dtype=np.int32)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 9)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, G)
    starts, counts = O.split_batch(w.B, G)
    for r in range(G):
        for i in range(counts[r]):
            b = starts[r] + i
            for t in range(w.T):
                v = Y[r][i, t]
                assert int(v[0]) + 256 * int(v[1]) == t
                row = int(v[2]) + (int(v[3]) << 8) + (int(v[4]) << 16)
                # the one index of bag (t, b) regenerated from the generator directly
                exp = synth.table_indices(9, t, np.array([b]), int(w.rows[t]), w.dist, w.alpha, perm_seed=w.table_seed)[0]
                assert row == exp


@pytest.mark.parametrize("k", [3, -5])
def test_p7_power_of_two_scaling(k):
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=40)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 21)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G)
    Ys = O.emb_forward([t * np.float32(2.0 ** k) for t in tabs], w.owner, offs, idxs, w.B, w.G)
    for a, b in zip(Y, Ys):
        assert np.array_equal((a * np.float32(2.0 ** k)).view(np.uint32), b.view(np.uint32))


def test_p8_linearity_and_bag_concat():
    w = synth.make_workload("tiny", G=2, mode="int", pmin=0, pmax=30)
    t1 = _tables(w)
    w2 = synth.make_workload("tiny", G=2, mode="int", pmin=0, pmax=30, table_seed=777)
    t2 = _tables(w2)
    offs, idxs = _csrs(w, 4)
    Y1 = O.emb_forward(t1, w.owner, offs, idxs, w.B, w.G)
    Y2 = O.emb_forward(t2, w.owner, offs, idxs, w.B, w.G)
    Y12 = O.emb_forward([a + b for a, b in zip(t1, t2)], w.owner, offs, idxs, w.B, w.G)
    for a, b, c in zip(Y1, Y2, Y12):
        assert np.array_equal(a + b, c)
    # bag concatenation: pool(bag_a ++ bag_b) = pool(bag_a) + pool(bag_b)
    W = t1[0]
    a_idx, b_idx = np.array([1, 5, 9]), np.array([9, 2])
    za = O.pool_table_f32(W, np.array([0, 3]), a_idx)
    zb = O.pool_table_f32(W, np.array([0, 2]), b_idx)
    zab = O.pool_table_f32(W, np.array([0, 5]), np.concatenate([a_idx, b_idx]))
    assert np.array_equal(za + zb, zab)


def test_p9_placement_invariance():
    base = synth.make_workload("tiny", G=2, pmin=0, pmax=50, T=6)
    owners = [np.array([0, 0, 0, 1, 1, 1]), np.array([0, 1, 0, 1, 0, 1]), np.array([1, 1, 0, 1, 0, 0]),
              np.array([0] * 6), np.array([1] * 6)]
    ref = None
    for own in owners:
        w = synth.make_workload("tiny", G=2, pmin=0, pmax=50, T=6, owner=own)
        tabs = _tables(w)
        offs, idxs = _csrs(w, 77)
        Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G)
        cat = np.concatenate(Y)
        if ref is None:
            ref = cat
        assert np.array_equal(cat.view(np.uint32), ref.view(np.uint32))
    assert base.T == 6


@pytest.mark.parametrize("G", [2, 3, 5])
def test_p10_concat_equals_single_rank(G):
    w1 = synth.make_workload("tiny", G=1, pmin=0, pmax=20, B=37, T=5)
    wg = synth.make_workload("tiny", G=G, pmin=0, pmax=20, B=37, T=5, owner=np.array([G - 1] * 5))  # ranks < G-1 own no tables (C22)
    tabs = _tables(w1)
    o1, x1 = _csrs(w1, 3)
    og, xg = _csrs(wg, 3)
    Y1 = O.emb_forward(tabs, w1.owner, o1, x1, w1.B, 1)[0]
    Yg = O.emb_forward(tabs, wg.owner, og, xg, wg.B, G)
    assert [y.shape[0] for y in Yg] == O.split_batch(37, G)[1]
    assert np.array_equal(np.concatenate(Yg).view(np.uint32), Y1.view(np.uint32))


def test_p11_matches_torch_embedding_bag():
    torch = pytest.importorskip("torch")
    w = synth.make_workload("tiny", G=1, pmin=0, pmax=64, B=200, dim=32)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 8)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, 1)[0]
    for t in range(w.T):
        o, lo, hi = O.rank_table_csr(offs[0], t, w.B)
        ref = torch.nn.functional.embedding_bag(torch.from_numpy(idxs[0][lo:hi]), torch.from_numpy(tabs[t]),
                                                torch.from_numpy(o[:-1]), mode="sum").numpy()
        Z64, S = O.pool_table_f64(tabs[t], o, idxs[0][lo:hi])
        assert O.s_normalized_error(Y[:, t], ref, S) <= 1e-6
        assert O.s_normalized_error(Y[:, t], Z64, S) <= 1e-6
    # integer tables: exact equality with the library routine
    wi = synth.make_workload("tiny", G=1, mode="int", pmin=0, pmax=64, B=200, dim=32)
    ti = _tables(wi)
    Yi = O.emb_forward(ti, wi.owner, offs, idxs, wi.B, 1)[0]
    for t in range(wi.T):
        o, lo, hi = O.rank_table_csr(offs[0], t, wi.B)
        ref = torch.nn.functional.embedding_bag(torch.from_numpy(idxs[0][lo:hi]), torch.from_numpy(ti[t]),
                                                torch.from_numpy(o[:-1]), mode="sum").numpy()
        assert np.array_equal(Yi[:, t], ref)


def test_p13_conservation_integer():
    w = synth.make_workload("tiny", G=3, mode="int", pmin=0, pmax=40, B=50, T=7)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 2)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G)
    total = sum(float(y.astype(np.float64).sum()) for y in Y)
    ref = 0.0
    for r in range(w.G):
        for tl, t in enumerate(w.local_tables(r)):
            o, lo, hi = O.rank_table_csr(offs[r], tl, w.B)
            ref += float(tabs[t][idxs[r][lo:hi]].astype(np.float64).sum())
    assert total == ref


def test_p15_paper_fig3_fig4_structure():
    g = json.load(open(os.path.join(GOLDEN, "fig3_fig4.json")))
    M, d, N = g["M"], g["d"], g["N"]
    i = np.arange(M)[:, None]
    k = np.arange(d)[None, :]
    tabs = [(1000 * t + 10 * i + k).astype(np.float32) for t in range(2)]
    bags = [g["bags"]["feature1"], g["bags"]["feature2"]]
    exp = np.array(g["expected_G1"], dtype=np.float32)
    # G = 1
    o = [0]
    x = []
    for t in range(2):
        for bag in bags[t]:
            x += bag
            o.append(len(x))
    Y1 = O.emb_forward(tabs, [0, 0], [np.array(o)], [np.array(x)], N, 1)[0]
    assert np.array_equal(Y1, exp)
    # G = 2, Fig. 4: feature 1 on GPU 0, feature 2 on GPU 1; each GPU pools its feature for the FULL batch
    ro, rx = [], []
    for t in range(2):
        oo, xx = [0], []
        for bag in bags[t]:
            xx += bag
            oo.append(len(xx))
        ro.append(np.array(oo))
        rx.append(np.array(xx, dtype=np.int64))
    Y2 = O.emb_forward(tabs, g["owner"], ro, rx, N, 2)
    assert np.array_equal(Y2[0], exp[g["expected_G2"]["rank0_samples"]])
    assert np.array_equal(Y2[1], exp[g["expected_G2"]["rank1_samples"]])
    assert np.all(Y2[1][0, 1] == 0)  # sample 3's NULL feature-2 input (L89)


def test_bf16_rounding_matches_torch():
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(1)
    x = rng.standard_normal(100000).astype(np.float32) * 100
    # exact ties and near-ties
    ties = (np.arange(1, 5000, dtype=np.uint32) << 16 | 0x8000).view(np.float32)
    x = np.concatenate([x, ties, -ties, (ties.view(np.uint32) + 1).view(np.float32)])
    ref = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(O.rne_bf16(x), ref)
    assert np.array_equal(O.bf16_to_f32(ref), torch.from_numpy(ref.view(np.int16)).view(torch.bfloat16).float().numpy())


def test_bf16_tables_tolerance():
    w = synth.make_workload("tiny", G=2, wdtype="bf16", odtype="bf16", pmin=1, pmax=100, dim=32)
    tabs_f = _tables(w)
    tabs = [synth.to_bf16_bits(t) for t in tabs_f]
    offs, idxs = _csrs(w, 6)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G, out_dtype="bf16", table_is_bf16=True)
    Yf = O.emb_forward(tabs_f, w.owner, offs, idxs, w.B, w.G)
    for a, b in zip(Y, Yf):
        assert np.array_equal(a, O.rne_bf16(b))
        # S-normalised tolerance of the north star (1e-2) vs fp64
    for r in range(w.G):
        for tl, t in enumerate(w.local_tables(r)):
            o, lo, hi = O.rank_table_csr(offs[r], tl, w.B)
            Z64, S = O.pool_table_f64(tabs_f[t], o, idxs[r][lo:hi])
            Yall = np.concatenate([O.bf16_to_f32(y) for y in Y])
            assert O.s_normalized_error(Yall[:, t], Z64, S) <= 1e-2


def test_validate_rejects_bad_csr():
    W = np.zeros((4, 4), np.float32)
    with pytest.raises(ValueError):
        O.pool_table_f32(W, np.array([0, 2, 1]), np.array([0]))
    with pytest.raises(ValueError):
        O.pool_table_f32(W, np.array([0, 1]), np.array([4]))
    with pytest.raises(ValueError):
        O.pool_table_f32(W, np.array([1, 1]), np.array([0]))


def test_split_batch_rule():
    assert O.split_batch(10, 3) == ([0, 4, 7], [4, 3, 3])
    assert O.split_batch(16384 * 8, 8)[1] == [16384] * 8


# ------------------------------------------------------------------------------- backward (f2)
def _dY(w, seed, integer=True):
    rng = np.random.default_rng(seed)
    starts, counts = O.split_batch(w.B, w.G)
    if integer:
        return [rng.integers(-8, 9, size=(counts[r], w.T, w.dim)).astype(np.float32) for r in range(w.G)]
    return [rng.standard_normal((counts[r], w.T, w.dim)).astype(np.float32) for r in range(w.G)]


def test_bwd_bruteforce():
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=5, B=9, T=3, dim=4, rows=7)
    offs, idxs = _csrs(w, 3)
    dY = _dY(w, 1, integer=False)
    dW, S, cnt = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    starts, counts = O.split_batch(w.B, w.G)
    for t in range(w.T):
        o = int(w.owner[t])
        tl = list(w.local_tables(o)).index(t)
        ref = [[0.0] * w.dim for _ in range(int(w.rows[t]))]
        for b in range(w.B):
            r = max(i for i in range(w.G) if starts[i] <= b)
            lo, hi = int(offs[o][tl * w.B + b]), int(offs[o][tl * w.B + b + 1])
            for j in range(lo, hi):
                for k in range(w.dim):
                    ref[int(idxs[o][j])][k] += float(dY[r][b - starts[r], t, k])
        assert np.allclose(dW[t], np.array(ref), rtol=0, atol=1e-12)


def test_bwd_adjoint_identity():
    """<pool(W), dY> == <W, dW> : the backward is the exact transpose of the forward."""
    w = synth.make_workload("tiny", G=3, mode="int", pmin=0, pmax=30, B=40, T=5, dim=8, rows=50)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 8)
    Y = O.emb_forward(tabs, w.owner, offs, idxs, w.B, w.G)
    dY = _dY(w, 2)
    dW, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, w.G)
    lhs = sum(float((Y[r].astype(np.float64) * dY[r]).sum()) for r in range(w.G))
    rhs = sum(float((tabs[t].astype(np.float64) * dW[t]).sum()) for t in range(w.T))
    assert lhs == rhs


def test_bwd_matches_torch_autograd():
    torch = pytest.importorskip("torch")
    w = synth.make_workload("tiny", G=1, pmin=0, pmax=20, B=30, T=2, dim=8, rows=40)
    tabs = _tables(w)
    offs, idxs = _csrs(w, 4)
    dY = _dY(w, 5, integer=False)
    dW, _, cnt = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, dY, w.B, 1)
    for t in range(w.T):
        o, lo, hi = O.rank_table_csr(offs[0], t, w.B)
        Wt = torch.from_numpy(tabs[t].astype(np.float64)).requires_grad_(True)
        y = torch.nn.functional.embedding_bag(torch.from_numpy(idxs[0][lo:hi]), Wt, torch.from_numpy(o[:-1]), mode="sum")
        y.backward(torch.from_numpy(dY[0][:, t].astype(np.float64)))
        assert np.allclose(Wt.grad.numpy(), dW[t], rtol=1e-12, atol=1e-12)
        assert cnt[t].sum() == hi - lo


def test_bwd_placement_invariance():
    outs = []
    for own in ([0, 0, 1, 1, 1], [1, 0, 1, 0, 1], [1, 1, 1, 1, 1]):
        w = synth.make_workload("tiny", G=2, pmin=0, pmax=9, B=21, T=5, dim=4, rows=30, owner=np.array(own))
        offs, idxs = _csrs(w, 6)
        dW, _, _ = O.emb_backward(w.rows, w.dim, w.owner, offs, idxs, _dY(w, 9), w.B, w.G)
        outs.append(dW)
    for d in outs[1:]:
        for a, b in zip(d, outs[0]):
            assert np.array_equal(a, b)


# ------------------------------------------------------------------------------- row-wise sharding (f3)
def _sharded_inputs(w, seed, shards):
    """Per rank: for each local shard (ascending (t, s)) the FULL CSR of table t."""
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


def _even_shards(w, nshard_of, owners_of):
    sh = []
    for t in range(w.T):
        S = nshard_of(t)
        cuts = np.linspace(0, int(w.rows[t]), S + 1).astype(int)
        for s in range(S):
            sh.append((t, s, int(cuts[s]), int(cuts[s + 1]), owners_of(t, s)))
    return sh


def test_f3_single_shard_equals_tablewise():
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=20, B=33, T=4, dim=8, rows=200)
    tabs = _tables(w)
    shards = [(t, 0, 0, int(w.rows[t]), int(w.owner[t])) for t in range(w.T)]
    offs, idxs = _sharded_inputs(w, 4, shards)
    Ys = O.emb_forward_sharded(tabs, shards, offs, idxs, w.B, w.G)
    o2, x2 = _csrs(w, 4)
    Y = O.emb_forward(tabs, w.owner, o2, x2, w.B, w.G)
    for a, b in zip(Ys, Y):
        assert np.array_equal(a.view(np.uint32), b.view(np.uint32))


def test_f3_integer_exact_and_bruteforce():
    w = synth.make_workload("tiny", G=3, mode="int", pmin=0, pmax=40, B=29, T=3, dim=4, rows=90)
    tabs = _tables(w)
    shards = _even_shards(w, lambda t: t + 1, lambda t, s: (t + s) % 3)
    offs, idxs = _sharded_inputs(w, 7, shards)
    Ys = O.emb_forward_sharded(tabs, shards, offs, idxs, w.B, w.G)
    starts, counts = O.split_batch(w.B, w.G)
    for r in range(w.G):
        for i in range(counts[r]):
            b = starts[r] + i
            for t in range(w.T):
                o, x = synth.table_csr(w, 7, t)
                ref = sum((tabs[t][int(v)].astype(np.float64) for v in x[o[b]:o[b + 1]]), np.zeros(w.dim))
                assert np.array_equal(Ys[r][i, t].astype(np.float64), ref)


def test_f3_shard_order_sum_and_tolerance():
    """Float data: the sharded result is the shard-order sum of canonical partials (not the
    unsharded canonical order) and stays within the S-normalised 1e-6 of the fp64 sum."""
    w = synth.make_workload("tiny", G=2, pmin=1, pmax=100, B=40, T=2, dim=16, rows=500)
    tabs = _tables(w)
    shards = _even_shards(w, lambda t: 4, lambda t, s: s % 2)
    offs, idxs = _sharded_inputs(w, 9, shards)
    Ys = np.concatenate(O.emb_forward_sharded(tabs, shards, offs, idxs, w.B, w.G))
    for t in range(w.T):
        o, x = synth.table_csr(w, 9, t)
        z64, S = O.pool_table_f64(tabs[t], o, x)
        assert O.s_normalized_error(Ys[:, t], z64, S) <= 1e-6
        cuts = np.linspace(0, int(w.rows[t]), 5).astype(int)
        for b in range(w.B):
            xb = x[o[b]:o[b + 1]]
            parts = [O.pool_bag_f32(tabs[t][xb[(xb >= cuts[s]) & (xb < cuts[s + 1])]]) for s in range(4)]
            acc = parts[0]
            for p_ in parts[1:]:
                acc = acc + p_
            assert np.array_equal(acc.view(np.uint32), Ys[b, t].view(np.uint32))


# ----------------------------------------------------------------------------- S-normalised metric
def test_s_normalized_error_and_S_hand_fixture():
    """s_normalized_error and S = sum |w| (the tolerance denominator of every float
    assertion) against hand-derived values: cancellation, a 0/0 element (-> 0), a nonzero
    diff over S = 0 (-> inf), and max over elements (not the mean)."""
    g = json.load(open(os.path.join(GOLDEN, "s_normalized_error.json")))
    x = float.fromhex
    rows = np.array([[x(v) for v in r] for r in g["rows"]], dtype=np.float32)
    z, S = O.pool_bag_f64(rows)
    assert np.array_equal(z, np.array([x(v) for v in g["bag_sum"]]))
    assert np.array_equal(S, np.array([x(v) for v in g["bag_S"]]))
    offs = np.array(g["table_offsets"], dtype=np.int64)
    Zt, St = O.pool_table_f64(rows, offs, np.arange(3, dtype=np.int64))
    assert np.array_equal(Zt, np.array([[x(v) for v in r] for r in g["table_sum"]]))
    assert np.array_equal(St, np.array([[x(v) for v in r] for r in g["table_S"]]))
    for c in g["cases"]:
        y = np.array([x(v) for v in c["y"]])
        with np.errstate(all="ignore"):
            got = O.s_normalized_error(y, z, S)
        if "expected" in c:
            exp = float("inf") if c["expected"] == "inf" else x(c["expected"])
        else:
            exp = x(c["expected_num"]) / x(c["expected_den"])
        assert got == exp, (c["what"], got, exp)


# ----------------------------------------------------------------------------- C7: IEEE specials
def test_c7_subnormal_sums_not_flushed():
    """C7 (no FTZ): rows of small multiples of the least subnormal 2^-149 sum exactly
    (sum_k k * 2^-149 is representable), including sums that stay subnormal and sums
    that cross into the normal range; a flush-to-zero implementation returns 0."""
    tiny = np.float32(2.0 ** -149)
    k = np.array([[1, 3, 7, 2 ** 20], [2, 5, 9, 2 ** 22], [4, 0, 1, 2 ** 23]], dtype=np.int64)
    W = (k.astype(np.float64) * 2.0 ** -149).astype(np.float32)
    assert W[0, 0] == tiny and W[2, 3] == np.float32(2.0 ** -126)   # subnormal .. least normal
    offs = np.array([0, 3, 5], dtype=np.int64)
    idx = np.array([0, 1, 2, 0, 0], dtype=np.int64)
    Z = O.pool_table_f32(W, offs, idx)
    exp = np.array([k.sum(axis=0), 2 * k[0]], dtype=np.float64) * 2.0 ** -149
    assert np.array_equal(Z.astype(np.float64), exp)
    assert np.all(Z[:, :3] > 0) and np.all(Z[:, :3] < 2.0 ** -126)     # still subnormal, not flushed


def test_c7_inf_nan_propagate_and_negative_zero():
    """C7 closed forms of IEEE 754 addition: x + Inf = Inf, Inf + (-Inf) = NaN, NaN + x = NaN,
    overflow of a finite sum -> Inf, (-0) + (-0) = -0 (a bag of -0 rows returns -0, C4)."""
    big = np.float32(3.0e38)
    W = np.array([[1.0, np.inf, np.nan, big, -0.0],
                  [2.0, -np.inf, 1.0, big, -0.0]], dtype=np.float32)
    offs = np.array([0, 1, 3], dtype=np.int64)
    with np.errstate(all="ignore"):
        Z = O.pool_table_f32(W, offs, np.array([0, 0, 1], dtype=np.int64))
    keep = [0, 1, 3, 4]                                                  # one-hot bag: the row's bits
    assert np.array_equal(Z[0, keep].view(np.uint32), W[0, keep].view(np.uint32)) and np.isnan(Z[0, 2])
    assert Z[1, 0] == 3.0 and np.isnan(Z[1, 1]) and np.isnan(Z[1, 2]) and Z[1, 3] == np.inf
    assert Z[1, 4] == 0 and np.signbit(Z[1, 4])


def test_c7_bf16_rounding_of_specials_matches_torch():
    """rne_bf16 on NaN / +-Inf / subnormals / overflowing finites: NaN stays NaN (the plain
    rounding rule would turn a low-payload NaN into Inf), everything else bit-equal to
    torch's float -> bf16 conversion."""
    torch = pytest.importorskip("torch")
    u = np.array([0x7F800001, 0xFF800001, 0x7FC00000, 0x7F800000, 0xFF800000, 0x00000001, 0x80000001,
                  0x00007FFF, 0x00008000, 0x00018000, 0x007FFFFF, 0x7F7FFFFF, 0x7F7F8000, 0xFF7FFFFF,
                  0x80000000, 0x00000000], dtype=np.uint32)
    x = u.view(np.float32)
    got = O.rne_bf16(x)
    ref = torch.from_numpy(x.copy()).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    nan = np.isnan(x)
    assert np.all(np.isnan(O.bf16_to_f32(got[nan])))
    assert np.array_equal(got[~nan], ref[~nan])
    assert got[3] == 0x7F80 and got[4] == 0xFF80 and got[11] == 0x7F80     # Inf, -Inf, overflow -> Inf
