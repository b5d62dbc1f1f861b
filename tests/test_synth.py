"""Input-generator checks (CPU).  The generators are shared by both sides, so they
are checked against the distributions the paper / north star name, not against
either implementation."""
import math

import numpy as np
import pytest

import synth


def test_hash_is_counter_based_and_deterministic():
    a = synth.hash3(synth.S_INDEX, 5, 3, np.arange(100))
    b = synth.hash3(synth.S_INDEX, 5, 3, np.arange(100))
    assert np.array_equal(a, b)
    assert np.array_equal(synth.hash3(synth.S_INDEX, 5, 3, np.arange(40, 60)), a[40:60])
    assert len(set(a.tolist())) == 100
    assert not np.array_equal(a, synth.hash3(synth.S_INDEX, 6, 3, np.arange(100)))
    assert not np.array_equal(a, synth.hash3(synth.S_POOL, 5, 3, np.arange(100)))


def test_table_values_exact_and_in_range():
    W = synth.table_rows(1, 0, 2000, 16, "float", "f32")
    assert W.dtype == np.float32 and np.all(W >= -1) and np.all(W < 1)
    q = W.astype(np.float64) * 2 ** 23
    assert np.array_equal(q, np.round(q))          # multiples of 2^-23
    assert not np.any((W == 0) & np.signbit(W))    # no -0.0 (C7)
    assert abs(W.mean()) < 0.02 and 0.3 < W.std() < 0.7
    Wb = synth.table_rows(1, 0, 2000, 16, "float", "bf16")
    bits = synth.to_bf16_bits(Wb)                  # raises if not representable
    assert np.array_equal(synth.bf16_bits_to_f32(bits), Wb)
    Wi = synth.table_rows(1, 0, 2000, 16, "int")
    assert set(np.unique(Wi).tolist()) == set(range(-8, 9))
    # row subset == full-table rows (counter-based)
    rows = np.array([7, 1999, 0, 7])
    assert np.array_equal(synth.table_values(1, 0, rows, 16), W[rows])


def test_identity_tables_encode_table_and_row():
    W = synth.table_values(0, 300, np.array([0, 70000, 16777215]), 8, "identity")
    assert W[1, 0] + 256 * W[1, 1] == 300
    assert int(W[1, 2]) + (int(W[1, 3]) << 8) + (int(W[1, 4]) << 16) == 70000
    assert int(W[2, 2]) + (int(W[2, 3]) << 8) + (int(W[2, 4]) << 16) == 16777215


@pytest.mark.parametrize("M", [1000, 1024, 999983, 2_000_000])
def test_perm_is_bijection(M):
    a, c = synth.perm_params(20241119, 3, M)
    assert math.gcd(a, M) == 1 and 0 <= c < M
    if M <= 1024:
        k = np.arange(M)
        assert len(set(((a * k + c) % M).tolist())) == M


def test_zipf_distribution():
    M, s = 1_000_000, 1.05
    x = synth.table_indices(42, 0, np.arange(400_000), M, "zipf", s, perm_seed=1)
    assert x.min() >= 0 and x.max() < M
    a, c = synth.perm_params(1, 0, M)
    # invert the bijection to ranks and compare the head of the rank histogram
    ainv = pow(a, -1, M)
    k0 = ((x - c) % M) * ainv % M
    H = np.sum(np.arange(1, M + 1, dtype=np.float64) ** -s)
    for r in range(5):
        p = (r + 1) ** -s / H
        f = np.mean(k0 == r)
        assert abs(f - p) < 5 * math.sqrt(p * (1 - p) / x.size) + 1e-4, (r, f, p)
    # heavy tail: fraction of distinct rows is far below uniform's
    assert np.unique(x).size < 0.5 * x.size


def test_uniform_distribution():
    x = synth.table_indices(42, 0, np.arange(200_000), 1000, "uniform")
    h = np.bincount(x, minlength=1000)
    chi2 = np.sum((h - 200.0) ** 2 / 200.0)
    assert chi2 < 1000 + 6 * math.sqrt(2000)


def test_pooling_lengths():
    L = synth.pooling_lengths(3, 1, 100000, 1, 128)
    assert L.min() == 1 and L.max() == 128 and abs(L.mean() - 64.5) < 0.5
    assert np.all(synth.pooling_lengths(3, 1, 10, 20, 20) == 20)


def test_rank_csr_is_table_major_and_placement_free():
    w2 = synth.make_workload("tiny", G=2, pmin=0, pmax=9, T=5)
    o0, x0 = synth.rank_csr(w2, 17, 0)
    o1, x1 = synth.rank_csr(w2, 17, 1)
    assert o0.size == len(w2.local_tables(0)) * w2.B + 1 and o0[-1] == x0.size and np.all(np.diff(o0) >= 0)
    # table 3's bags are identical whichever rank owns it
    w1 = synth.make_workload("tiny", G=1, pmin=0, pmax=9, T=5)
    oa, xa = synth.rank_csr(w1, 17, 0)
    tl1 = list(w2.local_tables(1)).index(3)
    seg2 = x1[o1[tl1 * w2.B]:o1[(tl1 + 1) * w2.B]]
    seg1 = xa[oa[3 * w1.B]:oa[4 * w1.B]]
    assert np.array_equal(seg1, seg2)


def test_workload_shapes():
    w = synth.make_workload("weak", G=8)
    assert w.T == 208 and w.B == 131072 and len(w.local_tables(3)) == 26
    s = synth.make_workload("strong", G=1)
    assert s.T == 208 and int(s.phys.max()) == 103          # C27 aliasing
    L = synth.make_workload("large", G=8)
    tb = [int(L.rows[L.owner == r].sum()) * 256 * 2 for r in range(8)]
    assert 1.15e12 < sum(tb) < 1.25e12 and max(tb) < 160e9
    assert [len(L.local_tables(r)) for r in range(8)] == [64] * 8
    st, ct = synth.batch_split(10, 4)
    assert st.tolist() == [0, 3, 6, 8] and ct.tolist() == [3, 3, 2, 2]
