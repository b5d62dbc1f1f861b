"""GPU parity: libemb.so (through the C ABI) vs the CPU oracle, element by element.

Bar (BASELINE.json north_star): bit-exact for placement/indices; fp32 values within
S-normalised 1e-6, bf16 within 1e-2.  The kernel keeps the canonical CSR summation
order (C4), so it is additionally required to be BIT-EXACT to the canonical oracle.
"""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import synth
from oracle import emb_oracle as O
import emb_test_helpers as H

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_sc_chenbyo24_b200 import emb as E  # noqa: E402
from paper_conf_sc_chenbyo24_b200.comm import LocalGroup, run_ranks  # noqa: E402
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding  # noqa: E402

DEV = torch.device("cuda", 0)


def _dev_tables(w, tabs_np, r):
    out = []
    for t in w.local_tables(r):
        a = tabs_np[int(w.phys[t])]
        if w.wdtype == "bf16":
            out.append(torch.from_numpy(synth.to_bf16_bits(a).view(np.int16)).to(DEV).view(torch.bfloat16))
        else:
            out.append(torch.from_numpy(a).to(DEV))
    return out


def _layers(w, tabs_np, options=None):
    """One PgasEmbedding per simulated rank (single process, one GPU)."""
    tabs_dev = [_dev_tables(w, tabs_np, r) for r in range(w.G)]
    if w.G == 1:
        return [PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tabs_dev[0], w.B, w.wdtype, w.odtype, None, options)]
    grp = LocalGroup(w.G)
    return run_ranks(w.G, lambda r: PgasEmbedding(r, w.G, 0, w.rows, w.owner, w.dim, tabs_dev[r], w.B, w.wdtype,
                                                  w.odtype, grp.allgather_for(r), options))


def _run(w, layers, csr_np, flags=0, streams=None, i32=False):
    offs, idxs = csr_np
    dt = torch.int32 if i32 else torch.int64
    dev_in = [(torch.from_numpy(offs[r]).to(DEV).to(dt), torch.from_numpy(idxs[r]).to(DEV).to(dt)) for r in range(w.G)]
    streams = streams or [torch.cuda.Stream() for _ in range(w.G)]
    torch.cuda.synchronize()
    ys = []
    for r in range(w.G):
        ys.append(layers[r].forward(dev_in[r][0], dev_in[r][1], flags, streams[r]))
    if flags & E.EMB_FWD_SEPARATE_WAIT:
        for r in range(w.G):
            layers[r].wait(streams[r])
    torch.cuda.synchronize()
    return [H.dev_out_to_np(y.clone()) for y in ys]


def _close(layers):
    if len(layers) == 1:
        layers[0].close()
    else:
        run_ranks(len(layers), lambda r: layers[r].close())


def _assert_exact(got, ref):
    assert got.shape == ref.shape
    gb, rb = H.bits(got), H.bits(ref)
    if not np.array_equal(gb, rb):
        bad = np.argwhere(gb != rb)
        raise AssertionError(f"{len(bad)} mismatches, first at {bad[0].tolist()}: got {got[tuple(bad[0])]} "
                             f"want {ref[tuple(bad[0])]}")


# ------------------------------------------------------------------------------- G = 1
CASES = [
    # name, overrides
    ("tiny", dict()),
    ("tiny", dict(pmin=0, pmax=9, B=1000, T=5, rows=777)),          # empty bags, ragged chunks
    ("tiny", dict(dim=64, pmin=1, pmax=128, B=300, rows=5000)),      # 256-B rows (LDG.64 path)
    ("tiny", dict(dim=128, pmin=0, pmax=40, B=513, rows=3000, dist="zipf")),
    ("tiny", dict(dim=256, pmin=1, pmax=20, B=257, rows=999)),       # 1-KB rows (2 vectors per lane)
    ("tiny", dict(dim=8, pmin=1, pmax=7, B=100)),                    # 32-B rows (2 active lanes)
    ("tiny", dict(dim=512, pmin=1, pmax=5, B=65, rows=100)),         # 2-KB rows
    ("tiny", dict(dim=128, wdtype="bf16", odtype="bf16", pmin=1, pmax=100, B=200, rows=4000)),
    ("tiny", dict(dim=256, wdtype="bf16", odtype="bf16", pmin=0, pmax=60, B=130, rows=4000)),
    ("tiny", dict(dim=64, wdtype="f32", odtype="bf16", pmin=1, pmax=33, B=200)),
    ("tiny", dict(dim=64, wdtype="bf16", odtype="f32", pmin=1, pmax=33, B=200)),
    ("tiny", dict(dim=16, pmin=1, pmax=1, B=64, T=3)),               # one-hot bags
]


@pytest.mark.parametrize("name,over", CASES)
def test_g1_bitexact_vs_oracle(name, over):
    w = synth.make_workload(name, G=1, **over)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 101)
    ref = H.oracle_outputs(w, 101, tabs, csr)
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, csr)
    finally:
        _close(layers)
    _assert_exact(got[0], ref[0])


def test_integer_tables_exact_and_tolerance_metric():
    w = synth.make_workload("tiny", G=1, mode="int", pmin=0, pmax=128, B=700, T=6, dim=64)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 5)
    ref = H.oracle_outputs(w, 5, tabs, csr)
    layers = _layers(w, tabs)
    got = _run(w, layers, csr)
    _close(layers)
    _assert_exact(got[0], ref[0])
    # and the north-star metric against fp64 for a float workload
    w = synth.make_workload("tiny", G=1, pmin=1, pmax=128, B=300, T=3, dim=32, rows=2000)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 6)
    layers = _layers(w, tabs)
    got = _run(w, layers, csr)[0]
    _close(layers)
    for t in range(w.T):
        o, lo, hi = O.rank_table_csr(csr[0][0], t, w.B)
        z64, S = O.pool_table_f64(tabs[t], o, csr[1][0][lo:hi])
        assert O.s_normalized_error(got[:, t], z64, S) <= 1e-6


def test_identity_routing_and_negative_zero():
    w = synth.make_workload("tiny", G=1, mode="identity", pmin=1, pmax=1, B=50, T=4)
    tabs = H.np_tables(w)
    tabs[2][:] = -0.0  # one-hot of a -0.0 row must return -0.0 bits (C4, P2)
    csr = H.np_csrs(w, 3)
    ref = H.oracle_outputs(w, 3, tabs, csr)
    layers = _layers(w, tabs)
    got = _run(w, layers, csr)[0]
    _close(layers)
    _assert_exact(got, ref[0])
    assert np.all(np.signbit(got[:, 2]))


# ------------------------------------------------------------------------------- simulated G > 1
@pytest.mark.parametrize("G,flags", [(2, 0), (3, 0), (2, 2), (4, 2)])
def test_simulated_ranks_bitexact(G, flags):
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=30, B=101, T=7, dim=32, rows=500)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 12)
    ref = H.oracle_outputs(w, 12, tabs, csr)
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, csr, flags)
        for r in range(G):
            _assert_exact(got[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)


def test_simulated_ranks_max_world_size():
    """kMaxG = 16 simulated ranks (the largest world size the kernel parameters carry):
    every rank owns one or two tables, uneven mini-batches (B mod G != 0), remote stores to
    15 peers, flags from 15 sources; bit-exact; a 17th rank is refused."""
    G = 16
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=9, B=16 * 7 + 5, T=24, dim=32, rows=200)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 23)
    ref = H.oracle_outputs(w, 23, tabs, csr)
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, csr)
        for r in range(G):
            _assert_exact(got[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)
    with pytest.raises(E.EmbError):
        E.emb_init(0, 17, 0, lambda b: b * 17)


@pytest.mark.parametrize("G,wdt,i32", [(4, "f32", False), (8, "f32", True), (3, "bf16", False)])
def test_simulated_ranks_medium_size_bitexact(G, wdt, i32):
    """Multi-rank parity beyond tiny shapes: G ranks (up to the 8 of the scaling run) with
    16-32 tables of 40 K rows, d = 128, 2-4 K samples and pooling up to 128, LPT-like mixed
    placement, zipf ids: every element bit-exact (remote stores, chunks crossing rank
    boundaries of the mini-batch, destination-staggered order)."""
    T = 4 * G
    rng = np.random.default_rng(G)
    owner = rng.permutation(np.arange(T) % G)
    w = synth.make_workload("tiny", G=G, pmin=1, pmax=128, B=512 * G + 3, T=T, dim=128, rows=40000, dist="zipf",
                            wdtype=wdt, odtype=wdt, owner=owner)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 61)
    ref = H.oracle_outputs(w, 61, tabs, csr)
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, csr, i32=i32)
        for r in range(G):
            _assert_exact(got[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)


def test_placement_invariance_and_rank_without_tables():
    outs = []
    for own in ([0, 0, 1, 1, 2, 2], [2, 1, 0, 2, 1, 0], [1, 1, 1, 1, 1, 1], [0, 2, 0, 2, 0, 2]):
        w = synth.make_workload("tiny", G=3, pmin=0, pmax=20, B=64, T=6, dim=16, owner=np.array(own))
        tabs = H.np_tables(w)
        csr = H.np_csrs(w, 44)
        layers = _layers(w, tabs)
        got = _run(w, layers, csr)
        _close(layers)
        outs.append(np.concatenate(got))
    for o in outs[1:]:
        _assert_exact(o, outs[0])


def test_epoch_ring_poisoned_slots_exactly_once():
    """P14: every returned slot is poisoned with NaN after it is read; the 3-slot ring
    rewrites it three epochs later, so from epoch 3 on every forward lands on poison and
    must leave no NaN and match the oracle (exactly-once, C21)."""
    w = synth.make_workload("tiny", G=2, pmin=0, pmax=12, B=90, T=5, dim=32, rows=300)
    tabs = H.np_tables(w)
    layers = _layers(w, tabs)
    try:
        for epoch in range(8):
            csr = H.np_csrs(w, 1000 + epoch)
            ref = H.oracle_outputs(w, 1000 + epoch, tabs, csr)
            offs, idxs = csr
            dev_in = [(torch.from_numpy(offs[r]).to(DEV), torch.from_numpy(idxs[r]).to(DEV)) for r in range(w.G)]
            streams = [torch.cuda.Stream() for _ in range(w.G)]
            torch.cuda.synchronize()
            ys = [layers[r].forward(dev_in[r][0], dev_in[r][1], 0, streams[r]) for r in range(w.G)]
            torch.cuda.synchronize()
            for r in range(w.G):
                _assert_exact(H.dev_out_to_np(ys[r].clone()), ref[r])
                ys[r].fill_(float("nan"))
            torch.cuda.synchronize()
    finally:
        _close(layers)


@pytest.mark.parametrize("i32", [False, True])
def test_bounds_check_flag(i32):
    """EMB_FWD_CHECK_BOUNDS: out-of-range ids (past the end, negative) are skipped and flagged;
    the result equals the oracle's pooling of the remaining ids, compared bit for bit."""
    w = synth.make_workload("tiny", G=1, pmin=1, pmax=6, B=40, T=2, dim=16, rows=100)
    tabs = H.np_tables(w)
    offs, idxs = H.np_csrs(w, 8)
    bad = idxs[0].copy()
    bad[3] = 100          # out of range
    bad[7] = -5
    bad[8] = 2 ** 31 - 1 if i32 else 2 ** 40
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, ([offs[0]], [bad]), E.EMB_FWD_CHECK_BOUNDS, i32=i32)[0]
        assert layers[0].device_error(clear=True) & E.EMB_DEVERR_BOUNDS
        assert layers[0].device_error() == 0
    finally:
        _close(layers)
    # expected: the offending indices contribute nothing
    for t in range(w.T):
        o, lo, hi = O.rank_table_csr(offs[0], t, w.B)
        for b in range(w.B):
            js = [j for j in range(lo + o[b], lo + o[b + 1]) if 0 <= bad[j] < 100]
            exp = O.pool_bag_f32(tabs[t][bad[js]]) if js else np.zeros(w.dim, np.float32)
            assert np.array_equal(got[b, t].view(np.uint32), exp.view(np.uint32)), (t, b)


def test_peer_timeout_sets_error_instead_of_hanging():
    w = synth.make_workload("tiny", G=2, pmin=1, pmax=4, B=16, T=2, dim=16)
    tabs = H.np_tables(w)
    offs, idxs = H.np_csrs(w, 2)
    layers = _layers(w, tabs, options={"timeout_ms": 200})
    try:
        o, x = torch.from_numpy(offs[0]).to(DEV), torch.from_numpy(idxs[0]).to(DEV)
        layers[0].forward(o, x)        # rank 1 never forwards
        torch.cuda.synchronize()
        assert layers[0].device_error(clear=True) & E.EMB_DEVERR_TIMEOUT
        # rank 1 catches up; both complete epoch 1 (rank 0 then re-runs epoch 2 with rank 1's epoch 2)
    finally:
        _close(layers)


# ------------------------------------------------------------------------------- comparison path
def test_baseline_pool_unpack_matches_pgas_bitwise():
    """P12: pool -> (simulated all-to-all with copies) -> unpack == PGAS output."""
    G = 3
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=25, B=77, T=7, dim=32, rows=400)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 31)
    ref = H.oracle_outputs(w, 31, tabs, csr)
    layers = _layers(w, tabs)
    try:
        dev_in = [(torch.from_numpy(csr[0][r]).to(DEV), torch.from_numpy(csr[1][r]).to(DEV)) for r in range(G)]
        sends, splits = [], []
        for r in range(G):
            sc, rc = E.emb_baseline_splits(layers[r].ctx)
            s = torch.full((max(sum(sc), 1),), float("nan"), device=DEV)
            E.emb_baseline_pool(layers[r].ctx, dev_in[r][0], dev_in[r][1], s)
            sends.append(s)
            splits.append((sc, rc))
        torch.cuda.synchronize()
        for r in range(G):  # all_to_all_single semantics, done with copies
            chunks = []
            for src in range(G):
                sc = splits[src][0]
                off = sum(sc[:r])
                chunks.append(sends[src][off: off + sc[r]])
            recv = torch.cat(chunks)
            assert recv.numel() == sum(splits[r][1])
            out = torch.full((layers[r].B_r, w.T, w.dim), float("nan"), device=DEV)
            E.emb_baseline_unpack(layers[r].ctx, recv, out)
            torch.cuda.synchronize()
            _assert_exact(out.cpu().numpy(), ref[r])
    finally:
        _close(layers)


def test_baseline_g1_equals_pgas():
    w = synth.make_workload("tiny", G=1, pmin=0, pmax=50, B=300, T=4, dim=64, rows=1000, dist="zipf")
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 9)
    layers = _layers(w, tabs)
    try:
        o, x = torch.from_numpy(csr[0][0]).to(DEV), torch.from_numpy(csr[1][0]).to(DEV)
        a = layers[0].forward(o, x).clone()
        b = layers[0].forward_baseline(o, x).clone()
        torch.cuda.synchronize()
        assert torch.equal(a.view(torch.int32), b.view(torch.int32))
    finally:
        _close(layers)


def test_forward_host_e2e_matches_device_path():
    w = synth.make_workload("tiny", G=1, pmin=0, pmax=30, B=500, T=3, dim=64, rows=2000)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 77)
    ref = H.oracle_outputs(w, 77, tabs, csr)
    layers = _layers(w, tabs)
    try:
        ho = torch.from_numpy(csr[0][0]).pin_memory()
        hx = torch.from_numpy(csr[1][0]).pin_memory()
        hout = torch.empty((w.B, w.T, w.dim), dtype=torch.float32).pin_memory()
        s = torch.cuda.current_stream()
        E.emb_forward_host(layers[0].ctx, ho, hx, hout, 0, s)
        s.synchronize()
        _assert_exact(hout.numpy(), ref[0])
    finally:
        _close(layers)


def test_api_errors():
    with pytest.raises(E.EmbError):
        E.emb_init(0, 0, 0)
    ctx = E.emb_init(0, 1, 0)
    try:
        with pytest.raises(E.EmbError) as ei:
            E.emb_forward(ctx, 0, 0)
        assert ei.value.status == 2  # EMB_ERR_STATE
        w = torch.zeros((10, 3), device=DEV)
        with pytest.raises(E.EmbError):
            E.emb_register_tables(ctx, [10], [0], 3, "f32", "f32", 4, [w])  # 12-byte rows unsupported
        with pytest.raises(E.EmbError):
            E.emb_register_tables(ctx, [10], [1], 4, "f32", "f32", 4, [w])  # owner out of range
        with pytest.raises(E.EmbError):
            E.emb_set_option(ctx, "nope", 1)
        w4 = torch.zeros((10, 4), device=DEV)
        with pytest.raises(E.EmbError) as ei:     # (T + 1) * B > 2^31 - 1: 32-bit work counter
            E.emb_register_tables(ctx, [10], [0], 4, "f32", "f32", 2 ** 30, [w4])
        assert ei.value.status == 1 and "2^31" in str(ei.value)
    finally:
        E.emb_finalize(ctx)


VARIANT_CASES = [dict(dim=128, pmin=0, pmax=70, B=333, rows=3000, dist="zipf"),       # 512-B rows, 16-B lanes
                 dict(dim=64, pmin=1, pmax=40, B=257, rows=2000),                     # 256-B rows, 8-B lanes
                 dict(dim=128, wdtype="bf16", odtype="bf16", pmin=0, pmax=50, B=129, rows=1000),
                 dict(dim=32, pmin=0, pmax=9, B=100),                                 # 128 B: 8 of 32 lanes
                 dict(dim=6, pmin=0, pmax=12, B=77, rows=300),                        # 24 B: 8-B lanes, 3 active
                 dict(dim=256, pmin=0, pmax=33, B=91, rows=700),                      # 1 KB: 2 vectors per lane
                 dict(dim=512, wdtype="bf16", odtype="f32", pmin=0, pmax=20, B=65, rows=400)]   # 1 KB bf16


@pytest.mark.parametrize("opts", [{}, {"chunk_rows": 1}, {"chunk_rows": 100000}, {"chunk_rows": 7}, {"chunk_rows": 3},
                                  {"stagger": 0}, {"fwd_interleave": 1}, {"tail_div": 1}, {"tail_div": 16},
                                  {"carveout": -1}, {"ctas_per_sm": 1}, {"tma_store": 1},
                                  {"tma_store": 1, "chunk_rows": 3}])
@pytest.mark.parametrize("i32", [False, True])
@pytest.mark.parametrize("case", range(len(VARIANT_CASES)))
def test_pipeline_variants_bitexact(opts, i32, case):
    """Every row tiling x chunking x store variant x index width is bit-exact, with and
    without the bounds-checking (per-id validity) kernel."""
    w = synth.make_workload("tiny", G=2, T=5, **VARIANT_CASES[case])
    if opts.get("tma_store") and w.dim * w.elem_bytes() not in (256, 512):
        pytest.skip("tma_store needs rows of exactly one vector per lane (256 or 512 B)")
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 71)
    ref = H.oracle_outputs(w, 71, tabs, csr)
    layers = _layers(w, tabs, options=opts)
    try:
        got = _run(w, layers, csr, i32=i32)
        got_chk = _run(w, layers, csr, E.EMB_FWD_CHECK_BOUNDS, i32=i32)
        for r in range(w.G):
            _assert_exact(got[r], ref[r])
            _assert_exact(got_chk[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)


def test_forward_host_async_pipeline_matches_oracle():
    """Pipelined host path: 5 calls in flight on alternating stages, each its own h_out."""
    w = synth.make_workload("tiny", G=1, pmin=0, pmax=30, B=300, T=3, dim=64, rows=2000)
    tabs = H.np_tables(w)
    layers = _layers(w, tabs)
    try:
        seeds = [900 + i for i in range(5)]
        csrs = [H.np_csrs(w, sd) for sd in seeds]
        hin = [(torch.from_numpy(c[0][0]).pin_memory(), torch.from_numpy(c[1][0]).pin_memory()) for c in csrs]
        houts = [torch.full((w.B, w.T, w.dim), float("nan")).pin_memory() for _ in seeds]
        s = torch.cuda.current_stream()
        for i in range(len(seeds)):
            E.emb_forward_host_async(layers[0].ctx, hin[i][0], hin[i][1], houts[i], 0, s)
        E.emb_host_drain(layers[0].ctx, s)
        s.synchronize()
        for i, sd in enumerate(seeds):
            _assert_exact(houts[i].numpy(), H.oracle_outputs(w, sd, tabs, csrs[i])[0])
    finally:
        _close(layers)


def test_trace_counts_every_stored_byte():
    """f1: per-chunk trace records add up to exactly the bytes each rank stores, split into
    local and remote by destination, with monotone globaltimer stamps inside the forward."""
    G = 2
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=20, B=200, T=6, dim=32, rows=500)
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 5)
    layers = _layers(w, tabs, options={"trace_capacity": 100000})
    try:
        got = _run(w, layers, csr)
        ref = H.oracle_outputs(w, 5, tabs, csr)
        for r in range(G):
            _assert_exact(got[r], ref[r])
            tr = E.emb_trace_read(layers[r].ctx, 100000)
            assert tr.shape[0] > 0
            remote = int((tr[:, 1] >> np.uint64(32)).sum())
            local = int((tr[:, 1] & np.uint64(0xFFFFFFFF)).sum())
            Tr = len(w.local_tables(r))
            starts, counts = O.split_batch(w.B, G)
            vec = w.dim * 4
            assert local == Tr * counts[r] * vec
            assert remote == Tr * (w.B - counts[r]) * vec
            assert np.all(tr[:, 0] > 0)
        # reading resets the trace
        assert E.emb_trace_read(layers[0].ctx, 10).shape[0] == 0
    finally:
        _close(layers)


def _c7_tables(w, seed):
    """Tables of IEEE special values (SURVEY reading C7: IEEE RN, no FTZ, NaN propagates):
    table 0 holds only small multiples of the least subnormal (its bag sums stay subnormal,
    an FTZ add would return 0) and -0.0; table 1 normal values sprinkled with +-Inf, NaN and
    near-max finites (sums overflow to Inf, Inf - Inf = NaN); table 2 large-magnitude
    cancellation (+-2^100 against O(1) values) and -0.0 rows.  All values are exact in the
    weight dtype (bf16 tables: multiples of 2^-133, quiet NaN 0x7FC00000)."""
    rng = np.random.default_rng(seed)
    M, d = int(w.rows[0]), w.dim
    bf = w.wdtype == "bf16"
    lsb = 2.0 ** (-133 if bf else -149)
    out = {}
    t0 = (rng.integers(-40, 41, size=(M, d)) * lsb).astype(np.float32)
    t0[rng.random((M, d)) < 0.1] = -0.0
    out[0] = t0
    t1 = (rng.integers(-128, 128, size=(M, d)) / 64.0).astype(np.float32)
    u = rng.random((M, d))
    big = np.float32(2.0 ** 127 * 1.5)                       # exact in bf16, two of them overflow
    t1[u < 0.02] = np.inf
    t1[(u >= 0.02) & (u < 0.04)] = -np.inf
    t1[(u >= 0.04) & (u < 0.06)] = np.uint32(0x7FC00000).view(np.float32)
    t1[(u >= 0.06) & (u < 0.08)] = big
    t1[(u >= 0.08) & (u < 0.10)] = -big
    out[1] = t1
    t2 = (rng.integers(-8, 9, size=(M, d)) / 4.0).astype(np.float32)
    v = rng.random((M, d))
    t2[v < 0.15] = np.float32(2.0 ** 100)
    t2[(v >= 0.15) & (v < 0.30)] = np.float32(-(2.0 ** 100))
    t2[rng.random(M) < 0.1] = -0.0
    out[2] = t2
    return out


def _assert_ieee_equal(got, ref):
    """bit-exact, except that a NaN matches any NaN (its payload is not specified, C7)"""
    gf = got.astype(np.float32) if got.dtype == np.float32 else O.bf16_to_f32(got)
    rf = ref.astype(np.float32) if ref.dtype == np.float32 else O.bf16_to_f32(ref)
    gn, rn = np.isnan(gf), np.isnan(rf)
    assert np.array_equal(gn, rn), f"NaN positions differ: {np.argwhere(gn != rn)[:3].tolist()}"
    gb, rb = H.bits(got), H.bits(ref)
    bad = (gb != rb) & ~gn
    assert not bad.any(), f"{int(bad.sum())} mismatches, first at {np.argwhere(bad)[0].tolist()}: " \
                          f"got {gf[tuple(np.argwhere(bad)[0])]!r} want {rf[tuple(np.argwhere(bad)[0])]!r}"


@pytest.mark.parametrize("dim,wdt,odt", [(128, "f32", "f32"), (64, "f32", "f32"), (256, "bf16", "bf16"),
                                         (128, "bf16", "f32"), (64, "f32", "bf16")])
@pytest.mark.parametrize("G", [1, 2])
def test_c7_ieee_special_values_bitexact(dim, wdt, odt, G):
    """C7 on the GPU: subnormal sums are not flushed, +-Inf / NaN propagate, overflow gives
    Inf, -0.0 one-hot bags keep their sign, large-magnitude cancellation follows the
    canonical order -- bit-exact against the oracle (NaN matched as NaN), through the
    direct kernel, the per-id validity kernel (CHECK_BOUNDS) and, at G = 2, remote stores."""
    w = synth.make_workload("tiny", G=G, T=3, rows=64, dim=dim, B=203, pmin=0, pmax=12, wdtype=wdt, odtype=odt)
    tabs = _c7_tables(w, 17)
    csr = H.np_csrs(w, 19)
    with np.errstate(all="ignore"):
        ref = H.oracle_outputs(w, 19, tabs, csr)
    r0 = ref[0].astype(np.float32) if ref[0].dtype == np.float32 else O.bf16_to_f32(ref[0])
    assert np.isnan(r0).any() and np.isinf(r0).any()                      # the specials do reach the output
    if G == 1 and (odt == "f32" or wdt == "bf16"):
        sub = r0[:, 0]
        assert ((sub != 0) & (np.abs(sub) < 2.0 ** -126)).any()            # subnormal results present
    layers = _layers(w, tabs)
    try:
        got = _run(w, layers, csr)
        got_chk = _run(w, layers, csr, E.EMB_FWD_CHECK_BOUNDS)
        for r in range(w.G):
            _assert_ieee_equal(got[r], ref[r])
            _assert_ieee_equal(got_chk[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)


@pytest.mark.parametrize("G,T", [(2, 9), (3, 13), (1, 3)])
@pytest.mark.parametrize("opts", [{}, {"chunk_rows": 7}, {"tail_div": 16, "chunk_rows": 40}, {"stagger": 0},
                                  {"fwd_interleave": 1}])
def test_chunk_grid_guided_tail_and_rotation_bitexact(G, T, opts):
    """the claim -> (table, first bag) decode: ranks with >= 4 local tables take the guided tail
    (the last table in smaller chunks), ranks with fewer do not; destination-staggered rotation
    of the chunk order at G > 1, with chunks crossing mini-batch boundaries; bit-exact"""
    w = synth.make_workload("tiny", G=G, T=T, dim=64, pmin=0, pmax=30, B=301, rows=500)
    assert G == 1 or min(len(w.local_tables(r)) for r in range(G)) >= 4
    tabs = H.np_tables(w)
    csr = H.np_csrs(w, 73)
    ref = H.oracle_outputs(w, 73, tabs, csr)
    layers = _layers(w, tabs, options=opts)
    try:
        got = _run(w, layers, csr)
        for r in range(w.G):
            _assert_exact(got[r], ref[r])
            assert layers[r].device_error() == 0
    finally:
        _close(layers)
