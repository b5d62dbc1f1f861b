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
