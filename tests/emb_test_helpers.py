"""Shared test plumbing: build inputs with the seeded generators (numpy side for the
oracle, numpy->H2D or libsynth for the CUDA side) and run both implementations."""
from __future__ import annotations

import numpy as np

import synth
from oracle import emb_oracle as O


def np_tables(w):
    """{physical id: float32 [M, d]} (bf16 tables: values are bf16-exact)."""
    out = {}
    for t in range(w.T):
        p = int(w.phys[t])
        if p not in out:
            out[p] = synth.table_rows(w.table_seed, p, int(w.rows[t]), w.dim, w.mode, w.wdtype)
    return out


def np_csrs(w, seed):
    offs, idxs = [], []
    for r in range(w.G):
        o, x = synth.rank_csr(w, seed, r)
        offs.append(o)
        idxs.append(x)
    return offs, idxs


def oracle_outputs(w, seed, tabs=None, csrs=None):
    """Oracle Y_r for every rank: float32 arrays, or uint16 bf16 bits."""
    tabs = tabs if tabs is not None else np_tables(w)
    offs, idxs = csrs if csrs is not None else np_csrs(w, seed)
    per_t = [tabs[int(w.phys[t])] for t in range(w.T)]
    if w.wdtype == "bf16":
        per_t = [synth.to_bf16_bits(x) for x in per_t]
    return O.emb_forward(per_t, w.owner, offs, idxs, w.B, w.G, out_dtype=w.odtype, table_is_bf16=(w.wdtype == "bf16"))


def bits(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a)
    return a.view(np.uint32) if a.dtype == np.float32 else a.view(np.uint16)


def dev_out_to_np(y):
    """torch device tensor -> numpy float32 or uint16 bf16 bits."""
    import torch
    y = y.detach().cpu()
    if y.dtype == torch.bfloat16:
        return y.view(torch.int16).numpy().view(np.uint16)
    return y.numpy()


def sample_bag_expected(w, batch_seed, t, b, tab_seed=None):
    """Oracle value of bag (t, b), regenerated from the counter generators only."""
    L = synth.pooling_lengths(batch_seed, t, w.B, w.pmin, w.pmax)
    start = int(L[:b].sum())
    pos = np.arange(start, start + int(L[b]), dtype=np.int64)
    x = synth.table_indices(batch_seed, t, pos, int(w.rows[t]), w.dist, w.alpha, perm_seed=w.table_seed)
    rows = synth.table_values(w.table_seed, int(w.phys[t]), x, w.dim, w.mode, w.wdtype)
    acc = O.pool_bag_f32(rows)
    z64, S = O.pool_bag_f64(rows)
    return acc, z64, S
