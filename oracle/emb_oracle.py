"""CPU oracle for the EMB-layer forward: EmbeddingBag(sum) + model->data-parallel layout.

*** TEST INFRASTRUCTURE ONLY. ***  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import or run this
module.  The product path (``paper_conf_sc_chenbyo24_b200``) never imports it and
shares no code with it; it imports nothing from the product path.

What it computes is the paper's plain definition, written out (numpy, slow, obvious):

  * Lookup + sum pooling (§II-B, Fig. 3 L83-89): for each sparse
    feature (table) t and sample b, read the rows W_t[x] named by the bag's indices
    and combine them "via element-wise summation".  A sample with no input for a
    feature ("NULL", L85/L89) yields the zero vector (SURVEY reading C2).
  * Hybrid parallelism / layout conversion (L99-113, §II-C, Fig. 4): tables are
    partitioned across GPUs (model parallel); each GPU pools its tables for the FULL
    batch; the batch is split into contiguous mini-batches (Fig. 4: "mini-batch size
    of N/2"), and after the exchange GPU r holds, for its mini-batch, the pooled
    embeddings of ALL features:  Y_r[i, t, :] = Z_t[s_r + i, :].

Readings of points the paper leaves open (listed in DESIGN.md "Readings"):
  C2  empty bag -> +0.0;     C3 sum only;      C4 canonical order = CSR order, the
  accumulator starts at the FIRST row, then float32 round-to-nearest adds;
  C5  float32 accumulation (also for bf16 tables, widened exactly);
  C6  bf16 output = RNE of the float32 accumulator, once;
  C7  IEEE arithmetic without flush-to-zero (numpy float32 adds keep subnormals); Inf and
      NaN propagate; NaN -> NaN in the bf16 rounding;
  C8  contiguous batch split, first B mod G ranks one extra sample;
  C9  output [B_r][T][d] row-major, tables in global id order;
  C11 per-rank CSR is table-major: bag (t_l, b) = offsets[t_l*B+b] .. offsets[t_l*B+b+1];
  C13 duplicate indices all count.

Pins (tests/test_oracle.py): brute-force Python loops (P1), one-hot/empty/duplicate
closed forms (P2-P4), the S-normalised metric and S = sum |w| against hand-derived values
(tests/golden/s_normalized_error.json), IEEE special values (subnormal sums, +-Inf, NaN;
C7) against closed forms and torch's bf16 conversion, integer tables exact in any order (P5), identity routing (P6),
power-of-two scaling (P7), linearity (P8), placement invariance (P9), rank concat
(P10), torch.nn.functional.embedding_bag + gloo all_to_all special cases (P11),
conservation (P13), the paper's Fig. 3 / Fig. 4 structure (P15), and torch's bf16
conversion for the rounding step.  Backward (§V):
`emb_backward` is the transpose of the pooling + layout conversion, pinned by a
pure-Python loop, the adjoint identity <pool(W), dY> = <W, dW> (exact on integer data),
torch autograd of embedding_bag(mode="sum"), and placement invariance.
"""
from __future__ import annotations

from typing import Callable, Dict, List, Optional, Sequence, Tuple

import numpy as np

__all__ = [
    "validate_csr", "pool_table_f32", "pool_table_f64", "rne_bf16", "bf16_to_f32",
    "split_batch", "rank_table_csr", "mp_to_dp", "emb_forward", "pool_bag_f32",
    "pool_bag_f64", "s_normalized_error", "emb_backward", "emb_forward_sharded",
]


# ----------------------------------------------------------------------------- validation
def validate_csr(offsets: np.ndarray, indices: np.ndarray, num_rows: int) -> None:
    """C1/C12: offsets start at 0, are non-decreasing, end at nnz; 0 <= x < M."""
    offsets = np.asarray(offsets)
    indices = np.asarray(indices)
    if offsets.ndim != 1 or offsets.size < 1:
        raise ValueError("offsets must be 1-D with at least one element")
    if offsets[0] != 0:
        raise ValueError("offsets[0] must be 0")
    if np.any(np.diff(offsets) < 0):
        raise ValueError("offsets must be non-decreasing")
    if offsets[-1] != indices.size:
        raise ValueError("offsets[-1] must equal len(indices)")
    if indices.size and (indices.min() < 0 or indices.max() >= num_rows):
        raise ValueError("index out of range [0, M)")


# ----------------------------------------------------------------------------- pooling
def pool_table_f32(W: np.ndarray, offsets: np.ndarray, indices: np.ndarray) -> np.ndarray:
    """Z[b] = W[x_o[b]] + W[x_o[b]+1] + ... in CSR order, float32 RN (L91-95; C4).

    Position-major form of the per-bag sequential loop: acc starts at the first row
    of every non-empty bag, then for p = 1, 2, ...  acc[bags longer than p] += row p.
    Each element sees exactly the additions of the sequential loop, in the same
    order, so the result is bit-identical to it (pinned by P1)."""
    W = np.asarray(W)
    assert W.dtype == np.float32 and W.ndim == 2
    offsets = np.asarray(offsets, dtype=np.int64)
    indices = np.asarray(indices, dtype=np.int64)
    validate_csr(offsets, indices, W.shape[0])
    B = offsets.size - 1
    L = np.diff(offsets)
    start = offsets[:-1]
    Z = np.zeros((B, W.shape[1]), dtype=np.float32)          # empty bag -> +0.0 (C2)
    has = L > 0
    Z[has] = W[indices[start[has]]]                          # acc = first row (C4)
    for p in range(1, int(L.max()) if B else 0):
        m = L > p
        Z[m] = Z[m] + W[indices[start[m] + p]]               # float32 + float32, RN
    return Z


def pool_table_f64(W: np.ndarray, offsets: np.ndarray, indices: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
    """Exact-as-fp64 sum and S = sum |w| per element (tolerance denominator)."""
    W64 = np.asarray(W, dtype=np.float64)
    offsets = np.asarray(offsets, dtype=np.int64)
    indices = np.asarray(indices, dtype=np.int64)
    validate_csr(offsets, indices, W64.shape[0])
    B = offsets.size - 1
    L = np.diff(offsets)
    start = offsets[:-1]
    Z = np.zeros((B, W64.shape[1]), dtype=np.float64)
    S = np.zeros_like(Z)
    for p in range(int(L.max()) if B else 0):
        m = L > p
        rows = W64[indices[start[m] + p]]
        Z[m] += rows
        S[m] += np.abs(rows)
    return Z, S


def pool_bag_f32(rows: np.ndarray) -> np.ndarray:
    """One bag, sequential: acc = rows[0]; acc += rows[j] (float32).  Empty -> +0."""
    rows = np.asarray(rows, dtype=np.float32)
    if rows.shape[0] == 0:
        return np.zeros(rows.shape[1], dtype=np.float32)
    acc = rows[0].copy()
    for j in range(1, rows.shape[0]):
        acc = acc + rows[j]
    return acc


def pool_bag_f64(rows: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
    r = np.asarray(rows, dtype=np.float64)
    return r.sum(axis=0) if r.shape[0] else np.zeros(r.shape[1]), np.abs(r).sum(axis=0) if r.shape[0] else np.zeros(r.shape[1])


# ----------------------------------------------------------------------------- bf16
def rne_bf16(x: np.ndarray) -> np.ndarray:
    """float32 -> bf16 bits, round to nearest even (C6): u += 0x7FFF + ((u>>16)&1); u >>= 16.
    Finite values overflow to +-Inf and subnormals round like any other value (the rule is
    monotone in the bit pattern); +-Inf map to +-Inf.  NaN stays NaN (C7): the rounding rule
    would carry a NaN whose payload sits in the low 16 bits into Inf, so NaN is mapped to
    the quiet NaN 0x7FC0 instead (any NaN pattern is accepted on the GPU side)."""
    f = np.ascontiguousarray(x, dtype=np.float32)
    u = f.view(np.uint32).astype(np.uint64)
    u = u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))
    out = (u >> np.uint64(16)).astype(np.uint16)
    out[np.isnan(f)] = np.uint16(0x7FC0)
    return out


def bf16_to_f32(bits: np.ndarray) -> np.ndarray:
    """Exact widening bf16 -> float32 (C5)."""
    return (np.asarray(bits, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


# ----------------------------------------------------------------------------- layout
def split_batch(B: int, G: int) -> Tuple[List[int], List[int]]:
    """Contiguous mini-batches (Fig. 4 / L111 'N/2'); first B mod G ranks +1 (C8)."""
    q, rem = divmod(B, G)
    counts = [q + 1 if r < rem else q for r in range(G)]
    starts = [sum(counts[:r]) for r in range(G)]
    return starts, counts


def rank_table_csr(offsets: np.ndarray, t_local: int, B: int) -> Tuple[np.ndarray, int, int]:
    """Bag (t_l, b) spans offsets[t_l*B+b] .. offsets[t_l*B+b+1] (C11).  Returns the
    table's offsets rebased to 0 plus the [lo, hi) range of its index run."""
    o = np.asarray(offsets[t_local * B: t_local * B + B + 1], dtype=np.int64)
    return o - o[0], int(o[0]), int(o[-1])


def mp_to_dp(Z_by_table: Sequence[np.ndarray], G: int) -> List[np.ndarray]:
    """Y_r[i, t, :] = Z_t[s_r + i, :]  (L111-113, Fig. 4; C8, C9)."""
    T = len(Z_by_table)
    B, d = Z_by_table[0].shape
    starts, counts = split_batch(B, G)
    out = []
    for r in range(G):
        Y = np.empty((counts[r], T, d), dtype=Z_by_table[0].dtype)
        for t in range(T):
            Y[:, t, :] = Z_by_table[t][starts[r]: starts[r] + counts[r]]
        out.append(Y)
    return out


def emb_forward(tables: Sequence[np.ndarray], owner: Sequence[int], rank_offsets: Sequence[np.ndarray],
                rank_indices: Sequence[np.ndarray], B: int, G: int, out_dtype: str = "f32",
                table_is_bf16: bool = False) -> List[np.ndarray]:
    """Whole distributed EMB forward, simulated for G ranks (L99-113).

    tables[t]        : W_t as float32 [M_t, d]  (bf16 tables: pass bf16 bits as uint16 and
                       table_is_bf16=True; they are widened exactly, C5)
    owner[t]         : rank holding table t (model parallel)
    rank_offsets[r]  : rank r's table-major CSR offsets [T_r*B + 1] (C11)
    rank_indices[r]  : rank r's local row ids
    returns Y_r for r in 0..G-1: float32 [B_r, T, d], or bf16 bits uint16 if out_dtype == "bf16".
    """
    T = len(tables)
    owner = [int(o) for o in owner]
    Z: List[Optional[np.ndarray]] = [None] * T
    for r in range(G):                                    # each rank: its tables, full batch
        local = [t for t in range(T) if owner[t] == r]    # ascending global id
        for tl, t in enumerate(local):
            o, lo, hi = rank_table_csr(rank_offsets[r], tl, B)
            W = bf16_to_f32(tables[t]) if table_is_bf16 else np.asarray(tables[t], dtype=np.float32)
            Z[t] = pool_table_f32(W, o, np.asarray(rank_indices[r][lo:hi]))
    Ys = mp_to_dp(Z, G)                                   # the exchange (all-to-all)
    if out_dtype == "bf16":
        return [rne_bf16(Y) for Y in Ys]
    return Ys


def s_normalized_error(y: np.ndarray, y_ref: np.ndarray, S: np.ndarray) -> float:
    """max |y - y_ref| / S with 0/0 := 0 (SURVEY §8(c) acceptance metric)."""
    diff = np.abs(np.asarray(y, dtype=np.float64) - np.asarray(y_ref, dtype=np.float64))
    S = np.asarray(S, dtype=np.float64)
    with np.errstate(divide="ignore", invalid="ignore"):
        q = np.where(diff == 0, 0.0, diff / S)
    return float(np.max(q)) if q.size else 0.0


# ----------------------------------------------------------------------------- backward (f2)
def emb_backward(rows: Sequence[int], dim: int, owner: Sequence[int], rank_offsets: Sequence[np.ndarray],
                 rank_indices: Sequence[np.ndarray], dY: Sequence[np.ndarray], B: int, G: int):
    """Adjoint of the forward (§V L378-382 for the exchange; the arithmetic is the
    transpose of sum pooling, L91-95):

        dW_t[x, :] = sum_{b} sum_{j in bag(t, b), x_t[j] = x} dY[b, t, :]

    dY[r] is rank r's gradient w.r.t. its outputs, [B_r][T][d] (data parallel, C8 split);
    the bags come from the owner's CSR (C11).  Returns (dW64, S, count): per global table
    the fp64 gradient [M_t][d], S = sum |dY| per element (tolerance denominator) and the
    number of contributions per row (for the order-independent error bound n*2^-24*S)."""
    T = len(rows)
    owner = [int(o) for o in owner]
    dY_full = np.concatenate([np.asarray(y, dtype=np.float64) for y in dY], axis=0)   # [B][T][d]
    assert dY_full.shape == (B, T, dim)
    dW, S, cnt = [], [], []
    for t in range(T):
        dW.append(np.zeros((int(rows[t]), dim)))
        S.append(np.zeros((int(rows[t]), dim)))
        cnt.append(np.zeros(int(rows[t]), dtype=np.int64))
    for r in range(G):
        local = [t for t in range(T) if owner[t] == r]
        for tl, t in enumerate(local):
            o, lo, hi = rank_table_csr(rank_offsets[r], tl, B)
            x = np.asarray(rank_indices[r][lo:hi], dtype=np.int64)
            validate_csr(o, x, int(rows[t]))
            bag_of = np.repeat(np.arange(B), np.diff(o))          # sample of every position
            g = dY_full[bag_of, t, :]
            np.add.at(dW[t], x, g)
            np.add.at(S[t], x, np.abs(g))
            np.add.at(cnt[t], x, 1)
    return dW, S, cnt


# ----------------------------------------------------------------------------- row-wise sharding (f3)
def emb_forward_sharded(tables: Sequence[np.ndarray], shards: Sequence[Tuple[int, int, int, int, int]],
                        rank_offsets: Sequence[np.ndarray], rank_indices: Sequence[np.ndarray], B: int, G: int,
                        out_dtype: str = "f32") -> List[np.ndarray]:
    """Row-wise sharded forward (§V: "partitioning by rows ... merge the sparse
    input partitioning into the computation kernel").

    shards: (t, s, lo, hi, owner) -- shard s of table t holds rows [lo, hi) on rank `owner`;
    a table with one shard (lo = 0, hi = M_t) is table-wise.  Each rank's CSR lists its
    local shards in ascending (t, s) order, each with the FULL bag list of table t and
    GLOBAL row ids (the partitioning happens in the kernel).  Definition:
      partial_{t,s}[b] = sum, in CSR order from the first kept row, of W_t[x] over the
                         bag's ids with lo <= x < hi (+0.0 if none)            (C4, C2)
      Z_t[b]           = partial_{t,0}[b] + partial_{t,1}[b] + ... in shard order (float32)
    then the usual layout conversion Y_r[i, t] = Z_t[s_r + i] (C8, C9)."""
    T = len(tables)
    by_t: Dict[int, list] = {}
    for (t, s, lo, hi, o) in shards:
        by_t.setdefault(int(t), []).append((int(s), int(lo), int(hi), int(o)))
    partial: Dict[Tuple[int, int], np.ndarray] = {}
    for r in range(G):
        local = sorted((int(t), int(s), int(lo), int(hi)) for (t, s, lo, hi, o) in shards if int(o) == r)
        for k, (t, s, lo, hi) in enumerate(local):
            o, a, b = rank_table_csr(rank_offsets[r], k, B)
            x = np.asarray(rank_indices[r][a:b], dtype=np.int64)
            validate_csr(o, x, int(np.asarray(tables[t]).shape[0]))
            keep = (x >= lo) & (x < hi)
            # re-pack the bag list with only the kept ids, preserving CSR order
            ck = np.concatenate([[0], np.cumsum(keep.astype(np.int64))])
            kept_per_bag = ck[o[1:]] - ck[o[:-1]]
            o2 = np.zeros(B + 1, dtype=np.int64)
            np.cumsum(kept_per_bag, out=o2[1:])
            W = np.asarray(tables[t], dtype=np.float32)
            partial[(t, s)] = pool_table_f32(W, o2, x[keep])
    Z = []
    for t in range(T):
        parts = sorted(by_t[t])
        acc = partial[(t, parts[0][0])].copy()
        for (s, _, _, _) in parts[1:]:
            acc = acc + partial[(t, s)]
        Z.append(acc)
    Ys = mp_to_dp(Z, G)
    return [rne_bf16(Y) for Y in Ys] if out_dtype == "bf16" else Ys
