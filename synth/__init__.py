"""Seeded synthetic inputs for the EMB-layer forward (tables, pooling factors, CSR).

This module is the ONE thing the oracle side (``oracle/``, via ``tests/``) and the
CUDA side (``paper_conf_sc_chenbyo24_b200``) both consume.  It holds none of the
method's arithmetic (no lookup, no pooling, no layout conversion): it only draws
the inputs the paper's experiments describe, with a counter-based generator so
that any element can be regenerated independently (numpy here, CUDA in
``synth/csrc/synth_gen.cu``; the two are cross-checked bit-exactly by
``tests/test_synth_gpu.py``).

Paper workload (``/root/reference/PAPER.md``):
  * L197 (§IV): "dense and sparse feature inputs are generated synthetically with a
    uniform random distribution" -> ``dist="uniform"`` control.
  * BASELINE.json north_star: "synthetic Criteo-shaped data (power-law indices,
    pooling factors as in the paper)" -> ``dist="zipf"``, s = 1.05.
  * L260 "pooling factor generated from a uniform distribution with a maximum size
    of 128", L329 "pooling factor of up to 32" -> U{1..Pmax}.
  * L79 (§II-A) indices are hashed into [0, M_t) before lookup; hashing is out of
    scope, so the generator emits in-range row ids directly.

Counter hash: ``h(stream, seed, a, b)`` = three splitmix64 finaliser
rounds.  Every stream is a pure function of its counters, so the data of table t
does not depend on which rank owns it (needed for the placement-invariance pin).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from functools import lru_cache
from typing import Optional, Sequence

import numpy as np

__all__ = [
    "S_TABLE", "S_POOL", "S_INDEX", "S_PERM", "hash3", "table_values", "table_rows",
    "to_bf16_bits", "bf16_bits_to_f32", "zipf_cdf", "perm_params", "pooling_lengths",
    "table_indices", "Workload", "make_workload", "batch_split", "rank_csr",
    "table_csr", "lpt_placement", "contiguous_placement",
]

_M64 = (1 << 64) - 1
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)

# stream identifiers (domain separation)
S_TABLE = 0x7AB1E
S_POOL = 0x9001
S_INDEX = 0x1D3
S_PERM = 0xBE11


def _u64(x) -> np.ndarray:
    a = np.asarray(x)
    if a.dtype != np.uint64:
        a = a.astype(np.int64).astype(np.uint64)
    return a


def _mix64(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser (wrapping uint64 arithmetic)."""
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def hash3(stream: int, seed: int, a, b) -> np.ndarray:
    """h = mix(mix(mix(seed*GOLDEN + stream) ^ a) + b), all uint64, wrapping."""
    with np.errstate(over="ignore"):
        s0 = np.array([(int(seed) * 0x9E3779B97F4A7C15 + int(stream)) & _M64], dtype=np.uint64)
        x = _mix64(s0)
        x = _mix64(x ^ _u64(a))
        return _mix64(x + _u64(b))


# ----------------------------------------------------------------------------- tables
def table_values(seed: int, t: int, rows: np.ndarray, dim: int, mode: str = "float",
                 wdtype: str = "f32") -> np.ndarray:
    """Values W_t[rows, 0:dim] as float32 (exactly representable in ``wdtype``).

    mode "float": f32 -> (h>>40 - 2^23) * 2^-23 in [-1,1) (24-bit exact);
                  bf16 -> (h>>56 - 128) * 2^-7 in [-1,1) (8-bit exact).
    mode "int":   (h mod 17) - 8, integers in [-8, 8]  (SURVEY pin P5).
    mode "identity": 8-bit fields [t&255, t>>8, i&255, (i>>8)&255, (i>>16)&255,
                  (i>>24)&255, k&255 ...]  (pin P6; exact in f32 and bf16).
    Element (i, k) uses counter i*dim + k of stream S_TABLE for table t.
    """
    rows = np.asarray(rows, dtype=np.int64).reshape(-1)
    if mode == "identity":
        out = np.empty((rows.size, dim), dtype=np.float32)
        k = np.arange(dim, dtype=np.int64)
        out[:] = (k & 255)[None, :]
        fields = [np.full(rows.size, t & 255), np.full(rows.size, (t >> 8) & 255),
                  rows & 255, (rows >> 8) & 255, (rows >> 16) & 255, (rows >> 24) & 255]
        for j, f in enumerate(fields[:dim]):
            out[:, j] = f
        return out
    ctr = (rows[:, None] * dim + np.arange(dim, dtype=np.int64)[None, :]).reshape(-1)
    h = hash3(S_TABLE, seed, t, ctr)
    if mode == "float":
        if wdtype == "f32":
            v = ((h >> np.uint64(40)).astype(np.int64) - (1 << 23)).astype(np.float64) * 2.0 ** -23
        elif wdtype == "bf16":
            v = ((h >> np.uint64(56)).astype(np.int64) - 128).astype(np.float64) * 2.0 ** -7
        else:
            raise ValueError(wdtype)
    elif mode == "int":
        v = ((h % np.uint64(17)).astype(np.int64) - 8).astype(np.float64)
    else:
        raise ValueError(mode)
    return v.astype(np.float32).reshape(rows.size, dim)


def table_rows(seed: int, t: int, num_rows: int, dim: int, mode: str = "float",
               wdtype: str = "f32") -> np.ndarray:
    """Whole table t as float32 [num_rows, dim]."""
    return table_values(seed, t, np.arange(num_rows, dtype=np.int64), dim, mode, wdtype)


def to_bf16_bits(x_f32: np.ndarray) -> np.ndarray:
    """Exact conversion of float32 values that ARE bf16-representable (generator only;
    truncation == rounding for them).  Not a rounding routine."""
    u = np.ascontiguousarray(x_f32, dtype=np.float32).view(np.uint32)
    if np.any(u & np.uint32(0xFFFF)):
        raise ValueError("value not representable in bf16")
    return (u >> np.uint32(16)).astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)


# ----------------------------------------------------------------------------- indices
@lru_cache(maxsize=8)
def zipf_cdf(num_rows: int, s: float) -> np.ndarray:
    """float64 CDF of the truncated zipf(s) over ranks 1..M (C15).  The CUDA
    generator receives THIS array, so both sides invert the identical table."""
    k = np.arange(1, num_rows + 1, dtype=np.float64)
    c = np.cumsum(k ** (-float(s)))
    c /= c[-1]
    c.setflags(write=False)
    return c


def perm_params(seed: int, t: int, num_rows: int) -> tuple[int, int]:
    """Per-table bijection rank->row: row = (a*(k) + c) mod M with gcd(a, M) = 1."""
    h = hash3(S_PERM, seed, t, np.array([0, 1], dtype=np.int64))
    if num_rows == 1:
        return 1, 0
    a = 1 + int(h[0] % np.uint64(num_rows - 1))
    while math.gcd(a, num_rows) != 1:
        a += 1
        if a >= num_rows:
            a = 1
    c = int(h[1] % np.uint64(num_rows))
    return a, c


def pooling_lengths(seed: int, t: int, batch: int, pmin: int, pmax: int) -> np.ndarray:
    """Bag sizes L(t, b) ~ U{pmin..pmax} (counter stream S_POOL, counter b)."""
    if pmin == pmax:
        return np.full(batch, pmin, dtype=np.int64)
    h = hash3(S_POOL, seed, t, np.arange(batch, dtype=np.int64))
    return pmin + (h % np.uint64(pmax - pmin + 1)).astype(np.int64)


def table_indices(seed: int, t: int, positions: np.ndarray, num_rows: int, dist: str,
                  alpha: float = 1.05, perm_seed: Optional[int] = None) -> np.ndarray:
    """Row ids x_t[j] for the given positions j of table t's index run.

    uniform: x = h mod M.   zipf: u = (h >> 11) * 2^-53, k0 = #{cdf <= u} (0-based
    rank, clamped to M-1), x = (a_t*k0 + c_t) mod M  with (a_t, c_t) = perm_params.
    """
    positions = np.asarray(positions, dtype=np.int64)
    h = hash3(S_INDEX, seed, t, positions)
    if dist == "uniform":
        return (h % np.uint64(num_rows)).astype(np.int64)
    if dist != "zipf":
        raise ValueError(dist)
    u = (h >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    cdf = zipf_cdf(num_rows, alpha)
    k0 = np.searchsorted(cdf, u, side="right").astype(np.int64)
    np.minimum(k0, num_rows - 1, out=k0)
    a, c = perm_params(seed if perm_seed is None else perm_seed, t, num_rows)
    return (a * k0 + c) % num_rows


# ----------------------------------------------------------------------------- workloads
@dataclass
class Workload:
    """One concrete instance of a BASELINE.json config at world size G."""
    name: str
    G: int
    T: int                       # logical tables (global)
    rows: np.ndarray             # [T] rows of each logical table
    dim: int
    B: int                       # global batch
    pmin: int
    pmax: int
    dist: str                    # "zipf" | "uniform"
    alpha: float
    wdtype: str                  # "f32" | "bf16"
    odtype: str                  # "f32" | "bf16"
    owner: np.ndarray            # [T] owning rank of each logical table
    phys: np.ndarray             # [T] physical table backing each logical table (C27)
    table_seed: int = 20241119
    mode: str = "float"
    extra: dict = field(default_factory=dict)

    def local_tables(self, r: int) -> np.ndarray:
        return np.nonzero(self.owner == r)[0].astype(np.int64)

    def phys_rows(self) -> dict:
        d = {}
        for t in range(self.T):
            d[int(self.phys[t])] = int(self.rows[t])
        return d

    def batch_seed(self, batch_id: int) -> int:
        cid = {"tiny": 0, "single": 1, "weak": 2, "weak_paper": 2, "strong": 3, "large": 4,
               "large_shard": 4}.get(self.name, 9)
        return 20241119 + 1000 * cid + int(batch_id)

    def elem_bytes(self) -> int:
        return 4 if self.wdtype == "f32" else 2

    def out_elem_bytes(self) -> int:
        return 4 if self.odtype == "f32" else 2


def batch_split(B: int, G: int) -> tuple[np.ndarray, np.ndarray]:
    """Contiguous DP split (Fig. 4): first B mod G ranks get one extra."""
    q, rem = divmod(B, G)
    counts = np.array([q + (1 if r < rem else 0) for r in range(G)], dtype=np.int64)
    starts = np.concatenate([[0], np.cumsum(counts)[:-1]]).astype(np.int64)
    return starts, counts


def contiguous_placement(T: int, G: int) -> np.ndarray:
    """Rank r owns the contiguous block [r*T/G, (r+1)*T/G) (SURVEY C10 default)."""
    s, _ = batch_split(T, G)
    owner = np.zeros(T, dtype=np.int32)
    for r in range(G):
        owner[s[r]:] = r
    return owner


def lpt_placement(rows: Sequence[int], G: int) -> np.ndarray:
    """Longest-processing-time by rows (large config)."""
    rows = np.asarray(rows, dtype=np.int64)
    order = sorted(range(len(rows)), key=lambda t: (-int(rows[t]), t))
    load = [0] * G
    owner = np.zeros(len(rows), dtype=np.int32)
    for t in order:
        r = min(range(G), key=lambda g: (load[g], g))
        owner[t] = r
        load[r] += int(rows[t])
    return owner


def large_rows(T: int = 512) -> np.ndarray:
    q = (np.arange(T, dtype=np.float64) + 0.5) / T
    return np.floor(1e5 * 200.0 ** (q ** 0.7656)).astype(np.int64)


def make_workload(name: str, G: int = 1, *, dist: Optional[str] = None, mode: str = "float",
                  owner: Optional[np.ndarray] = None, **over) -> Workload:
    """BASELINE.json configs (SURVEY §8(d) 'Concrete inputs')."""
    if name == "tiny":
        kw = dict(T=4, rows=1000, dim=16, B=32, pmin=4, pmax=4, dist="uniform", wdtype="f32", odtype="f32")
    elif name == "single":
        kw = dict(T=26, rows=1_000_000, dim=64, B=16384, pmin=20, pmax=20, dist="zipf", wdtype="f32", odtype="f32")
    elif name == "weak":          # primary reading C16: B_r = 16,384 per GPU
        kw = dict(T=26 * G, rows=2_000_000, dim=128, B=16384 * G, pmin=1, pmax=128, dist="zipf", wdtype="f32", odtype="f32")
    elif name == "weak_paper":    # paper reading C16: global B = 16,384
        kw = dict(T=26 * G, rows=2_000_000, dim=128, B=16384, pmin=1, pmax=128, dist="zipf", wdtype="f32", odtype="f32")
    elif name == "strong":
        kw = dict(T=208, rows=2_000_000, dim=128, B=65536, pmin=1, pmax=32, dist="zipf", wdtype="f32", odtype="f32")
    elif name == "large":
        kw = dict(T=512, rows=large_rows(512), dim=256, B=65536, pmin=1, pmax=100, dist="zipf", wdtype="bf16", odtype="bf16")
    elif name == "large_shard":   # one rank's LPT share of `large` (64 tables, 150 GB bf16) run at G = 1
        share = large_rows(512)[lpt_placement(large_rows(512), 8) == 0]
        kw = dict(T=len(share), rows=share, dim=256, B=65536, pmin=1, pmax=100, dist="zipf", wdtype="bf16",
                  odtype="bf16")
    else:
        raise ValueError(name)
    kw.update(over)
    if dist is not None:
        kw["dist"] = dist
    T = int(kw["T"])
    rows = np.broadcast_to(np.asarray(kw["rows"], dtype=np.int64), (T,)).copy()
    if owner is None:
        owner = lpt_placement(rows, G) if name == "large" else contiguous_placement(T, G)
    owner = np.asarray(owner, dtype=np.int32)
    phys = np.arange(T, dtype=np.int64)
    if name == "strong" and G == 1 and kw.get("alias", True):
        phys = phys // 2          # C27: 104 physical tables back 208 logical tables
    return Workload(name=name, G=G, T=T, rows=rows, dim=int(kw["dim"]), B=int(kw["B"]),
                    pmin=int(kw["pmin"]), pmax=int(kw["pmax"]), dist=kw["dist"], alpha=float(kw.get("alpha", 1.05)),
                    wdtype=kw["wdtype"], odtype=kw["odtype"], owner=owner, phys=phys, mode=mode,
                    table_seed=int(kw.get("table_seed", 20241119)))


def table_csr(w: Workload, batch_seed: int, t: int) -> tuple[np.ndarray, np.ndarray]:
    """Per-table CSR (offsets [B+1], indices [nnz_t]) of logical table t."""
    L = pooling_lengths(batch_seed, t, w.B, w.pmin, w.pmax)
    off = np.zeros(w.B + 1, dtype=np.int64)
    np.cumsum(L, out=off[1:])
    # the rank->row bijection is keyed by the TABLE seed: hot rows stay hot across batches
    idx = table_indices(batch_seed, t, np.arange(off[-1], dtype=np.int64), int(w.rows[t]), w.dist, w.alpha,
                        perm_seed=w.table_seed)
    return off, idx


def rank_csr(w: Workload, batch_seed: int, r: int) -> tuple[np.ndarray, np.ndarray]:
    """Rank r's combined table-major CSR: bag (t_l, b) spans
    offsets[t_l*B + b] .. offsets[t_l*B + b + 1]; indices are local row ids."""
    offs, idxs = [np.zeros(1, dtype=np.int64)], []
    base = 0
    for t in w.local_tables(r):
        o, x = table_csr(w, batch_seed, int(t))
        offs.append(o[1:] + base)
        idxs.append(x)
        base += int(o[-1])
    return np.concatenate(offs), (np.concatenate(idxs) if idxs else np.zeros(0, dtype=np.int64))
