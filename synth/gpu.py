"""Device-side generation of the synthetic workload (tables + per-rank CSR) with
libsynth.so, the bit-exact twin of synth/__init__.py.  Input generation only."""
from __future__ import annotations

import ctypes as C
import os
from typing import Dict, List, Tuple

import numpy as np
import torch

from . import Workload, perm_params, zipf_cdf

_LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libsynth.so")
_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `python -m paper_conf_sc_chenbyo24_b200.build`")
        L = C.CDLL(_LIB_PATH)
        L.synth_gen_table.argtypes = [C.c_void_p, C.c_int64, C.c_int32, C.c_int32, C.c_int32, C.c_uint64, C.c_int64, C.c_void_p]
        L.synth_gen_lengths.argtypes = [C.c_void_p, C.c_int64, C.c_uint64, C.c_int64, C.c_int64, C.c_int64, C.c_void_p]
        L.synth_gen_indices.argtypes = [C.c_void_p, C.c_int64, C.c_int64, C.c_uint64, C.c_int64, C.c_int64, C.c_int32,
                                        C.c_void_p, C.c_int64, C.c_int64, C.c_void_p]
        for f in (L.synth_gen_table, L.synth_gen_lengths, L.synth_gen_indices):
            f.restype = C.c_int
        _lib = L
    return _lib


def _ck(rc: int, what: str):
    if rc != 0:
        raise RuntimeError(f"{what} failed with cudaError {rc}")


def _s():
    return torch.cuda.current_stream().cuda_stream


_MODES = {"float": 0, "int": 1, "identity": 2}


def gen_table(w: Workload, phys: int, rows: int, device) -> torch.Tensor:
    dt = torch.float32 if w.wdtype == "f32" else torch.bfloat16
    W = torch.empty((rows, w.dim), dtype=dt, device=device)
    _ck(lib().synth_gen_table(W.data_ptr(), rows, w.dim, 0 if w.wdtype == "f32" else 1, _MODES[w.mode],
                              w.table_seed, phys, _s()), "synth_gen_table")
    return W


def local_tables(w: Workload, r: int, device) -> Tuple[List[torch.Tensor], Dict[int, torch.Tensor]]:
    """This rank's tables (ascending global id); aliased logical tables share storage (C27)."""
    phys: Dict[int, torch.Tensor] = {}
    out = []
    for t in w.local_tables(r):
        p = int(w.phys[t])
        if p not in phys:
            phys[p] = gen_table(w, p, int(w.rows[t]), device)
        out.append(phys[p])
    return out, phys


_cdf_cache: Dict[tuple, torch.Tensor] = {}


def _cdf_dev(M: int, alpha: float, device) -> torch.Tensor:
    key = (M, alpha, str(device))
    if key not in _cdf_cache:
        _cdf_cache[key] = torch.from_numpy(np.array(zipf_cdf(M, alpha))).to(device)
    return _cdf_cache[key]


def rank_csr(w: Workload, batch_seed: int, r: int, device) -> Tuple[torch.Tensor, torch.Tensor]:
    """Rank r's table-major CSR on the device; identical to synth.rank_csr."""
    lt = w.local_tables(r)
    Tr, B = len(lt), w.B
    lens = torch.empty(max(Tr * B, 1), dtype=torch.int64, device=device)
    for i, t in enumerate(lt):
        _ck(lib().synth_gen_lengths(lens.data_ptr() + 8 * i * B, B, batch_seed, int(t), w.pmin, w.pmax, _s()),
            "synth_gen_lengths")
    offsets = torch.zeros(Tr * B + 1, dtype=torch.int64, device=device)
    if Tr:
        torch.cumsum(lens[: Tr * B], 0, out=offsets[1:])
    starts = offsets[:: B].cpu().tolist() if Tr else [0]
    nnz = int(starts[-1]) if Tr else 0
    indices = torch.empty(max(nnz, 1), dtype=torch.int64, device=device)
    for i, t in enumerate(lt):
        M = int(w.rows[t])
        cnt = int(starts[i + 1] - starts[i])
        if w.dist == "zipf":
            a, c = perm_params(w.table_seed, int(t), M)
            cdf = _cdf_dev(M, w.alpha, device)
            _ck(lib().synth_gen_indices(indices.data_ptr() + 8 * int(starts[i]), cnt, 0, batch_seed, int(t), M, 1,
                                        cdf.data_ptr(), a, c, _s()), "synth_gen_indices")
        else:
            _ck(lib().synth_gen_indices(indices.data_ptr() + 8 * int(starts[i]), cnt, 0, batch_seed, int(t), M, 0,
                                        None, 0, 0, _s()), "synth_gen_indices")
    return offsets, indices[:nnz] if nnz else indices[:0]
