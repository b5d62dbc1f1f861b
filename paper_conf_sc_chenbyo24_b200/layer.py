"""Rank-level EMB layer on top of the C ABI (Listing 1: the DLRM
calls LookupFunction.apply(weights, offsets, indices, outputs) and continues with
`outputs`).  Holds the context, exposes the PGAS forward and the conventional
comparison path (pool kernel -> NCCL all_to_all_single -> unpack kernel, L155/L193).
Marshalling only: all arithmetic runs in libemb.so.
"""
from __future__ import annotations

from typing import Optional, Sequence

import torch

from . import emb as E


class _CAI:
    def __init__(self, ptr: int, shape, typestr: str):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def wrap_device(ptr: int, shape, dtype: torch.dtype, device) -> torch.Tensor:
    """Zero-copy torch view of a library-owned device buffer."""
    if dtype == torch.float32:
        return torch.as_tensor(_CAI(ptr, shape, "<f4"), device=device)
    if dtype == torch.bfloat16:
        return torch.as_tensor(_CAI(ptr, shape, "<i2"), device=device).view(torch.bfloat16)
    raise ValueError(dtype)


def _tdt(code: int) -> torch.dtype:
    return torch.float32 if code == E.EMB_F32 else torch.bfloat16


class PgasEmbedding:
    """One rank's share of a table-wise model-parallel EMB layer."""

    def __init__(self, rank: int, world_size: int, device: int, rows: Sequence[int], owner: Sequence[int], dim: int,
                 local_weights: Sequence[torch.Tensor], global_batch: int, weight_dtype="f32", out_dtype="f32",
                 allgather=None, options: Optional[dict] = None, backward: bool = False, shards=None):
        self.device = torch.device("cuda", device)
        self.ctx = E.emb_init(rank, world_size, device, allgather)
        if backward:
            E.emb_set_option(self.ctx, "enable_backward", 1)
        self._weights = list(local_weights)  # zero-copy: keep alive
        if shards is None:
            E.emb_register_tables(self.ctx, rows, owner, dim, weight_dtype, out_dtype, global_batch, self._weights)
        else:  # f3: shards = [(t, s, lo, hi, owner)], local_weights in ascending (t, s) of this rank
            sh = sorted((int(t), int(s_), int(lo), int(o)) for (t, s_, lo, hi, o) in shards)
            nsh = [sum(1 for x in sh if x[0] == t) for t in range(len(rows))]
            E.emb_register_sharded_tables(self.ctx, rows, nsh, [x[3] for x in sh], [x[2] for x in sh], dim,
                                          weight_dtype, out_dtype, global_batch, self._weights)
        for k, v in (options or {}).items():
            E.emb_set_option(self.ctx, k, v)
        self.info = E.emb_get_info(self.ctx)
        self.T = self.info["num_tables"]
        self.T_r = self.info["num_local_tables"]
        self.dim = dim
        self.B = global_batch
        self.B_r = self.info["local_batch"]
        self.out_dtype = _tdt(self.info["out_dtype"])
        self.sharded = shards is not None
        self._send = self._recv = self._out = None

    # ---- PGAS fused path (Listing 2) ----------------------------------------------------
    def forward(self, offsets: torch.Tensor, indices: torch.Tensor, flags: int = 0, stream=None) -> torch.Tensor:
        ptr = E.emb_forward(self.ctx, offsets, indices, flags, stream)
        return wrap_device(ptr, (self.B_r, self.T, self.dim), self.out_dtype, self.device)

    def wait(self, stream=None) -> None:
        E.emb_wait(self.ctx, stream)

    # ---- comparison path (L155, L193) ---------------------------------------------------
    def _baseline_buffers(self):
        if self._send is None:
            sc, rc = E.emb_baseline_splits(self.ctx)
            self._send_counts, self._recv_counts = sc, rc
            # f3 row-sharded tables exchange fp32 partials (combined in shard order by the unpack)
            xdt = torch.float32 if self.sharded else self.out_dtype
            self._send = torch.empty(max(sum(sc), 1), dtype=xdt, device=self.device)
            self._recv = torch.empty(max(sum(rc), 1), dtype=xdt, device=self.device)
            self._out = torch.empty((self.B_r, self.T, self.dim), dtype=self.out_dtype, device=self.device)
        return self._send, self._recv, self._out

    def forward_baseline(self, offsets: torch.Tensor, indices: torch.Tensor, group=None, flags: int = 0,
                         stream=None, single_float: bool = False, pool_only: bool = False,
                         always_exchange: bool = False) -> torch.Tensor:
        """pool kernel -> all_to_all_single(async_op=True).wait() -> unpack kernel (L155, L193).
        single_float: the exchange sends ONE float per peer instead of the pooled vectors and the
        unpack still runs over the (stale) receive buffer -- the paper's probe for the
        sync + unpack share of the exchange phase (L286-292); pool_only: stop after the pool;
        always_exchange: run the collective + unpack even at G = 1 (a self-exchange)."""
        send, recv, out = self._baseline_buffers()
        E.emb_baseline_pool(self.ctx, offsets, indices, send, flags, stream)
        if pool_only:
            return send
        if self.ctx.world_size == 1 and not always_exchange:
            if self.sharded:     # G = 1, row shards: no exchange, the partials still need their combine
                E.emb_baseline_unpack(self.ctx, send, out, stream)
                return out
            # G = 1: send already is [B][T][d]; no exchange, no unpack
            return send[: self.B_r * self.T * self.dim].view(self.B_r, self.T, self.dim)
        import torch.distributed as dist
        G = self.ctx.world_size
        sc, rc = self._send_counts, self._recv_counts
        s_in, s_out = (send, recv) if not single_float else (send[:G], recv[:G])
        if single_float:
            sc, rc = [1] * G, [1] * G
        if dist.get_backend(group) == "nccl":
            work = dist.all_to_all_single(s_out, s_in, output_split_sizes=rc, input_split_sizes=sc, group=group,
                                          async_op=True)
            work.wait()
        else:  # gloo (CPU test harness): stage the exchange through host memory
            torch.cuda.current_stream(self.device).synchronize() if stream is None else stream.synchronize()
            hs, hr = s_in.cpu(), torch.empty(s_out.shape, dtype=s_out.dtype)
            dist.all_to_all_single(hr, hs, output_split_sizes=rc, input_split_sizes=sc, group=group)
            s_out.copy_(hr)
        E.emb_baseline_unpack(self.ctx, recv, out, stream)
        return out

    def info_now(self) -> dict:
        """emb_get_info of the context (epoch, launch shape, kernels per call, ...)."""
        return E.emb_get_info(self.ctx)

    # ---- f2 backward (§V) ---------------------------------------------
    def grad_slot(self, stream=None) -> torch.Tensor:
        """fp32 [B_r][T][d] view of this rank's output-gradient slot for the next backward;
        fill it on `stream` before calling backward()."""
        ptr = E.emb_backward_grad_slot(self.ctx, stream)
        return wrap_device(ptr, (self.B_r, self.T, self.dim), torch.float32, self.device)

    def grad_ready(self, stream=None) -> None:
        """Publish this rank's filled gradient slot to the peers (release)."""
        E.emb_backward_grad_ready(self.ctx, stream)

    def backward(self, offsets: torch.Tensor, indices: torch.Tensor, dW: Sequence[torch.Tensor], flags: int = 0,
                 stream=None, publish: bool = True) -> None:
        """Accumulate dL/dW of this rank's tables into dW[t_l] (fp32 [M_t][d]).  With
        publish=True the slot is published first (one rank per GPU); ranks sharing a GPU
        call grad_ready() on all ranks first and pass publish=False."""
        if publish:
            E.emb_backward_grad_ready(self.ctx, stream)
        E.emb_backward(self.ctx, offsets, indices, list(dW), flags, stream)

    def device_error(self, clear: bool = False) -> int:
        return E.emb_query_device_error(self.ctx, clear)

    def close(self) -> None:
        if self.ctx is not None and self.ctx.ptr:
            E.emb_finalize(self.ctx)
        self.ctx = None
