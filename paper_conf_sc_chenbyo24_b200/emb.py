"""Thin Python binding of include/emb.h -- same names, argument marshalling only.

Every step of the forward runs in libemb.so's kernels; this module converts torch
tensors / streams / Python lists into the plain pointers and sizes of the C ABI and
turns non-OK statuses into EmbError.  (Listing 1: the paper wraps
its backend as torch.ops.PGAS.forward; here the boundary is a C ABI.)
"""
from __future__ import annotations

import ctypes as C
from typing import Callable, List, Optional, Sequence, Tuple

from . import _lib
from ._lib import (EMB_BF16, EMB_DEVERR_BOUNDS, EMB_DEVERR_CAPACITY, EMB_DEVERR_TIMEOUT, EMB_F32,  # noqa: F401
                   EMB_FWD_CHECK_BOUNDS, EMB_FWD_SEPARATE_WAIT, STATUS_NAMES, EmbInfo)


class EmbError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else status}: {msg}")
        self.status = status


class EmbCtx:
    """Owns the opaque emb_ctx_t* plus the ctypes callback that must outlive it."""

    def __init__(self, ptr: int, callback, rank: int, world_size: int, device: int):
        self.ptr = ptr
        self._callback = callback
        self.rank = rank
        self.world_size = world_size
        self.device = device

    @property
    def _as_parameter_(self):
        return C.c_void_p(self.ptr)


def _ptr(x) -> Optional[int]:
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    raise TypeError(f"cannot take a device pointer of {type(x)}")


def _stream(s) -> Optional[int]:
    if s is None:
        try:
            import torch
            return torch.cuda.current_stream().cuda_stream
        except Exception:
            return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _is_i32(offsets, indices) -> bool:
    """Index width of a CSR given as torch tensors (int32 -> the *_i32 entry points, C12);
    plain integer addresses are int64."""
    wo = getattr(offsets, "dtype", None)
    wi = getattr(indices, "dtype", None)
    names = {str(wo), str(wi)} - {"None"}
    if not names:
        return False
    if len(names) != 1:
        raise TypeError(f"offsets and indices must have the same dtype, got {wo} and {wi}")
    n = names.pop()
    if n in ("torch.int32", "int32"):
        return True
    if n in ("torch.int64", "int64"):
        return False
    raise TypeError(f"offsets / indices must be int64 or int32, got {n}")


def _check(ctx: Optional[EmbCtx], st: int) -> None:
    if st != 0:
        msg = _lib.lib().emb_last_error(ctx.ptr if ctx is not None else None)
        raise EmbError(st, (msg or b"").decode(errors="replace"))


def _dtype_code(d) -> int:
    if d in (EMB_F32, EMB_BF16):
        return int(d)
    s = str(d)
    if s in ("f32", "float32", "torch.float32"):
        return EMB_F32
    if s in ("bf16", "bfloat16", "torch.bfloat16"):
        return EMB_BF16
    raise ValueError(f"unsupported dtype {d}")


def emb_init(rank: int, world_size: int, cuda_device: int, allgather: Optional[Callable[[bytes], bytes]] = None) -> EmbCtx:
    """allgather(my_bytes) -> concatenated bytes of all ranks (rank order)."""
    if allgather is not None:
        def _cb(user, send, recv, nbytes):
            try:
                mine = C.string_at(send, nbytes)
                allb = allgather(mine)
                if len(allb) != nbytes * world_size:
                    return 1
                C.memmove(recv, allb, len(allb))
                return 0
            except Exception:  # never let an exception cross the C ABI
                import traceback
                traceback.print_exc()
                return 1
        cb = _lib.ALLGATHER_FN(_cb)
    else:
        cb = C.cast(None, _lib.ALLGATHER_FN)
    out = C.c_void_p()
    st = _lib.lib().emb_init(rank, world_size, cuda_device, cb, None, C.byref(out))
    _check(None, st)
    return EmbCtx(out.value, cb, rank, world_size, cuda_device)


def emb_register_tables(ctx: EmbCtx, rows: Sequence[int], owner: Sequence[int], dim: int, weight_dtype,
                        out_dtype, global_batch: int, local_weights: Sequence) -> None:
    T = len(rows)
    rows_a = (C.c_int64 * T)(*[int(r) for r in rows])
    own_a = (C.c_int32 * T)(*[int(o) for o in owner])
    nl = len(local_weights)
    w_a = (C.c_void_p * max(nl, 1))(*[_ptr(w) for w in local_weights])
    st = _lib.lib().emb_register_tables(ctx, T, rows_a, own_a, int(dim), _dtype_code(weight_dtype),
                                        _dtype_code(out_dtype), int(global_batch), w_a)
    _check(ctx, st)


def emb_register_sharded_tables(ctx: EmbCtx, rows: Sequence[int], num_shards: Sequence[int],
                                shard_owner: Sequence[int], shard_row_start: Sequence[int], dim: int, weight_dtype,
                                out_dtype, global_batch: int, local_weights: Sequence) -> None:
    T = len(rows)
    n = sum(int(x) for x in num_shards)
    rows_a = (C.c_int64 * T)(*[int(r) for r in rows])
    ns_a = (C.c_int32 * T)(*[int(x) for x in num_shards])
    own_a = (C.c_int32 * n)(*[int(o) for o in shard_owner])
    lo_a = (C.c_int64 * n)(*[int(x) for x in shard_row_start])
    nl = len(local_weights)
    w_a = (C.c_void_p * max(nl, 1))(*[_ptr(w) for w in local_weights])
    st = _lib.lib().emb_register_sharded_tables(ctx, T, rows_a, ns_a, own_a, lo_a, int(dim), _dtype_code(weight_dtype),
                                                _dtype_code(out_dtype), int(global_batch), w_a)
    _check(ctx, st)


def emb_forward(ctx: EmbCtx, offsets, indices, flags: int = 0, stream=None) -> int:
    """Returns the device address of this epoch's Y_r = [B_r][T][d] (int32 tensors call
    emb_forward_i32)."""
    out = C.c_void_p()
    fn = _lib.lib().emb_forward_i32 if _is_i32(offsets, indices) else _lib.lib().emb_forward
    st = fn(ctx, _ptr(offsets), _ptr(indices), int(flags), _stream(stream), C.byref(out))
    _check(ctx, st)
    return out.value


def emb_wait(ctx: EmbCtx, stream=None) -> None:
    _check(ctx, _lib.lib().emb_wait(ctx, _stream(stream)))


def emb_forward_host(ctx: EmbCtx, h_offsets, h_indices, h_out, flags: int = 0, stream=None) -> None:
    """Host (ideally pinned) CSR in, host Y_r out; asynchronous on `stream`."""
    st = _lib.lib().emb_forward_host(ctx, _ptr(h_offsets), _ptr(h_indices), int(flags), _stream(stream), _ptr(h_out))
    _check(ctx, st)


def emb_forward_host_async(ctx: EmbCtx, h_offsets, h_indices, h_out, flags: int = 0, stream=None) -> None:
    """Pipelined host path: H2D / kernel / D2H of consecutive calls overlap (int32 host
    tensors call emb_forward_host_async_i32)."""
    fn = _lib.lib().emb_forward_host_async_i32 if _is_i32(h_offsets, h_indices) else _lib.lib().emb_forward_host_async
    st = fn(ctx, _ptr(h_offsets), _ptr(h_indices), int(flags), _stream(stream), _ptr(h_out))
    _check(ctx, st)


def emb_host_drain(ctx: EmbCtx, stream=None) -> None:
    _check(ctx, _lib.lib().emb_host_drain(ctx, _stream(stream)))


def emb_finalize(ctx: EmbCtx) -> None:
    if ctx.ptr:
        st = _lib.lib().emb_finalize(ctx)
        ctx.ptr = 0
        if st != 0:
            raise EmbError(st, "emb_finalize failed")


def emb_local_batch(ctx: EmbCtx, rank: int) -> Tuple[int, int]:
    s, n = C.c_int64(), C.c_int64()
    _check(ctx, _lib.lib().emb_local_batch(ctx, int(rank), C.byref(s), C.byref(n)))
    return s.value, n.value


def emb_get_info(ctx: EmbCtx) -> dict:
    i = EmbInfo()
    _check(ctx, _lib.lib().emb_get_info(ctx, C.byref(i)))
    return i.as_dict()


def emb_set_option(ctx: EmbCtx, key: str, value: int) -> None:
    _check(ctx, _lib.lib().emb_set_option(ctx, key.encode(), int(value)))


def emb_query_device_error(ctx: EmbCtx, clear: bool = False) -> int:
    w = C.c_uint32()
    _check(ctx, _lib.lib().emb_query_device_error(ctx, C.byref(w), 1 if clear else 0))
    return w.value


def emb_backward_grad_slot(ctx: EmbCtx, stream=None) -> int:
    """Device address of this rank's fp32 [B_r][T][d] gradient slot for the next backward."""
    out = C.c_void_p()
    _check(ctx, _lib.lib().emb_backward_grad_slot(ctx, _stream(stream), C.byref(out)))
    return out.value


def emb_backward_grad_ready(ctx: EmbCtx, stream=None) -> None:
    _check(ctx, _lib.lib().emb_backward_grad_ready(ctx, _stream(stream)))


def emb_backward(ctx: EmbCtx, offsets, indices, dW: Sequence, flags: int = 0, stream=None) -> None:
    n = len(dW)
    arr = (C.c_void_p * max(n, 1))(*[_ptr(x) for x in dW])
    _check(ctx, _lib.lib().emb_backward(ctx, _ptr(offsets), _ptr(indices), arr, int(flags), _stream(stream)))


def emb_trace_read(ctx: EmbCtx, capacity: int):
    """f1 trace: numpy uint64 [n, 2] = {globaltimer ns, remote_bytes << 32 | local_bytes}."""
    import numpy as np
    buf = np.zeros((max(int(capacity), 1), 2), dtype=np.uint64)
    n = C.c_int64()
    _check(ctx, _lib.lib().emb_trace_read(ctx, buf.ctypes.data, int(capacity), C.byref(n)))
    return buf[: n.value]


def emb_last_error(ctx: Optional[EmbCtx]) -> str:
    return (_lib.lib().emb_last_error(ctx.ptr if ctx is not None else None) or b"").decode(errors="replace")


def emb_baseline_splits(ctx: EmbCtx) -> Tuple[List[int], List[int]]:
    G = ctx.world_size
    s, r = (C.c_int64 * G)(), (C.c_int64 * G)()
    _check(ctx, _lib.lib().emb_baseline_splits(ctx, s, r))
    return list(s), list(r)


def emb_baseline_pool(ctx: EmbCtx, offsets, indices, send, flags: int = 0, stream=None) -> None:
    fn = _lib.lib().emb_baseline_pool_i32 if _is_i32(offsets, indices) else _lib.lib().emb_baseline_pool
    _check(ctx, fn(ctx, _ptr(offsets), _ptr(indices), int(flags), _stream(stream), _ptr(send)))


def emb_baseline_unpack(ctx: EmbCtx, recv, out, stream=None) -> None:
    _check(ctx, _lib.lib().emb_baseline_unpack(ctx, _ptr(recv), _stream(stream), _ptr(out)))
