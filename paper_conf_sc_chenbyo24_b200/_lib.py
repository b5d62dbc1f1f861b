"""ctypes loader for the in-tree libemb.so (include/emb.h).  No fallback: if the
library is missing or fails to load this raises, loudly."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libemb.so")
if os.environ.get("EMB_LIB"):            # experiment builds (tools/variants.py) only
    LIB_PATH = os.environ["EMB_LIB"]

EMB_OK, EMB_ERR_ARG, EMB_ERR_STATE, EMB_ERR_CUDA, EMB_ERR_NOMEM, EMB_ERR_PEER, EMB_ERR_TIMEOUT, EMB_ERR_BOUNDS = range(8)
STATUS_NAMES = ["EMB_OK", "EMB_ERR_ARG", "EMB_ERR_STATE", "EMB_ERR_CUDA", "EMB_ERR_NOMEM", "EMB_ERR_PEER",
                "EMB_ERR_TIMEOUT", "EMB_ERR_BOUNDS"]
EMB_F32, EMB_BF16 = 0, 1
EMB_FWD_CHECK_BOUNDS = 0x1
EMB_FWD_SEPARATE_WAIT = 0x2
EMB_DEVERR_TIMEOUT = 0x1
EMB_DEVERR_BOUNDS = 0x2
EMB_DEVERR_CAPACITY = 0x4

ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t)


class EmbInfo(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world_size", C.c_int32), ("device", C.c_int32), ("num_sms", C.c_int32),
                ("num_tables", C.c_int32), ("num_local_tables", C.c_int32), ("dim", C.c_int32),
                ("weight_dtype", C.c_int32), ("out_dtype", C.c_int32), ("global_batch", C.c_int64),
                ("local_batch_start", C.c_int64), ("local_batch", C.c_int64), ("epoch", C.c_uint64),
                ("grid", C.c_int32), ("block", C.c_int32), ("lanes", C.c_int32), ("vec_bytes", C.c_int32),
                ("vecs_per_lane", C.c_int32), ("out_slot_bytes", C.c_int64), ("out_slots", C.c_int32),
                ("fwd_launches", C.c_int32), ("bwd_launches", C.c_int32), ("reserved", C.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


# symbol -> (restype, argtypes); must match include/emb.h (checked by tests/test_abi.py)
SIGNATURES = {
    "emb_init": (C.c_int, [C.c_int, C.c_int, C.c_int, ALLGATHER_FN, C.c_void_p, C.POINTER(C.c_void_p)]),
    "emb_register_tables": (C.c_int, [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int32), C.c_int32,
                                      C.c_int, C.c_int, C.c_int64, C.POINTER(C.c_void_p)]),
    "emb_register_sharded_tables": (C.c_int, [C.c_void_p, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int32),
                                              C.POINTER(C.c_int32), C.POINTER(C.c_int64), C.c_int32, C.c_int, C.c_int,
                                              C.c_int64, C.POINTER(C.c_void_p)]),
    "emb_forward": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.POINTER(C.c_void_p)]),
    "emb_forward_i32": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.POINTER(C.c_void_p)]),
    "emb_wait": (C.c_int, [C.c_void_p, C.c_void_p]),
    "emb_forward_host": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    "emb_forward_host_async": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    "emb_forward_host_async_i32": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    "emb_host_drain": (C.c_int, [C.c_void_p, C.c_void_p]),
    "emb_finalize": (C.c_int, [C.c_void_p]),
    "emb_local_batch": (C.c_int, [C.c_void_p, C.c_int, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
    "emb_get_info": (C.c_int, [C.c_void_p, C.POINTER(EmbInfo)]),
    "emb_set_option": (C.c_int, [C.c_void_p, C.c_char_p, C.c_int64]),
    "emb_query_device_error": (C.c_int, [C.c_void_p, C.POINTER(C.c_uint32), C.c_int]),
    "emb_last_error": (C.c_char_p, [C.c_void_p]),
    "emb_backward_grad_slot": (C.c_int, [C.c_void_p, C.c_void_p, C.POINTER(C.c_void_p)]),
    "emb_backward_grad_ready": (C.c_int, [C.c_void_p, C.c_void_p]),
    "emb_backward": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.POINTER(C.c_void_p), C.c_uint32, C.c_void_p]),
    "emb_trace_read": (C.c_int, [C.c_void_p, C.c_void_p, C.c_int64, C.POINTER(C.c_int64)]),
    "emb_baseline_splits": (C.c_int, [C.c_void_p, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
    "emb_baseline_pool": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    "emb_baseline_pool_i32": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
    "emb_baseline_unpack": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]),
}

_lib = None


def lib() -> C.CDLL:
    """Load libemb.so (built by __graft_entry__.build()).  Raises if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libemb.so not found at {LIB_PATH}: run `python -m paper_conf_sc_chenbyo24_b200.build` "
                               "(there is no CPU fallback)")
        L = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib
