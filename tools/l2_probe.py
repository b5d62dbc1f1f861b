"""Measure L2 and HBM streaming read bandwidth on the GPU box (tool; see l2_probe.cu)."""
import ctypes
import json
import os
import subprocess

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "csrc", "libl2probe.so")
if not os.path.exists(SO):
    subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared",
                           "-Xcompiler", "-fPIC", os.path.join(HERE, "csrc", "l2_probe.cu"), "-o", SO])
L = ctypes.CDLL(SO)
L.l2_probe.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                       ctypes.c_void_p]
sink = torch.zeros(1, dtype=torch.int64, device="cuda")
res = {}
for mb, reps in [(16, 200), (48, 80), (96, 40), (4096, 2)]:
    buf = torch.randint(0, 255, (mb << 20,), dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    for grid_mult in (4, 8, 16):
        grid = 148 * grid_mult
        L.l2_probe(buf.data_ptr(), buf.numel(), 2, grid, 256, sink.data_ptr(), s.cuda_stream)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        L.l2_probe(buf.data_ptr(), buf.numel(), reps, grid, 256, sink.data_ptr(), s.cuda_stream)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        gbs = buf.numel() * reps / ms / 1e6
        res[f"{mb}MB_grid{grid}"] = round(gbs, 1)
    del buf
print(json.dumps({"read_GBps": res, "note": "ld.global.cg 16 B streaming reads; <=96 MB buffers are L2-resident"}))
