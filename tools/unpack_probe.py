"""Throughput of the comparison path's unpack kernel (emb_baseline_unpack) at the weak
config's output size (B_r = 16 384, T = 26, d = 128 fp32: 218 MB read + 218 MB written),
against the HBM copy peak.  Tables are tiny (the unpack does not read them)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

from paper_conf_sc_chenbyo24_b200 import emb as E
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

dev = torch.device("cuda", 0)
T, d, B = int(os.environ.get("T", 26)), int(os.environ.get("D", 128)), int(os.environ.get("B", 16384))
tabs = [torch.zeros((1000, d), device=dev) for _ in range(T)]
layer = PgasEmbedding(0, 1, 0, [1000] * T, [0] * T, d, tabs, B)
recv = torch.randn(B * T * d, device=dev)
out = torch.empty((B, T, d), device=dev)
s = torch.cuda.Stream()
for _ in range(5):
    E.emb_baseline_unpack(layer.ctx, recv, out, s)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
n = 50
e0.record(s)
for _ in range(n):
    E.emb_baseline_unpack(layer.ctx, recv, out, s)
e1.record(s)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / n
nbytes = 2 * B * T * d * 4
assert torch.equal(out.view(-1), recv)          # G = 1: the unpack map is the identity
print(json.dumps({"unpack_ms": ms, "bytes": nbytes, "GBs": nbytes / ms / 1e6}))
layer.close()
