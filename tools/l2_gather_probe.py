"""Attainable L2->SM read bandwidth for THIS access pattern: the fused kernel itself on an
L2-resident variant of the weak config (26 tables x 4000 rows x 512 B = 53 MB, uniform
ids).  Run under ncu to read lts__t_sectors_srcunit_tex_op_read for the kernel."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch

import synth
import synth.gpu as SG
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

dev = torch.device("cuda", 0)
w = synth.make_workload("weak", G=1, rows=int(os.environ.get("ROWS", "4000")), dist="uniform")
tables, _ = SG.local_tables(w, 0, dev)
off, idx = SG.rank_csr(w, w.batch_seed(0), 0, dev)
layer = PgasEmbedding(0, 1, 0, w.rows, w.owner, w.dim, tables, w.B)
for _ in range(5):
    layer.forward(off, idx)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
for _ in range(20):
    layer.forward(off, idx)
e1.record()
torch.cuda.synchronize()
print("ms", e0.elapsed_time(e1) / 20)
layer.close()
