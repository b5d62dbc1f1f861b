"""Small end-to-end run for compute-sanitizer (memcheck / racecheck / synccheck):
forward at G=1 and simulated G=2 (fused kernel, flags, unpack), pipelined host path and
backward (both algorithms).  Usage: compute-sanitizer --tool memcheck python tools/sanitize.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np
import torch

import emb_test_helpers as H
import synth
from paper_conf_sc_chenbyo24_b200 import emb as E
from paper_conf_sc_chenbyo24_b200.comm import LocalGroup, run_ranks
from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding

dev = torch.device("cuda", 0)
for G in (1, 2):
    w = synth.make_workload("tiny", G=G, pmin=0, pmax=20, B=67, T=4, dim=64, rows=300, dist="zipf")
    tabs = H.np_tables(w)
    offs, idxs = H.np_csrs(w, 3)
    ref = H.oracle_outputs(w, 3, tabs, (offs, idxs))
    tdev = [[torch.from_numpy(tabs[int(w.phys[t])]).to(dev) for t in w.local_tables(r)] for r in range(G)]
    grp = LocalGroup(G) if G > 1 else None
    layers = run_ranks(G, lambda r: PgasEmbedding(r, G, 0, w.rows, w.owner, w.dim, tdev[r], w.B,
                                                  allgather=grp.allgather_for(r) if grp else None,
                                                  options={"timeout_ms": 60000}, backward=True))
    ins = [(torch.from_numpy(offs[r]).to(dev), torch.from_numpy(idxs[r]).to(dev)) for r in range(G)]
    streams = [torch.cuda.Stream() for _ in range(G)]
    # separate waits: the sanitizer may serialize kernels, and an in-kernel wait on a peer
    # whose kernel cannot start would only end at the timeout
    fl = E.EMB_FWD_CHECK_BOUNDS | (E.EMB_FWD_SEPARATE_WAIT if G > 1 else 0)
    for ep in range(3):
        ys = [layers[r].forward(ins[r][0], ins[r][1], fl, streams[r]) for r in range(G)]
        if G > 1:
            for r in range(G):
                layers[r].wait(streams[r])
        torch.cuda.synchronize()
        for r in range(G):
            assert np.array_equal(ys[r].cpu().numpy(), ref[r]), "sanitize run: mismatch"
    for r in range(G):
        b = layers[r].forward_baseline(ins[r][0], ins[r][1]) if G == 1 else None
    dW = [[torch.zeros((int(w.rows[t]), w.dim), device=dev) for t in w.local_tables(r)] for r in range(G)]
    for r in range(G):
        with torch.cuda.stream(streams[r]):
            layers[r].grad_slot(streams[r]).fill_(1.0)
        layers[r].grad_ready(streams[r])
    torch.cuda.synchronize()
    for r in range(G):
        layers[r].backward(ins[r][0], ins[r][1], dW[r], 0, streams[r], publish=False)
    torch.cuda.synchronize()
    # sorted backward algorithm (radix sort + segmented sum), same slots and flags
    for algo in (1,):
        for r in range(G):
            E.emb_set_option(layers[r].ctx, "bwd_algo", algo)
            with torch.cuda.stream(streams[r]):
                layers[r].grad_slot(streams[r]).fill_(1.0)
            layers[r].grad_ready(streams[r])
        torch.cuda.synchronize()
        for r in range(G):
            layers[r].backward(ins[r][0], ins[r][1], dW[r], 0, streams[r], publish=False)
        torch.cuda.synchronize()
    if G == 1:
        ho, hx = torch.from_numpy(offs[0]).pin_memory(), torch.from_numpy(idxs[0]).pin_memory()
        hout = torch.empty((w.B, w.T, w.dim)).pin_memory()
        E.emb_forward_host_async(layers[0].ctx, ho, hx, hout)
        E.emb_host_drain(layers[0].ctx)
        torch.cuda.synchronize()
        assert np.array_equal(hout.numpy(), ref[0])
    for r in range(G):
        assert layers[r].device_error() == 0
    run_ranks(G, lambda r: layers[r].close())
print("sanitize workload OK")
