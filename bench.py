#!/usr/bin/env python
"""Benchmark of the PGAS-style EMB-layer forward (BASELINE.json metric: EMB fwd
samples/sec at 1/2/4/8 B200, max over ranks, + % of the HBM/NVLink roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config weak|single|strong|weak_paper|tiny]
                    [--dist zipf|uniform] [--impl ours|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N

One JSON line on rank 0.  A "step" is one whole EMB forward (lookup + pool + MP->DP
exchange, PAPER.md L197 timed scope) over one batch of synthetic Criteo-shaped input
already resident in HBM; `e2e` repeats it through emb_forward_host with pinned host
CSR in and the host output out.  `--impl reference` times the CPU oracle (this tier's
reference arm) on a bounded sample of the same workload.  Nothing here reads
/root/reference.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "EMB fwd samples/sec at 1/2/4/8 B200 (max over ranks); % of HBM/NVLink roofline"   # BASELINE.json
NVLINK_GBS = 770.0      # measured peer copy per direction (B200_PROFILING.md); nominal 900
HBM_FALLBACK = 6650.0   # B200_PROFILING.md fallback if MEASURED_PEAKS.json is absent


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=100)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--config", default="weak")
    p.add_argument("--dist", default=None, help="override index distribution (zipf|uniform)")
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--mode", default="forward", choices=["forward", "backward"],
                   help="backward = SURVEY row f2 (emb_backward: pull output gradients, scatter into dW)")
    p.add_argument("--batches", type=int, default=4, help="distinct pre-generated batches cycled")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-control", action="store_true", help="skip the uniform-index control measurement")
    p.add_argument("--no-compare", action="store_true", help="skip the NCCL comparison path")
    p.add_argument("--opt", action="append", default=[], help="libemb option key=value")
    p.add_argument("--shards", type=int, default=1,
                   help="f3: split every table into this many row shards (owners round-robin from the table's owner);"
                        " the kernel partitions the full CSR in-kernel and combines partials in shard order")
    p.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                   help="process-group backend (gloo: test harness only; a2a staged through host)")
    p.add_argument("--same-device", action="store_true",
                   help="test harness: every rank on cuda:0 (N>1 on a 1-GPU box; ranks time-slice)")
    return p.parse_args()


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return HBM_FALLBACK, "fallback"


def config_desc(w, N):
    return {"workload": w.name, "tables_total": int(w.T), "tables_per_gpu": int(w.T // max(N, 1)) if w.name != "large" else None,
            "rows_per_table": int(w.rows[0]), "dim": w.dim, "global_batch": int(w.B), "local_batch": int(w.B // N),
            "pooling": f"U{{{w.pmin}..{w.pmax}}}", "indices": f"{w.dist}({w.alpha})" if w.dist == "zipf" else "uniform",
            "weights": w.wdtype, "out": w.odtype, "parallelism": f"table-wise MP x{N} + batch DP x{N}",
            "aliased": int(w.T // (int(w.phys.max()) + 1)) if int(w.phys.max()) + 1 < w.T else 1,
            "l2": "inputs larger than L2 (tables >> 126 MB, rotating CSR batches); no flush",
            "row_shards_per_table": getattr(w, "_shards", 1)}


def unique_rows(w, rank, batch):
    """Distinct (table, row) pairs a batch touches: the rows that must come from HBM
    at least once (compulsory traffic under zipf reuse)."""
    import torch
    off, idx = batch
    lt = w.local_tables(rank)
    starts = off[:: w.B].tolist()
    tot = 0
    for i in range(len(lt)):
        seg = idx[starts[i]: starts[i + 1]]
        if seg.numel():
            tot += int(torch.unique(seg).numel())
    return tot


def compulsory_bytes(w, uniq, nnz, nbags):
    """Unique rows once + every index + every offset + every output vector written."""
    return uniq * w.dim * w.elem_bytes() + nnz * 8 + nbags * (8 + w.dim * w.out_elem_bytes())


def algorithmic_bytes(w, nnz, nbags, remote_bags):
    """per lookup d*e + 8 (row + index); per bag 8 (offset) + d*e_o (output)."""
    e, eo = w.elem_bytes(), w.out_elem_bytes()
    hbm = nnz * (w.dim * e + 8) + nbags * (8 + w.dim * eo)
    nvl = remote_bags * w.dim * eo
    return hbm, nvl


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    def __init__(self, device_index: int):
        self.samples = []
        self.reasons = set()
        self._stop = threading.Event()
        self._th = None
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    _NAMES = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap",
              0x80: "hw_power_brake_slowdown", 0x1: "gpu_idle", 0x2: "applications_clocks_setting"}

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self._NAMES.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.nv:
            self._th = threading.Thread(target=self._run, daemon=True)
            self._th.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._th:
            self._th.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------------------ CPU oracle timing
_POOL_STATE = {}


def _pool_one(i):
    """Worker: the oracle's pool_table_f32 on sampled table i (inputs inherited by fork)."""
    st = _POOL_STATE
    o, x = st["csrs"][i]
    return st["O"].pool_table_f32(st["W"], o, x)


class OracleSampler:
    """Time the oracle AS IT STANDS (oracle.emb_oracle, untuned) on this rank's tables over
    the full batch plus the MP->DP layout step.  The per-table pooling runs as one process
    per host core (fork; the oracle code is unchanged, the tables are independent), the
    layout step in the parent.  If the budget ends first, the result is extrapolated to
    the whole rank workload by table count.  Inputs are generated once, untimed."""

    def __init__(self, w, rank, max_tables=64):
        from oracle import emb_oracle as O
        self.O = O
        self.w = w
        self.lt = list(w.local_tables(rank))
        t0 = self.lt[0]
        self.W = synth.table_rows(w.table_seed, int(w.phys[t0]), int(w.rows[t0]), w.dim, w.mode, w.wdtype)
        M0 = int(w.rows[t0])
        self.folded = any(int(w.rows[t]) != M0 for t in self.lt[:max_tables])
        # mixed table sizes (large config): fold the sampled tables' ids into the one
        # physical table generated for timing (values do not change the oracle's work)
        self.csrs = [(o, x % M0) for o, x in (synth.table_csr(w, w.batch_seed(0), int(t)) for t in self.lt[:max_tables])]
        try:
            self.cores = max(1, len(os.sched_getaffinity(0)))
        except AttributeError:
            self.cores = os.cpu_count() or 1

    def run(self, budget_s=12.0, min_tables=1, parallel=True):
        import multiprocessing as mp
        O, w = self.O, self.w
        n = len(self.csrs)
        # tiny tables: process start-up would dominate, run in one process
        big = int(self.csrs[0][0][-1]) * w.dim >= 10_000_000
        cores = min(self.cores, n) if (parallel and big) else 1
        _POOL_STATE.update(O=O, W=self.W, csrs=self.csrs)
        if cores > 1 and getattr(self, "_pool", None) is None:
            self._pool = mp.get_context("fork").Pool(cores)   # workers inherit W and the CSRs
            self._pool.map(_pool_one, range(min(cores, n)))   # warm the workers (untimed)
        t0 = time.perf_counter()
        Zs, done = [], 0
        if cores > 1:
            while done < n and (done < min_tables or time.perf_counter() - t0 < budget_s):
                k = min(cores, n - done)                      # one wave: a table per core
                Zs += self._pool.map(_pool_one, range(done, done + k))
                done += k
        else:
            while done < n and (done < min_tables or time.perf_counter() - t0 < budget_s):
                Zs.append(_pool_one(done))
                done += 1
        O.mp_to_dp(Zs, w.G)
        dt = time.perf_counter() - t0
        lookups = sum(int(self.csrs[i][0][-1]) for i in range(done))
        per_rank_s = dt * len(self.lt) / done
        return {"value": w.B / per_rank_s, "unit": "samples/s", "cores": cores, "kind": "oracle",
                "sample": f"{done} of {len(self.lt)} local tables x full batch {w.B} ({lookups} lookups; table values "
                          f"from one physical {int(w.rows[self.lt[0]])}x{w.dim} table{', ids folded into it' if self.folded else ''}) "
                          f"+ MP->DP layout, {dt:.2f}s on {cores} process(es), "
                          f"extrapolated to the rank's workload by table count",
                "seconds": dt, "rank_seconds": per_rank_s}


def oracle_sample(w, rank, budget_s=20.0):
    smp = OracleSampler(w, rank)
    try:
        return smp.run(budget_s)
    finally:
        if getattr(smp, "_pool", None) is not None:
            smp._pool.terminate()


def reference_arm(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    N = args.gpus
    w = synth.make_workload(args.config, G=N, dist=args.dist)
    smp = OracleSampler(w, 0)
    per_step = []
    cb = None
    for s in range(args.warmup + args.steps):
        r = smp.run(budget_s=0.0, min_tables=1)             # one wave (a table per core) per step
        if s >= args.warmup:
            per_step.append(r["rank_seconds"])
            cb = r
    if getattr(smp, "_pool", None) is not None:
        smp._pool.terminate()
    sec = float(np.mean(per_step))
    val = w.B / sec
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "samples/s",
            "n_gpus": N, "steps": args.steps, "warmup": args.warmup, "ms_per_step": sec * 1e3,
            "higher_is_better": True, "scaling": "weak" if args.config.startswith("weak") else "strong",
            "vs_baseline": None, "dtype": "f32" if w.wdtype == "f32" else "bf16", "data": "synthetic",
            "config": config_desc(w, N),
            "cpu_baseline": {"value": val, "unit": "samples/s", "cores": cb["cores"], "kind": "oracle",
                             "sample": "per step: " + cb["sample"]},
            "e2e": {"value": val, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "gpu_launches": 0}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------ backward (f2)
def run_backward(args, w, N, rank, local, dev, stream, layer, batches, nnz, uniq, nbags, remote_bags, barrier, timed):
    """One step = publish this rank's output-gradient slot + the fused backward kernel
    (one-sided loads of dY from the DP ranks, red.add into dW).  dY is synthetic
    (standard normal, filled once per slot, untimed); dW accumulates across steps."""
    import torch
    import torch.distributed as dist
    dW = [torch.zeros((int(w.rows[t]), w.dim), device=dev) for t in w.local_tables(rank)]
    gen = torch.Generator(device=dev).manual_seed(1234 + rank)
    for _ in range(2):                                    # fill both ring slots once (untimed)
        with torch.cuda.stream(stream):
            g = layer.grad_slot(stream)
            g.normal_(generator=gen)
        layer.grad_ready(stream)
        o, x = batches[0]
        layer.backward(o, x, dW, 0, stream, publish=False)
    torch.cuda.synchronize()

    def bwd(s):
        o, x = batches[s % len(batches)]
        layer.grad_slot(stream)                           # ring protocol (waits for peers' reads)
        layer.backward(o, x, dW, 0, stream)

    for s in range(args.warmup):
        bwd(s)
    barrier()
    with ClockSampler(local) as clk:
        ms = timed(bwd, args.steps)
    assert layer.device_error() == 0, "device error during the timed region"
    value = w.B / (ms * 1e-3)
    e, row = 4, w.dim * 4                                 # dW and dY are fp32
    nnz_m, uniq_m = float(np.mean(nnz)), float(np.mean(uniq))
    lookup_bytes = nnz_m * (2 * row + 8) + nbags * (8 + row)      # row RMW per lookup + dY/offset per bag
    comp_bytes = uniq_m * 2 * row + nnz_m * 8 + nbags * (8 + row)  # each touched dW row read+written once
    nvl = remote_bags * row
    peak, peak_kind = hbm_peak()
    t_hbm, t_nvl = comp_bytes / (peak * 1e9), nvl / (NVLINK_GBS * 1e9)
    bound = "hbm" if t_hbm >= t_nvl else "nvlink"
    ach = (comp_bytes if bound == "hbm" else nvl) / (ms * 1e-3) / 1e9
    pk = peak if bound == "hbm" else NVLINK_GBS
    roof = {"bound": bound, "achieved": ach, "peak": pk, "unit": "GB/s", "frac": ach / pk, "traffic": None,
            "kernel": "emb_bwd_kernel (one-sided dY loads + red.add.v4.f32 into dW)",
            "algorithmic_bytes_per_launch": comp_bytes if bound == "hbm" else nvl,
            "basis": "compulsory: each touched dW row read+written once (2*d*4) + every index + every offset + "
                     "every dY vector read once",
            "lookup_counted": {"bytes": lookup_bytes, "achieved": lookup_bytes / (ms * 1e-3) / 1e9,
                               "frac": lookup_bytes / (ms * 1e-3) / 1e9 / peak},
            "peak_source": f"{peak_kind} MEASURED_PEAKS.json hbm_gbs", "t_roof_ms": max(t_hbm, t_nvl) * 1e3}
    if not args.opt:                                       # default kernel only: ncu of that kernel
        try:
            with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
                tb = json.load(f).get(f"{w.name}:{w.dist}:G{N}:backward")
            if tb:
                roof["traffic"] = tb["dram_bytes_per_launch"]
                roof["traffic_source"] = tb.get("source")
        except (OSError, ValueError):
            pass
    layer.close()
    if N > 1:
        dist.barrier()
    if rank == 0:
        line = {"metric": "EMB bwd samples/sec (max over ranks)", "value": value, "unit": "samples/s", "n_gpus": N,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "weak" if w.name.startswith("weak") else "strong", "vs_baseline": None, "dtype": "f32",
                "data": "synthetic", "config": {**config_desc(w, N), "mode": "backward (SURVEY f2)"},
                "roofline": roof, "cpu_baseline": None, "e2e": None, "gpu_launches": args.steps * (2 if N > 1 else 1),
                "clocks": clk.summary()}
        print(json.dumps(line), flush=True)
    if N > 1:
        dist.destroy_process_group()
    return 0


# ------------------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    if args.impl == "reference":
        return reference_arm(args)
    import torch
    import torch.distributed as dist

    from paper_conf_sc_chenbyo24_b200 import emb as E
    from paper_conf_sc_chenbyo24_b200.comm import torch_allgather
    from paper_conf_sc_chenbyo24_b200.layer import PgasEmbedding
    import synth.gpu as SG

    N = args.gpus
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != N:
        raise SystemExit(f"--gpus {N} but WORLD_SIZE={world}")
    if args.same_device:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if N > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    w = synth.make_workload(args.config, G=N, dist=args.dist)
    stream = torch.cuda.Stream(device=dev)

    # ---- inputs in HBM (untimed)
    with torch.cuda.stream(stream):
        tables, _phys = SG.local_tables(w, rank, dev)
        batches = [SG.rank_csr(w, w.batch_seed(i), rank, dev) for i in range(args.batches)]
    torch.cuda.synchronize()
    opts = {}
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = int(v)
    nnz = [int(b[0][-1].item()) for b in batches]
    uniq = [unique_rows(w, rank, b) for b in batches]     # untimed: compulsory-traffic basis
    w._shards = args.shards
    shards = None
    if args.shards > 1:
        # f3: table t -> S row shards, shard s on rank (owner[t] + s) % N; each rank needs the
        # FULL CSR of every table it holds a shard of.  Tables are generated where the
        # table's owner is; at N = 1 every shard is a view of the local table.
        if N > 1:
            raise SystemExit("--shards > 1 is exercised at N = 1 in this round (all shards local)")
        args.no_control = True       # the uniform control and the comparison path are table-wise
        args.no_compare = True
        S = args.shards
        shards = []
        for t in range(w.T):
            cuts = np.linspace(0, int(w.rows[t]), S + 1).astype(np.int64)
            for sh in range(S):
                shards.append((t, sh, int(cuts[sh]), int(cuts[sh + 1]), (int(w.owner[t]) + sh) % N))
        tables = [tables[list(w.local_tables(rank)).index(t)][lo:hi] for (t, sh, lo, hi, o) in sorted(shards)]

        def shard_csr(batch):
            off, idx = batch
            lt = list(w.local_tables(rank))
            o_parts, x_parts, base = [torch.zeros(1, dtype=torch.int64, device=dev)], [], 0
            for (t, sh, lo, hi, o) in sorted(shards):
                tl = lt.index(t)
                seg = off[tl * w.B: (tl + 1) * w.B + 1]
                o_parts.append(seg[1:] - seg[0] + base)
                x_parts.append(idx[int(seg[0]): int(seg[-1])])
                base += int(seg[-1] - seg[0])
            return torch.cat(o_parts), torch.cat(x_parts)
        batches = [shard_csr(b) for b in batches]
        torch.cuda.synchronize()
    layer = PgasEmbedding(rank, N, local, w.rows, w.owner, w.dim, tables, w.B, w.wdtype, w.odtype,
                          torch_allgather() if N > 1 else None, opts, backward=(args.mode == "backward"),
                          shards=shards)
    T_r = len(w.local_tables(rank))
    nbags = T_r * w.B
    B_r = layer.B_r
    remote_bags = T_r * (w.B - B_r)

    def barrier():
        if N > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def timed(fn, steps, finish=None):
        barrier()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for s in range(steps):
            fn(s)
        if finish is not None:
            finish()
        ev1.record(stream)
        torch.cuda.synchronize()
        ms = ev0.elapsed_time(ev1) / steps
        if N > 1:
            t = torch.tensor([ms], device=dev if args.backend == "nccl" else "cpu")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    def fwd(s):
        o, x = batches[s % len(batches)]
        layer.forward(o, x, 0, stream)

    if args.mode == "backward":
        return run_backward(args, w, N, rank, local, dev, stream, layer, batches, nnz, uniq, nbags, remote_bags,
                            barrier, timed)

    for s in range(args.warmup):
        fwd(s)
    barrier()
    with ClockSampler(local) as clk:
        ms = timed(fwd, args.steps)
    assert layer.device_error() == 0, "device error during the timed region"
    value = w.B / (ms * 1e-3)

    lookup_bytes, nvl_bytes = algorithmic_bytes(w, float(np.mean(nnz)), nbags, remote_bags)
    hbm_bytes = float(np.mean([compulsory_bytes(w, u, z, nbags) for u, z in zip(uniq, nnz)]))
    peak, peak_kind = hbm_peak()
    t_hbm = hbm_bytes / (peak * 1e9)
    t_nvl = nvl_bytes / (NVLINK_GBS * 1e9)
    bound = "hbm" if t_hbm >= t_nvl else "nvlink"
    achieved = (hbm_bytes if bound == "hbm" else nvl_bytes) / (ms * 1e-3) / 1e9
    pk = peak if bound == "hbm" else NVLINK_GBS
    traffic = None
    l2 = None
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tj = json.load(f)
        key = f"{w.name}:{w.dist}:G{N}"  # profiles/traffic.json: ncu --set full of this workload
        if key in tj:
            traffic = tj[key]["dram_bytes_per_launch"]
            with open(os.path.join(ROOT, "profiles", "l2_probe.json")) as f:
                l2_peak = float(json.load(f)["l2_read_peak_gbs"])
            l2_bytes = tj[key].get("l2_read_bytes_per_launch")
            if l2_bytes:
                # second roof: L2->SM read traffic of this kernel (ncu) over the measured L2
                # streaming read bandwidth (tools/l2_probe.py); binds under zipf reuse
                l2 = {"bytes": l2_bytes, "achieved": l2_bytes / (ms * 1e-3) / 1e9, "peak": l2_peak, "unit": "GB/s",
                      "frac": l2_bytes / (ms * 1e-3) / 1e9 / l2_peak,
                      "source": "ncu lts__t_sectors_srcunit_tex_op_read x 32 B (profiles/traffic.json) / "
                                "profiles/l2_probe.json"}
    except Exception:
        pass
    roof = {"bound": bound, "achieved": achieved, "peak": pk, "unit": "GB/s", "frac": achieved / pk,
            "traffic": traffic, "kernel": "emb_fwd_kernel (fused gather+pool+store+flags)",
            "algorithmic_bytes_per_launch": hbm_bytes if bound == "hbm" else nvl_bytes,
            "basis": "compulsory HBM bytes: each distinct (table,row) of the batch once (d*e) + every index (8 B) "
                     "+ every offset (8 B) + every pooled output vector written once (d*e_o); SURVEY §8(d) fraction 3",
            "lookup_counted": {"bytes": lookup_bytes, "achieved": lookup_bytes / (ms * 1e-3) / 1e9,
                               "frac": lookup_bytes / (ms * 1e-3) / 1e9 / peak,
                               "note": "every lookup's row counted (SURVEY §8(d) fraction 1); >1 under zipf "
                                       "because L1/L2 serve repeated rows"},
            "unique_rows_per_batch": float(np.mean(uniq)), "lookups_per_batch": float(np.mean(nnz)),
            "peak_source": f"{peak_kind} MEASURED_PEAKS.json hbm_gbs" if bound == "hbm" else "measured peer copy 770 GB/s (B200_PROFILING.md)",
            "t_roof_ms": max(t_hbm, t_nvl) * 1e3, "frac_of_roofline_time": max(t_hbm, t_nvl) * 1e3 / ms,
            "l2": l2}

    extra = {}
    # ---- uniform-index control (lookup bytes ~= DRAM bytes; no zipf reuse)
    if not args.no_control and w.dist == "zipf":
        wu = synth.make_workload(args.config, G=N, dist="uniform")
        with torch.cuda.stream(stream):
            ub = [SG.rank_csr(wu, wu.batch_seed(100 + i), rank, dev) for i in range(2)]
        torch.cuda.synchronize()
        for s in range(3):
            layer.forward(ub[s % 2][0], ub[s % 2][1], 0, stream)

        def fwd_u(s):
            layer.forward(ub[s % 2][0], ub[s % 2][1], 0, stream)
        ms_u = timed(fwd_u, max(args.steps // 2, 3))
        nnz_u = [int(b[0][-1].item()) for b in ub]
        hb_u, _ = algorithmic_bytes(wu, float(np.mean(nnz_u)), nbags, remote_bags)
        cb_u = float(np.mean([compulsory_bytes(wu, unique_rows(wu, rank, b), z, nbags) for b, z in zip(ub, nnz_u)]))
        extra["uniform_control"] = {"ms_per_step": ms_u, "value": w.B / (ms_u * 1e-3),
                                    "achieved_gbs": cb_u / (ms_u * 1e-3) / 1e9, "frac": cb_u / (ms_u * 1e-3) / 1e9 / peak,
                                    "lookup_counted_frac": hb_u / (ms_u * 1e-3) / 1e9 / peak,
                                    "note": "uniform indices: lookup-counted ~= compulsory ~= DRAM bytes"}
        del ub

    # ---- conventional comparison path: pool kernel -> NCCL all_to_all_single -> unpack kernel
    if not args.no_compare:
        def fwd_b(s):
            o, x = batches[s % len(batches)]
            with torch.cuda.stream(stream):
                layer.forward_baseline(o, x, None, 0, stream)
        for s in range(3):
            fwd_b(s)
        ms_b = timed(fwd_b, max(args.steps // 2, 3))
        extra["comparison_nccl_path"] = {"ms_per_step": ms_b, "value": w.B / (ms_b * 1e-3),
                                         "pgas_speedup": ms_b / ms,
                                         "note": "G=1: pool kernel only (no exchange, no unpack)" if N == 1 else
                                         f"pool kernel + {args.backend} all_to_all_single + unpack kernel"
                                         + (" (gloo: host-staged test harness, not a measurement)"
                                            if args.backend == "gloo" else "")}

    # ---- e2e through the public C ABI with host buffers
    e2e = None
    if not args.no_e2e:
        hb = []
        for o, x in batches[:2]:
            hb.append((o.cpu().pin_memory(), x.cpu().pin_memory()))
        houts = [torch.empty((B_r, w.T, w.dim), dtype=layer.out_dtype).pin_memory() for _ in range(2)]

        def fwd_h(s):
            ho, hx = hb[s % 2]
            E.emb_forward_host_async(layer.ctx, ho, hx, houts[s % 2], 0, stream)

        def drain():
            E.emb_host_drain(layer.ctx, stream)
        for s in range(2):
            fwd_h(s)
        drain()
        k_e2e = max(min(args.steps, 20), 3)
        ms_e = timed(fwd_h, k_e2e, drain)
        h2d = float(np.mean([(ho.numel() + hx.numel()) * 8 for ho, hx in hb]))
        d2h = B_r * w.T * w.dim * w.out_elem_bytes()
        e2e = {"value": w.B / (ms_e * 1e-3), "unit": "samples/s", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": ms_e, "steps": k_e2e,
               "path": "emb_forward_host_async (public C ABI): pinned H2D of offsets+indices on a copy-in stream, "
                       "fused kernel on the caller's stream, D2H of Y_r on a copy-out stream; consecutive steps "
                       "overlap; the timed region ends after emb_host_drain"}

    cpu = None
    if rank == 0 and N == 1 and not args.no_cpu_baseline:
        cpu = oracle_sample(w, 0)

    layer.close()
    if N > 1:
        dist.barrier()
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": N,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
                "scaling": "weak" if w.name.startswith("weak") else "strong", "vs_baseline": None,
                "dtype": "f32" if (w.wdtype == "f32") else "bf16", "data": "synthetic",
                "config": config_desc(w, N), "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
                "pooled_vectors_per_s": w.B * w.T / (ms * 1e-3),
                "scaling_note": "table-wise model parallelism: each GPU adds its tables AND (weak) its 16,384 samples, so "
                                "every GPU pools its tables for the whole global batch; ideal samples/s is flat in N, "
                                "pooled_vectors_per_s (samples x tables) is the quantity that ideally grows with N",
                "gpu_launches": args.steps, "clocks": clk.summary(), **extra}
        print(json.dumps(line), flush=True)
    if N > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
