"""bench.py contract on the GPU box: the N=1 JSON line, and the N>1 code path (torchrun,
max over ranks, IPC peer mapping) exercised with 2 ranks on one GPU over gloo."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"}


def _last_json(out):
    lines = [l for l in out.splitlines() if l.startswith("{")]
    assert lines, out[-2000:]
    return json.loads(lines[-1])


def test_bench_n1_contract():
    r = subprocess.run([sys.executable, "bench.py", "--config", "tiny", "--steps", "5", "--warmup", "3"], cwd=ROOT,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _last_json(r.stdout)
    assert KEYS <= set(d), KEYS - set(d)
    assert d["n_gpus"] == 1 and d["steps"] == 5 and d["gpu_launches"] == 5 and d["value"] > 0
    assert d["repeats"] == 5 and len(d["ms_per_step_repeats"]) == 5
    assert d["ms_per_step"] == sorted(d["ms_per_step_repeats"])[2]               # the median repeat
    assert len(d["clocks"]["per_repeat_sm_mhz"]) <= 5
    assert d["roofline"]["bound"] in ("hbm", "nvlink") and d["roofline"]["peak"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["config"]["workload"] == "tiny"


def test_bench_reference_arm():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny", "--steps", "3",
                        "--warmup", "1"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _last_json(r.stdout)
    assert d["impl"] == "reference" and d["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_two_ranks_one_gpu():
    """The driver's N > 1 line, produced by 2 ranks time-slicing one GPU (gloo harness):
    cpu_baseline present, roofline from max_r t_roof over per-rank bytes, the paper's
    compute / communication / sync+unpack breakdown of the comparison path, and a per-rank
    f1 communication timeline."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", "29561", "bench.py", "--gpus", "2", "--steps", "5", "--warmup", "3",
           "--config", "tiny", "--backend", "gloo", "--same-device", "--repeats", "3"]
    # f3 at N = 2: shards spread over both ranks, fused path and comparison path (fp32 partials)
    rs = subprocess.run(cmd[:-2] + ["--repeats", "2", "--shards", "2", "--no-cpu-baseline", "--no-e2e"], cwd=ROOT,
                        capture_output=True, text=True, timeout=900)
    assert rs.returncode == 0, rs.stderr[-3000:]
    ds = _last_json(rs.stdout)
    assert ds["config"]["row_shards_per_table"] == 2 and ds["value"] > 0
    assert ds["comparison_nccl_path"]["breakdown"]["exchange_phase_ms"] >= 0
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _last_json(r.stdout)
    assert KEYS <= set(d), KEYS - set(d)
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["global_batch"] == 32 and d["repeats"] == 3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] > 0
    roof = d["roofline"]
    assert len(roof["per_rank"]) == 2 and roof["binding_rank"] in (0, 1)
    assert abs(roof["t_roof_ms"] - max(p["t_roof_ms"] for p in roof["per_rank"])) < 1e-9
    assert abs(roof["frac"] - roof["t_roof_ms"] / d["ms_per_step"]) < 1e-9
    assert roof["nvlink"]["egress_bytes_max"] > 0
    bd = d["comparison_nccl_path"]["breakdown"]
    assert {"computation_ms", "communication_ms", "sync_unpack_ms", "exchange_phase_ms"} <= set(bd)
    tl = d["comm_timeline"]["per_rank"]
    assert len(tl) == 2 and all(t["records"] > 0 and t["remote_bytes"] > 0 for t in tl)
    assert d["e2e"]["h2d_bytes_per_step"] > 0


def test_bench_int32_and_shards_lines():
    """--index-bits 32 (C12 option) and --shards 2 (f3) produce complete lines at N = 1;
    their roofline carries no ncu traffic of the default kernel."""
    for extra in (["--index-bits", "32"], ["--shards", "2"]):
        r = subprocess.run([sys.executable, "bench.py", "--config", "tiny", "--steps", "5", "--warmup", "3",
                            "--repeats", "2", "--no-cpu-baseline", *extra], cwd=ROOT, capture_output=True, text=True,
                           timeout=600)
        assert r.returncode == 0, r.stderr[-3000:]
        d = _last_json(r.stdout)
        assert d["value"] > 0 and (d["roofline"]["traffic"] is None or extra[0] == "--index-bits")
        if extra[0] == "--index-bits":
            assert d["config"]["index_bits"] == 32 and "i32" in d["e2e"]["path"]
