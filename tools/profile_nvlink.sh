#!/bin/bash
# NVLink evidence for the N > 1 forward (SURVEY §8(d) "NVLink egress GB/s vs ~900 GB/s"),
# for a multi-GPU box: run under gpurun/torchrun on N GPUs.  Usage: bash tools/profile_nvlink.sh N [OUT]
#
# The guide's rule "never wrap a multi-rank command in ncu" is kept: ncu wraps ONE rank
# (rank 0) of the torchrun job, collecting only metrics that fit a single pass (no kernel
# replay -- a replayed PGAS kernel would wait for peers that do not replay), so the other
# ranks run unprofiled.  Metric names were verified offline with
#   ncu --query-metrics --chip gb100 | grep -E '^nvl(tx|rx)__'   (profiles/nvlink_metrics_gb100.txt)
# nvltx__bytes_data_user = payload this GPU sent over NVLink, nvlrx__* = received;
# per launch / gpu__time_duration.sum = achieved NVLink GB/s of the fused kernel.
N=${1:-2}
OUT=${2:-gpurun_out/nvlink}
mkdir -p $OUT
METRICS=gpu__time_duration.sum,nvltx__bytes.sum,nvltx__bytes_data_user.sum,nvlrx__bytes.sum,nvlrx__bytes_data_user.sum
BENCH="bench.py --gpus $N --steps 20 --warmup 3 --repeats 1 --no-cpu-baseline --no-e2e --no-control --no-trace"
python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 29571 \
  --no-python bash -c "
    if [ \$RANK = 0 ]; then
      ncu --metrics $METRICS --replay-mode application --app-replay-match grid --clock-control none \
          -k regex:'emb_fwd_kernel|emb_unpack|nccl' -c 60 --csv --log-file $OUT/nvlink_rank0.csv python $BENCH
    else
      python $BENCH
    fi" > $OUT/bench_nvlink.log 2>&1
tail -3 $OUT/bench_nvlink.log
python - "$OUT/nvlink_rank0.csv" <<'PY'
import csv, sys, collections
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]; k = hdr.index("Kernel Name"); m = hdr.index("Metric Name"); v = hdr.index("Metric Value")
agg = collections.defaultdict(lambda: collections.defaultdict(list))
for r in rows[1:]:
    agg[r[k][:60]][r[m]].append(float(r[v].replace(",", "")))
for kern, d in agg.items():
    t = sum(d["gpu__time_duration.sum"]) / max(len(d["gpu__time_duration.sum"]), 1)
    tx = sum(d["nvltx__bytes_data_user.sum"]) / max(len(d["nvltx__bytes_data_user.sum"]), 1)
    print(f"{kern}: {t:.0f} ns/launch, NVLink tx user {tx/1e6:.1f} MB/launch = {tx / t:.1f} GB/s")
PY
