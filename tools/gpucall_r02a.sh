set -u
O=gpurun_out/r02a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 120 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 tools/probe_nccl_same_gpu.py > $O/nccl_probe.log 2>&1
echo "nccl probe exit $?" >> $O/nccl_probe.log
B="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $O/full_large_shard -f $B --config large_shard > $O/full_large_shard.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $O/full_single -f $B --config single > $O/full_single.log 2>&1
timeout 600 python bench.py --config large_shard --no-cpu-baseline --no-e2e > $O/bench_large_shard.json 2> $O/bench_large_shard.err
timeout 300 python bench.py --config single --no-cpu-baseline --no-e2e > $O/bench_single.json 2> $O/bench_single.err
ls -la $O
