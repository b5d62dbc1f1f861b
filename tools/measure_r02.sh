#!/bin/bash
# Round-2 evidence on one B200 (run under gpurun): every bench line, the ncu launch list of
# the default bench command, full ncu captures of the hot kernels, compute-sanitizer.
# Output under gpurun_out/r02m/ (summaries are copied to profiles/r02/ afterwards).
set -u
O=${OUT:-gpurun_out/r02m}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/smi.txt 2>&1
B="python bench.py"
$B > $O/bench_r02.json 2> $O/bench_r02.err
sleep 5; $B --index-bits 32 --no-cpu-baseline > $O/bench_r02_int32.json 2>/dev/null
sleep 5; $B --config single > $O/bench_r02_single.json 2>/dev/null
sleep 5; $B --config strong --no-e2e > $O/bench_r02_strong.json 2>/dev/null
sleep 5; $B --config large_shard --no-e2e > $O/bench_r02_large_shard.json 2>/dev/null
sleep 5; $B --config weak_paper --no-cpu-baseline --no-e2e > $O/bench_r02_weak_paper.json 2>/dev/null
sleep 5; $B --shards 2 --no-cpu-baseline --no-e2e > $O/bench_r02_shards2.json 2>/dev/null
sleep 5; $B --opt tma_store=1 --no-cpu-baseline --no-e2e > $O/bench_r02_f4_tma_store.json 2>/dev/null
sleep 5; $B --mode backward > $O/bench_r02_backward_weak_zipf.json 2>/dev/null
sleep 5; $B --mode backward --dist uniform > $O/bench_r02_backward_weak_uniform.json 2>/dev/null
sleep 5; $B --mode backward --opt bwd_algo=1 > $O/bench_r02_backward_sorted_weak_zipf.json 2>/dev/null
$B --impl reference --steps 3 --warmup 1 > $O/bench_r02_reference_arm.json 2>/dev/null
python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29581 \
  bench.py --gpus 2 --config weak --backend gloo --same-device --steps 20 --warmup 3 --repeats 3 \
  > $O/bench_harness_g2_same_device_gloo.json 2> $O/harness.err
# ncu: launch list of the default bench command (cold-cache, serialised: compare SHARES)
NB="python bench.py --steps 10 --warmup 3 --repeats 1 --no-cpu-baseline --no-e2e --no-control --no-compare --no-trace"
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"emb_|nccl" -c 200 --csv \
    --log-file $O/launches_weak_zipf.csv $NB > $O/launches.log 2>&1
for spec in "weak_zipf:" "weak_uniform:--dist uniform" "single_zipf:--config single" "large_shard_zipf:--config large_shard" "weak_zipf_int32:--index-bits 32"; do
  name=${spec%%:*}; args=${spec#*:}
  ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $O/full_$name -f \
      $NB $args > $O/full_$name.log 2>&1
done
ncu --set full --clock-control none --import-source on -k regex:emb_bwd_kernel -s 3 -c 1 -o $O/full_weak_zipf_backward -f \
    $NB --mode backward > $O/full_bwd.log 2>&1
python tools/pcie_bw.py > $O/pcie_bw.txt 2>&1
python tools/unpack_probe.py > $O/unpack_probe.txt 2>&1
# compute-sanitizer is closed on this GPU pool (runs under it left GPUs needing a reset);
# profiles/r02/sanitizers.txt is from the first r02 measurement run of the same kernels.
for t in; do
  compute-sanitizer --tool $t --kernel-name kns=emb python tools/sanitize.py > $O/san_$t.log 2>&1
done
python tools/profile_summary.py r02 $O/*.ncu-rep > $O/summaries.log 2>&1
mkdir -p $O/summ && cp profiles/r02/full_*.summary.json $O/summ/ 2>/dev/null
rm -f $O/*.ncu-rep
true
ls -la $O
