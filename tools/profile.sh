#!/bin/bash
# ncu evidence for the bench workload (run under gpurun; one GPU).  Usage: bash tools/profile.sh TAG
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
BENCH="python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare"
# launch list of the same command bench.py times (cold-cache, serialised: compare SHARES)
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"emb_|nccl" -c 200 --csv --log-file $OUT/launches_weak_zipf.csv $BENCH > $OUT/launches.log 2>&1
# one full capture of the hot kernel, zipf (headline) and uniform (control)
ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $OUT/full_weak_zipf -f $BENCH > $OUT/full_zipf.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $OUT/full_weak_uniform -f $BENCH --dist uniform > $OUT/full_uniform.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o $OUT/full_single_zipf -f $BENCH --config single > $OUT/full_single.log 2>&1
ls -la $OUT
# f2 backward (zipf)
ncu --set full --clock-control none --import-source on -k regex:emb_bwd_kernel -s 3 -c 1 -o $OUT/full_weak_zipf_backward -f $BENCH --mode backward > $OUT/full_bwd.log 2>&1
