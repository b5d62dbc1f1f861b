set -x
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_weak.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare > gpurun_out/launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o gpurun_out/prof_weak_zipf -f python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare > gpurun_out/prof_weak.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:emb_fwd_kernel -s 3 -c 1 -o gpurun_out/prof_weak_uniform -f python bench.py --dist uniform --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare > gpurun_out/prof_weaku.log 2>&1
ls -la gpurun_out
