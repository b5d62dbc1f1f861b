set -u
O=gpurun_out/r02w; mkdir -p $O
timeout 1200 python -m pytest tests/test_shard_gpu.py tests/test_emb_gpu.py tests/test_bench_gpu.py -x -q > $O/tests.log 2>&1; tail -n 3 $O/tests.log
python bench.py --shards 2 --no-cpu-baseline --no-e2e > $O/bench_shards2.json 2> $O/bench_shards2.err; tail -c 400 $O/bench_shards2.json
