# Round-1 evidence refresh on one B200: bench lines of every workload/mode, ncu launch list +
# full captures (tools/profile.sh), compute-sanitizer.  Output under gpurun_out/r01/.
set -u
O=gpurun_out/r01; mkdir -p $O
python bench.py > $O/bench_r01.json 2> $O/bench_r01.err
python bench.py --config single > $O/bench_r01_single.json 2>/dev/null
python bench.py --config strong > $O/bench_r01_strong.json 2>/dev/null
python bench.py --config large_shard > $O/bench_r01_large_shard.json 2>/dev/null
python bench.py --shards 2 --no-cpu-baseline --no-e2e > $O/bench_r01_shards2.json 2>/dev/null
python bench.py --opt tma_store=1 --no-cpu-baseline --no-e2e > $O/bench_r01_f4_tma_store.json 2>/dev/null
python bench.py --mode backward > $O/bench_r01_backward_weak_zipf.json 2>/dev/null
python bench.py --mode backward --dist uniform > $O/bench_r01_backward_weak_uniform.json 2>/dev/null
python bench.py --mode backward --opt bwd_algo=1 > $O/bench_r01_backward_sorted_weak_zipf.json 2>/dev/null
python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_r01_reference_arm.json 2>/dev/null
bash tools/profile.sh r01
for t in memcheck racecheck synccheck; do
  compute-sanitizer --tool $t --kernel-name kns=emb python tools/sanitize.py > $O/san_$t.log 2>&1
done
python tools/profile_summary.py r01 $O/*.ncu-rep > $O/summaries.log 2>&1
mkdir -p $O/summ && cp profiles/r01/full_*.summary.json $O/summ/ 2>/dev/null
rm -f $O/*.ncu-rep
tail -3 $O/san_*.log
ls -la $O
