set -u
O=gpurun_out/r02d; mkdir -p $O
timeout 1200 python -m pytest tests/test_shard_gpu.py tests/test_multiproc_gpu.py tests/test_emb_gpu.py -x -q > $O/tests.log 2>&1
tail -3 $O/tests.log
bash tools/ab.sh $O/ab.txt "single weak large_shard" "exp_so/libemb_base.so exp_so/libemb_diet1.so exp_so/libemb_diet2.so" 2 zipf
# TLB / footprint probe: the weak gather over 26 tables of 11.3M rows (150 GB, like large_shard) vs 2M rows (26.6 GB)
for r in 2000000 11300000; do
  EMB_LIB=exp_so/libemb_diet2.so timeout 900 python tools/sweep.py --config weak --rows $r --dists uniform,zipf --steps 50 --gap 2 2>&1 | grep -v summary | sed "s/^/rows$r /"
done | tee $O/tlb_probe.txt
