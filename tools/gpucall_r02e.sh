set -u
O=gpurun_out/r02e; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1
tail -3 $O/tests.log
bash tools/ab.sh $O/ab.txt "single weak large_shard" "exp_so/libemb_base.so exp_so/libemb_diet1.so exp_so/libemb_diet3.so" 3 zipf
bash tools/ab_bwd.sh $O/ab_bwd.txt "exp_so/libemb_diet2.so exp_so/libemb_diet3.so" 2 "zipf uniform"
