set -u
O=gpurun_out/r02f; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1
tail -3 $O/tests.log
bash tools/ab.sh $O/ab.txt "single" "exp_so/libemb_base.so exp_so/libemb_ur4e.so exp_so/libemb_ur8e.so" 3 zipf,uniform
bash tools/ab.sh $O/ab2.txt "weak large_shard" "exp_so/libemb_base.so exp_so/libemb_ur4e.so" 2 zipf
