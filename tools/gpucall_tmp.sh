set -u
O=gpurun_out/r02t; mkdir -p $O
EMB_LIB=exp_so/libemb_diet4.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q > $O/tests4.log 2>&1; tail -n 1 $O/tests4.log
EMB_LIB=exp_so/libemb_diet5.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q -k "pipeline or g1_bitexact or c7 or medium" > $O/tests5.log 2>&1; tail -n 1 $O/tests5.log
bash tools/ab.sh $O/ab.txt "single weak large_shard" "exp_so/libemb_head.so exp_so/libemb_diet4.so exp_so/libemb_diet5.so" 3 zipf
