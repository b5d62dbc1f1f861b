set -u
O=gpurun_out/r02u; mkdir -p $O
EMB_LIB=exp_so/libemb_s8.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q -k "pipeline or g1_bitexact" > $O/tests.log 2>&1; tail -n 1 $O/tests.log
bash tools/ab.sh $O/ab.txt "single" "exp_so/libemb_diet4b.so exp_so/libemb_s8.so" 4 zipf,uniform
