set -u
O=gpurun_out/r02g; mkdir -p $O
EMB_LIB=exp_so/libemb_g3m5.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q -k "pipeline_variants or g1_bitexact or c7" > $O/tests_g3m5.log 2>&1; tail -1 $O/tests_g3m5.log
EMB_LIB=exp_so/libemb_g3m6.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q -k "pipeline_variants or g1_bitexact" > $O/tests_g3m6.log 2>&1; tail -1 $O/tests_g3m6.log
bash tools/ab.sh $O/ab.txt "single" "exp_so/libemb_ur4e.so exp_so/libemb_g3m6.so exp_so/libemb_g3m5.so" 3 zipf,uniform
