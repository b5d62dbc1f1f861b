set -u
O=gpurun_out/r02h; mkdir -p $O
EMB_LIB=exp_so/libemb_w3.so timeout 900 python -m pytest tests/test_emb_gpu.py -x -q -k "pipeline_variants or g1_bitexact" > $O/tests_w3.log 2>&1; tail -n 1 $O/tests_w3.log
bash tools/ab.sh $O/ab.txt "weak large_shard" "exp_so/libemb_ur4e.so exp_so/libemb_w3.so" 3 zipf
