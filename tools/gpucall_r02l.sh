set -u
O=gpurun_out/r02l; mkdir -p $O
EMB_LIB=exp_so/libemb_bwdb.so timeout 1200 python -m pytest tests/test_bwd_gpu.py tests/test_multiproc_gpu.py -x -q -k "bwd or backward" > $O/tests.log 2>&1; tail -n 1 $O/tests.log
bash tools/ab_bwd.sh $O/ab_bwd.txt "exp_so/libemb_nofence.so exp_so/libemb_bwdb.so" 2 "zipf uniform"
