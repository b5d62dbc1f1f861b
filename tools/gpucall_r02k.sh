set -u
O=gpurun_out/r02k; mkdir -p $O
timeout 1200 python -m pytest tests/test_emb_gpu.py tests/test_bwd_gpu.py tests/test_multiproc_gpu.py -x -q > $O/tests.log 2>&1; tail -n 1 $O/tests.log
bash tools/ab.sh $O/ab.txt "single weak" "exp_so/libemb_w3f.so exp_so/libemb_nofence.so" 3 zipf
bash tools/ab_bwd.sh $O/ab_bwd.txt "exp_so/libemb_w3f.so exp_so/libemb_nofence.so" 2 "zipf"
