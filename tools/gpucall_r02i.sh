set -u
O=gpurun_out/r02i; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1; tail -n 2 $O/tests.log
bash tools/ab.sh $O/ab.txt "weak strong" "exp_so/libemb_ur4e.so exp_so/libemb_w3f.so" 3 zipf,uniform
