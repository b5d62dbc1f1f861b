set -u
O=gpurun_out/r02p; mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1; tail -n 1 $O/tests.log
for L in exp_so/libemb_cur.so exp_so/libemb_unpack2.so exp_so/libemb_cur.so exp_so/libemb_unpack2.so; do
  echo "$L $(EMB_LIB=$L python tools/unpack_probe.py 2>&1 | tail -1)"
done | tee $O/unpack.txt
