set -u
O=gpurun_out/r02j; mkdir -p $O
for rep in 1 2 3; do
  for L in exp_so/libemb_slot2.so exp_so/libemb_slot3.so; do
    EMB_LIB=$L python tools/sweep.py --config weak --dists zipf --steps 100 --gap 2 2>/dev/null | grep -v summary | sed "s|^|$(basename $L .so) weak |"
    EMB_LIB=$L python tools/sweep.py --config weak --dists zipf --steps 100 --gap 2 --baseline 2>/dev/null | grep -v summary | sed "s|^|$(basename $L .so)_pool weak |"
  done
done | tee $O/ab.txt
