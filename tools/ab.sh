# A/B of libemb builds on one B200 (run under gpurun).  Usage:
#   bash tools/ab.sh OUT "cfg1 cfg2" "exp_so/libemb_a.so exp_so/libemb_b.so" [reps] [dists]
# interleaves the builds (ABAB...) with idle gaps so clock/thermal drift hits both alike.
OUT=$1; CFGS=$2; LIBS=$3; REPS=${4:-3}; DISTS=${5:-zipf,uniform}
mkdir -p $(dirname $OUT)
for cfg in $CFGS; do
  for rep in $(seq $REPS); do
    for L in $LIBS; do
      EMB_LIB=$L timeout 900 python tools/sweep.py --config $cfg --dists $DISTS --steps 100 --gap 2 2>/dev/null \
        | grep -v summary | sed "s|^|$(basename $L .so) $cfg |"
    done
  done
done | tee $OUT
