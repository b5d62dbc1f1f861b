# A/B of libemb builds on the f2 backward (bench.py --mode backward).  Usage:
#   bash tools/ab_bwd.sh OUT "exp_so/libemb_a.so exp_so/libemb_b.so" [reps] [dists] [extra bench args]
OUT=$1; LIBS=$2; REPS=${3:-2}; DISTS=${4:-"zipf uniform"}; EXTRA=${5:-}
mkdir -p $(dirname $OUT)
for d in $DISTS; do
  for rep in $(seq $REPS); do
    for L in $LIBS; do
      sleep 2
      EMB_LIB=$L timeout 900 python bench.py --mode backward --dist $d --steps 30 --warmup 3 --repeats 3 \
        --no-cpu-baseline --no-e2e --no-control --no-compare $EXTRA 2>/dev/null | tail -1 | \
        python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $L .so) $d', round(d['ms_per_step'],4), round(d['roofline']['frac'],3), d['clocks']['per_repeat_sm_mhz'])"
    done
  done
done | tee $OUT
