# usage: bash tools/bwd_sweep.sh "opt=v,opt=v" "opt=v" ...   (backward A/B, zipf + uniform)
mkdir -p gpurun_out/s3
python -m pytest tests/test_bwd_gpu.py -x -q > gpurun_out/s3/bwd_tests.log 2>&1; tail -2 gpurun_out/s3/bwd_tests.log
for d in zipf uniform; do
for rep in 1 2; do
for o in "$@"; do
  sleep 2
  args=""; for kv in ${o//,/ }; do args="$args --opt $kv"; done
  python bench.py --mode backward --dist $d --steps 30 --warmup 3 --no-cpu-baseline --no-e2e --no-control --no-compare $args 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$d $o', round(d['ms_per_step'],3), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done; done; done 2>&1 | tee gpurun_out/s3/bwd_sweep.txt
