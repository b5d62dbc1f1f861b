set -u
O=gpurun_out/r02n; mkdir -p $O
timeout 1200 python -m pytest tests/test_bwd_gpu.py -x -q > $O/tests.log 2>&1; tail -n 3 $O/tests.log
for d in zipf uniform; do for rep in 1 2; do for b in 0 2 4; do
  sleep 2
  python bench.py --mode backward --dist $d --steps 30 --warmup 3 --repeats 3 --no-cpu-baseline --no-e2e --no-control --no-compare --opt bwd_bulk=$b 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bulk$b $d', round(d['ms_per_step'],4), round(d['roofline']['frac'],3), d['clocks']['per_repeat_sm_mhz'])"
done; done; done | tee $O/ab_bwd.txt
M=gpu__time_duration.sum,l1tex__t_requests_pipe_lsu_mem_global_op_red.sum,lts__t_requests_op_red.sum,lts__t_sectors_op_red.sum,lts__d_atomic_input_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_red_lookup_miss.sum
for b in 0 2; do
ncu --metrics $M --clock-control none -k regex:emb_bwd_kernel -s 3 -c 1 --csv --log-file $O/bwd_red_bulk$b.csv python bench.py --mode backward --steps 5 --warmup 3 --repeats 1 --no-cpu-baseline --no-e2e --no-control --no-compare --opt bwd_bulk=$b > /dev/null 2>&1
done
