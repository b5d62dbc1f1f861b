set -u
O=gpurun_out/r02r; mkdir -p $O
python tools/sweep.py --config weak --dists zipf,uniform --steps 100 --gap 2 --repeat 4 --opts "" "tail_div=8" "tail_div=16" "tail_div=8,chunk_rows=160" 2>&1 | tee $O/sweep_weak.txt | grep summary
python tools/sweep.py --config single --dists zipf --steps 100 --gap 2 --repeat 4 --opts "" "tail_div=8" "tail_div=16" 2>&1 | tee $O/sweep_single.txt | grep summary
python tools/sweep.py --config large_shard --dists zipf --steps 30 --gap 2 --repeat 2 --opts "" "tail_div=8" 2>&1 | tee $O/sweep_ls.txt | grep summary
