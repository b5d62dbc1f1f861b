# A/B of the default library vs an experiment build: bash tools/ab.sh exp/libemb_X.so config dists
mkdir -p gpurun_out/s3
X=$1; C=$2; D=$3
for rep in 1 2 3; do
  python tools/sweep.py --config $C --dists $D --steps 60 --gap 2 | grep -v summary | sed "s/^/new /"
  EMB_LIB=paper_conf_sc_chenbyo24_b200/$X python tools/sweep.py --config $C --dists $D --steps 60 --gap 2 | grep -v summary | sed "s/^/old /"
done
