# GPU test suite + one default bench line (under gpurun).  Usage: bash tools/gpucall_tests.sh TAG
set -u
TAG=${1:-r02}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $O/gpu_tests.log 2>&1
echo "pytest rc $?" >> $O/gpu_tests.log
tail -5 $O/gpu_tests.log
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
tail -c 600 $O/bench.json
