# usage: bash scripts/gpu_r02.sh <tag> [bench configs...] -- build, all GPU tests, smoke, bench lines
set -x
TAG=${1:-a}; shift
CONFIGS=${@:-rmat22 ba1m dense800}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
tail -30 gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo smoke rc=$?
for c in $CONFIGS; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_$c.log 2>&1; echo bench $c rc=$?
  tail -c 600 gpurun_out/${TAG}_bench_$c.log
done
