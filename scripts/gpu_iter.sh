# usage: bash scripts/gpu_iter.sh <tag> [rmat22_timeout]  -- tests, bench lines, launch lists
set -x
TAG=${1:-it}; RT=${2:-300}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_er2000.log 2>&1; echo bench er rc=$?
MCE_VERBOSE=1 timeout $RT python bench.py --config rmat22 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config dense800 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_dense800.log 2>&1; echo bench dense rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_ba1m.csv \
  python bench.py --config ba1m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_ba1m.log 2>&1; echo launches rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_rmat22.csv \
  python bench.py --config rmat22 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_rmat22.log 2>&1; echo launches rmat rc=$?
