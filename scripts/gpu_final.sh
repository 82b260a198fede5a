# usage: bash scripts/gpu_final.sh <tag> -- all GPU tests, smoke, bench lines of ba1m (default), rmat22, dense800, er2000
set -x
TAG=${1:-f}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo smoke rc=$?
timeout 300 python bench.py > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench default rc=$?
timeout 600 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config dense800 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_dense800.log 2>&1; echo bench dense rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_er2000.log 2>&1; echo bench er rc=$?
