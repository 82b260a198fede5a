# usage: bash scripts/gpu_iter.sh <tag>  -- GPU tests + ba1m / rmat22 / er2000 bench lines + rmat24 probe
set -x
TAG=${1:-it}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_er2000.log 2>&1; echo bench er rc=$?
timeout 300 python scripts/probe_rmat26.py 24 > gpurun_out/${TAG}_probe_rmat24.log 2>&1; echo probe24 rc=$?
