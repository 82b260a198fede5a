# usage: bash scripts/gpu_rmat.sh <tag> [timeout]
set -x
TAG=${1:-rm}; RT=${2:-600}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
MCE_VERBOSE=1 timeout $RT python bench.py --config rmat22 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
