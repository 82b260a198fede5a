# usage: bash scripts/gpu_root.sh <tag>  -- all GPU tests + ba1m bench line + ncu --set full of the root kernel
set -x
TAG=${1:-r}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 1200 python -m pytest tests -q -m gpu -x > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config ba1m --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:root_expand -c 1 -o gpurun_out/${TAG}_full_root_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full_root.log 2>&1; echo full root rc=$?
