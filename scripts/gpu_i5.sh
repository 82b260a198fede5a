set -x
TAG=${1:-i5}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 600 python bench.py --config rmat22 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"kcore_peel|orient_kernel|root_expand" -c 4 -o gpurun_out/${TAG}_full_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full_ba1m.log 2>&1; echo full rc=$?
