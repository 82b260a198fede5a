set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r23_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/r23_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r23_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r23_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config dense800 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r23_bench_dense800.log 2>&1; echo bench dense rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r23_launches_ba1m.csv \
  python bench.py --config ba1m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r23_launches_ba1m.log 2>&1; echo launches ba rc=$?
