set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r9_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/r9_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r9_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python bench.py --config rmat22 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r9_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 1200 python scripts/probe_rmat26.py 26 > gpurun_out/r9_probe_rmat26.log 2>&1; echo probe26 rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kcore_async -c 1 -o gpurun_out/r9_full_kcore_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r9_full_kcore.log 2>&1; echo full kcore rc=$?
