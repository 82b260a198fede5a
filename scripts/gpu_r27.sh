set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r27_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/r27_pytest.log 2>&1; echo pytest rc=$?
MCE_VERBOSE=1 timeout 300 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r27_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python scripts/probe_rmat26.py 24 > gpurun_out/r27_probe_rmat24.log 2>&1; echo probe24 rc=$?
