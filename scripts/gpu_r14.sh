set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r14_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/r14_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config rmat22 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r14_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config dense800 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r14_bench_dense800.log 2>&1; echo bench dense rc=$?
MCE_VERBOSE=1 timeout 300 python bench.py --config dense800 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r14_dense_verbose.log 2>&1; echo dv rc=$?
