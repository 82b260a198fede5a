set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r18_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/r18_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r18_smoke.log 2>&1; echo smoke rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r18_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r18_bench_er2000.log 2>&1; echo bench er rc=$?
