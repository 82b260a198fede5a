set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r16_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu -x -k "heuristic or smoke or config or enumerate_matches" > gpurun_out/r16_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python bench.py --config rmat22 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r16_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 300 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r16_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 300 python scripts/probe_rmat26.py 24 > gpurun_out/r16_probe_rmat24.log 2>&1; echo probe24 rc=$?
