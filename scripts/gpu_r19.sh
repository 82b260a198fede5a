set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r19_build.log 2>&1; echo build rc=$?
timeout 1500 python bench.py --config rmat26 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r19_bench_rmat26.log 2>&1; echo bench rmat26 rc=$?
