set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
timeout 600 python bench.py --config er2000 --steps 5 --warmup 3 > gpurun_out/bench_er2000.log 2>&1; echo bench er rc=$?
timeout 900 python bench.py --config ba1m --steps 5 --warmup 3 > gpurun_out/bench_ba1m.log 2>&1; echo bench ba rc=$?
