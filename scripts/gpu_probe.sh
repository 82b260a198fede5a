# usage: bash scripts/gpu_probe.sh <tag>   -- bench lines + ncu launch list + one full capture
set -x
TAG=${1:-probe}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 600 python bench.py --config ba1m --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench ba rc=$?
timeout 900 python bench.py --config rmat22 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_ba1m.csv \
  python bench.py --config ba1m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_ba1m.log 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"kcore_peel|expand_thread|greedy_kernel" -c 4 -o gpurun_out/${TAG}_full_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full_ba1m.log 2>&1; echo full rc=$?
