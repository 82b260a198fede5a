# usage: bash scripts/gpu_headline.sh <tag> -- smoke, the default bench line (ba1m, e2e + CPU baseline),
# the reference arm, er2000, the ba1m ncu launch list
set -x
TAG=${1:-h}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo smoke rc=$?
timeout 300 python bench.py > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench default rc=$?
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_ref.log 2>&1; echo bench ref rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_er2000.log 2>&1; echo bench er rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_ba1m.csv \
  python bench.py --config ba1m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_ba1m.log 2>&1; echo launches ba rc=$?
