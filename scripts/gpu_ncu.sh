# usage: bash scripts/gpu_ncu.sh <tag> <config> [kernel-regex]
set -x
mkdir -p gpurun_out
TAG=$1; CFG=$2; K=${3:-expand}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches.log 2>&1
echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -c 3 -o gpurun_out/${TAG}_full \
  python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full.log 2>&1
echo full rc=$?
