set -x
TAG=${1:-a9}; KREGEX=${2:-kcore_async}
bash scripts/gpu_all.sh $TAG
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$KREGEX" -c ${3:-2} -o gpurun_out/${TAG}_full_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full_ba1m.log 2>&1; echo full rc=$?
