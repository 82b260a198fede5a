# full GPU tests + smoke + bench lines (rmat22 ba1m dense800 er2000) + rmat22 launch list + rmat26 bench
TAG=${1:-s10}
bash scripts/gpu_r02.sh $TAG rmat22 ba1m dense800 er2000
bash scripts/gpu_launches.sh ${TAG}l rmat22
timeout 900 python bench.py --config rmat26 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat26.log 2>&1; echo rmat26 rc=$?
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m "gpu and slow" -p no:cacheprovider > gpurun_out/${TAG}_slow.log 2>&1; echo slow rc=$?; tail -3 gpurun_out/${TAG}_slow.log
