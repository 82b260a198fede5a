# large-config checks: golden tests (slow), rmat26 one run with per-level log
TAG=${1:-b}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m "gpu and slow" -p no:cacheprovider > gpurun_out/${TAG}_slow.log 2>&1; echo slow rc=$?
tail -3 gpurun_out/${TAG}_slow.log
MCE_VERBOSE=1 timeout 1200 python scripts/dense_once.py rmat26 > gpurun_out/${TAG}_rmat26.log 2>&1; echo rmat26 rc=$?
tail -2 gpurun_out/${TAG}_rmat26.log
