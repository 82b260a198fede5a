# ncu --set full of rmat26's level-2 expansion launch (W = 64, ~1e5 entries) + reroot parity tests
TAG=${1:-m}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -p no:cacheprovider -k "wide_lockstep and K257" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/${TAG}_pytest.log
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"expand_wide" -s 1 -c 1 \
   -o gpurun_out/${TAG}_rmat26_k2 python scripts/dense_once.py rmat26 > gpurun_out/${TAG}_ncu.log 2>&1
echo ncu rc=$?
tail -2 gpurun_out/${TAG}_ncu.log
MCE_WIDE_G=32 timeout 900 python scripts/dense_once.py rmat26 > gpurun_out/${TAG}_rmat26_g32.log 2>&1; echo rmat26 g32 rc=$?
tail -1 gpurun_out/${TAG}_rmat26_g32.log
