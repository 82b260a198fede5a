# wide count pass: parity tests + rmat26 one run per tile width
TAG=${1:-w}; shift
GS=${@:-16 8}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -p no:cacheprovider -k "wide or reroot or smem" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/${TAG}_pytest.log
for g in $GS; do
  MCE_WIDE_G=$g timeout 900 python scripts/dense_once.py rmat26 > gpurun_out/${TAG}_rmat26_g$g.log 2>&1; echo rmat26 g$g rc=$?
  tail -1 gpurun_out/${TAG}_rmat26_g$g.log
done
