# ncu --set full of rmat22's top kernels (one launch each)
TAG=${1:-q}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on \
   -k regex:"greedy_big_kernel|kcore_async|build_adj_block|expand_small|greedy_kernel" -c 6 \
   -o gpurun_out/${TAG}_rmat22_top python scripts/dense_once.py rmat22 > gpurun_out/${TAG}_ncu.log 2>&1
echo ncu rc=$?
tail -2 gpurun_out/${TAG}_ncu.log
