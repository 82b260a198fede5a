# ncu --set full of the dense800 count-pass kernel at its largest level (k = 4 of the first window), both variants
TAG=${1:-n}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
for w in 99 8; do
  MCE_SMEM_MIN_W=$w timeout 600 ncu --set full --clock-control none --import-source on -k regex:"expand_(smem|tile)" -s 3 -c 1 \
     -o gpurun_out/${TAG}_dense_w$w python scripts/dense_once.py dense800 > gpurun_out/${TAG}_ncu_w$w.log 2>&1
  echo ncu w$w rc=$?
done
