set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r15_build.log 2>&1; echo build rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:greedy -c 2 -o gpurun_out/r15_full_greedy_rmat22 \
  python bench.py --config rmat22 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r15_full_greedy.log 2>&1; echo full greedy rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:root_expand -c 1 -o gpurun_out/r15_full_root_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r15_full_root.log 2>&1; echo full root rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:expand_thread --launch-skip 30 -c 2 -o gpurun_out/r15_full_expand_rmat22 \
  python bench.py --config rmat22 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r15_full_expand.log 2>&1; echo full expand rc=$?
