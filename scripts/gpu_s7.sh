python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests -q -m gpu -x -k "core_numbers or enumerate_matches" -p no:cacheprovider 2>&1 | tail -1
bash scripts/gpu_ab.sh s7ab "rmat22 ba1m" "" "-DKCORE_LOCAL=0" "-DKCORE_LOCAL_BATCHES=1"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"expand_lock" -c 14 \
   -o gpurun_out/s7_dense800 python scripts/dense_once.py dense800 > gpurun_out/s7_ncu.log 2>&1; echo ncu rc=$?
timeout 900 python scripts/ab_env.py rmat26 "" 2>&1 | grep rep
