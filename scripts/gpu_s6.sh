# kcore local-stack A/B + parity + dense800 ncu of the lockstep pass
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -q -m gpu -x -k "core_numbers or enumerate_matches or heuristic or distributed or config" -p no:cacheprovider 2>&1 | tail -2
bash scripts/gpu_ab.sh s6ab "rmat22 ba1m" "" "-DKCORE_LOCAL=0"
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"expand_lock|build_adj_block" -c 3 \
   -o gpurun_out/s6_dense800 python scripts/dense_once.py dense800 > gpurun_out/s6_ncu.log 2>&1; echo ncu rc=$?
