# session 3 batch: smem W=4 A/B, colour spin A/B, dense800 window sweep
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB_REPS=3 timeout 600 python scripts/ab_env.py rmat22 "" MCE_SMEM_MIN_W=4 MCE_SMEM_MIN_W=4,MCE_SMEM_KIND=thr 2>&1 | grep rep
AB_REPS=3 timeout 600 python scripts/ab_env.py dense800 "" MCE_ROOT_COLOUR_MIN_S=1 MCE_SMEM_MIN_W=4 2>&1 | grep rep
timeout 600 python scripts/window_sweep.py --reps 3 --windows 8,16,32,48,64,96,128 > gpurun_out/s5_window_sweep.json 2> gpurun_out/s5_window_sweep.err; tail -c 1500 gpurun_out/s5_window_sweep.json
bash scripts/gpu_ab.sh s5ab "rmat22" "" "-DCOL_SPIN=16" "-DCOL_SPIN=100000000"
