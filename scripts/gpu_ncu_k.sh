# ncu --set full of chosen kernels of one config: bash scripts/gpu_ncu_k.sh <tag> <config> "<kernel regex>" <count> [EXTRA]
TAG=$1; CFG=$2; RX=$3; CNT=${4:-4}; EX=${5:-}
mkdir -p gpurun_out
if [ -n "$EX" ]; then make -s -C paper_conf_ipps_geilpo23_b200/csrc clean >/dev/null; make -s -j16 -C paper_conf_ipps_geilpo23_b200/csrc EXTRA="$EX" > gpurun_out/${TAG}_build.log 2>&1;
else python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; fi
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"$RX" -c $CNT \
   -o gpurun_out/${TAG}_${CFG} python scripts/dense_once.py $CFG > gpurun_out/${TAG}_ncu.log 2>&1
echo ncu rc=$?
tail -2 gpurun_out/${TAG}_ncu.log
