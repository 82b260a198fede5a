# launch list (ncu gpu__time_duration per launch) of the library's kernels in one run of a config:
#   bash scripts/gpu_launches.sh <tag> <config>
# (only mce:: kernels are measured: the graph generator's torch kernels are skipped)
TAG=${1:-l}; CFG=${2:-dense800}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base mangled -k regex:"_ZN3mce" \
   --csv --log-file gpurun_out/${TAG}_launches_${CFG}.csv \
   python scripts/dense_once.py $CFG > gpurun_out/${TAG}_launches_${CFG}.log 2>&1
echo ncu rc=$?
gzip -f gpurun_out/${TAG}_launches_${CFG}.csv
