# round 2, session 3: tests + smoke + bench lines + rmat22 launch list
TAG=${1:-s3}
bash scripts/gpu_r02.sh $TAG rmat22 ba1m dense800
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_rmat22.csv \
   python scripts/dense_once.py rmat22 > gpurun_out/${TAG}_launches_rmat22.log 2>&1
echo ncu rc=$?
gzip -f gpurun_out/${TAG}_launches_rmat22.csv
