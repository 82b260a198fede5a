# usage: bash scripts/gpu_evidence.sh <tag> -- the round's evidence set: GPU tests, smoke, every
# single-GPU bench line (+ reference arm), the dense800 window sweep, launch lists, ncu --set full of
# the headline expansion kernel
set -x
TAG=${1:-ev}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo smoke rc=$?
timeout 300 python bench.py > gpurun_out/${TAG}_bench_ba1m.log 2>&1; echo bench default rc=$?
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_ref.log 2>&1; echo bench ref rc=$?
timeout 300 python bench.py --config er2000 --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_er2000.log 2>&1; echo bench er rc=$?
timeout 300 python bench.py --config dense800 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_dense800.log 2>&1; echo bench dense rc=$?
timeout 600 python bench.py --config rmat22 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_rmat22.log 2>&1; echo bench rmat22 rc=$?
timeout 600 python scripts/window_sweep.py > gpurun_out/${TAG}_window_sweep.json 2> gpurun_out/${TAG}_window_sweep.log; echo sweep rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_ba1m.csv \
  python bench.py --config ba1m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_ba1m.log 2>&1; echo launches ba rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_rmat22.csv \
  python bench.py --config rmat22 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_launches_rmat22.log 2>&1; echo launches rmat rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:root_expand -c 1 -o gpurun_out/${TAG}_full_root_ba1m \
  python bench.py --config ba1m --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_full_root.log 2>&1; echo full root rc=$?
timeout 1500 python bench.py --config rmat26 --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_rmat26.log 2>&1; echo bench rmat26 rc=$?
