# usage: bash scripts/gpu_rootsweep.sh <tag> "<EXTRA flags 1>" "<EXTRA flags 2>" ...
#   root-level build variants (compile-time macros of roots.cu) timed on ba1m
TAG=$1; shift
mkdir -p gpurun_out
k=0
for ex in "$@"; do
  k=$((k+1))
  touch paper_conf_ipps_geilpo23_b200/csrc/roots.cu
  make -s -C paper_conf_ipps_geilpo23_b200/csrc EXTRA="$ex" > gpurun_out/${TAG}_build_$k.log 2>&1
  timeout 600 python -m pytest tests -q -m gpu -x -k "enumerate_matches or random_small or config" > gpurun_out/${TAG}_pytest_$k.log 2>&1; echo "[$ex] pytest rc=$?"
  for rep in 1 2; do
    timeout 300 python bench.py --config ba1m --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_${k}_$rep.log 2>&1
    python -c "
import json;l=[x for x in open('gpurun_out/${TAG}_bench_${k}_$rep.log') if x.startswith('{')][-1];d=json.loads(l);print('[$ex]', d['ms_per_step'],d['roofline']['frac'],d['config']['phases_ms']['root_kernel_ms'])"
  done
done
touch paper_conf_ipps_geilpo23_b200/csrc/roots.cu
make -s -C paper_conf_ipps_geilpo23_b200/csrc > /dev/null 2>&1
