# usage: bash scripts/gpu_variant_sweep.sh <tag> <source.cu> <config> "<EXTRA flags 1>" "<EXTRA flags 2>" ...
#   compile-time variants of one source file, GPU parity subset + bench lines of one config
TAG=$1; SRC=$2; CFG=$3; shift 3
mkdir -p gpurun_out
k=0
for ex in "$@"; do
  k=$((k+1))
  touch paper_conf_ipps_geilpo23_b200/csrc/$SRC
  make -s -C paper_conf_ipps_geilpo23_b200/csrc EXTRA="$ex" > gpurun_out/${TAG}_build_$k.log 2>&1
  timeout 600 python -m pytest tests -q -m gpu -x -k "enumerate_matches or random_small or config" > gpurun_out/${TAG}_pytest_$k.log 2>&1; echo "[$ex] pytest rc=$? $(tail -1 gpurun_out/${TAG}_pytest_$k.log)"
  for rep in 1 2; do
    timeout 300 python bench.py --config $CFG --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_${k}_$rep.log 2>&1
    python -c "
import json;l=[x for x in open('gpurun_out/${TAG}_bench_${k}_$rep.log') if x.startswith('{')][-1];d=json.loads(l);p=d['config']['phases_ms'];print('[$ex]', d['ms_per_step'], p['preprocess_ms'], p['heuristic_ms'], p['host_enum_ms'], d['config']['omega'], d['config']['multiplicity'])"
  done
done
touch paper_conf_ipps_geilpo23_b200/csrc/$SRC
make -s -C paper_conf_ipps_geilpo23_b200/csrc > /dev/null 2>&1
