# usage: bash scripts/gpu_ab.sh <tag> "<configs>" "<EXTRA flags 1>" "<EXTRA flags 2>" ...
#   compile-time variants (all sources rebuilt with EXTRA), bench lines of each config per variant
TAG=$1; CFGS=$2; shift 2
mkdir -p gpurun_out
k=0
for ex in "$@"; do
  k=$((k+1))
  make -s -C paper_conf_ipps_geilpo23_b200/csrc clean > /dev/null
  make -s -j16 -C paper_conf_ipps_geilpo23_b200/csrc EXTRA="$ex" > gpurun_out/${TAG}_build_$k.log 2>&1 || { echo "[$ex] build failed"; continue; }
  for c in $CFGS; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_${k}_$c.log 2>&1
    python -c "
import json;l=[x for x in open('gpurun_out/${TAG}_bench_${k}_$c.log') if x.startswith('{')][-1];d=json.loads(l);p=d['details']['phases_ms'];print('[$ex] $c', d['details'].get('heuristic'), round(d['ms_per_step'],3), 'pre', round(p['preprocess_ms'],3), 'heur', round(p['heuristic_ms'],3), 'enum', round(p['host_enum_ms'],3), 'rootk', round(d['roofline'].get('kernel_ms_per_step') or 0,4), 'frac', round(d['roofline']['frac'],3), d['details']['omega'], d['details']['multiplicity'], d.get('verified',{}).get('ok'))" || tail -5 gpurun_out/${TAG}_bench_${k}_$c.log
  done
done
make -s -C paper_conf_ipps_geilpo23_b200/csrc clean > /dev/null
make -s -j16 -C paper_conf_ipps_geilpo23_b200/csrc > /dev/null 2>&1
