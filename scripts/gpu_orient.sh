# orientation sweep: bash scripts/gpu_orient.sh <tag> "<configs>" "<orientations>"
TAG=$1; CFGS=$2; OS=$3
mkdir -p gpurun_out
for c in $CFGS; do for o in $OS; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --orientation $o > gpurun_out/${TAG}_bench_${c}_$o.log 2>&1
  python -c "
import json;l=[x for x in open('gpurun_out/${TAG}_bench_${c}_$o.log') if x.startswith('{')][-1];d=json.loads(l);p=d['details']['phases_ms'];print('$c $o', round(d['ms_per_step'],3), 'pre', round(p['preprocess_ms'],3), 'heur', round(p['heuristic_ms'],3), 'enum', round(p['host_enum_ms'],3), d['details']['omega'], d['details']['multiplicity'], d.get('verified',{}).get('ok'), 'frac', round(d['roofline']['frac'],3))" || tail -3 gpurun_out/${TAG}_bench_${c}_$o.log
done; done
