# heuristic sweep: bash scripts/gpu_heur.sh <tag> "<configs>" "<heuristics>"
TAG=$1; CFGS=$2; HS=$3
mkdir -p gpurun_out
for c in $CFGS; do for h in $HS; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --heuristic $h > gpurun_out/${TAG}_bench_${c}_$h.log 2>&1
  python -c "
import json;l=[x for x in open('gpurun_out/${TAG}_bench_${c}_$h.log') if x.startswith('{')][-1];d=json.loads(l);p=d['details']['phases_ms'];print('$c $h', round(d['ms_per_step'],3), 'pre', round(p['preprocess_ms'],3), 'heur', round(p['heuristic_ms'],3), 'enum', round(p['host_enum_ms'],3), d['details']['omega'], d['details']['multiplicity'], d.get('verified',{}).get('ok'))" || tail -3 gpurun_out/${TAG}_bench_${c}_$h.log
done; done
