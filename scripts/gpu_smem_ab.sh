# usage: bash scripts/gpu_smem_ab.sh <tag> -- build, smem parity tests, dense800 / rmat22 A/B of the shared-memory count pass
TAG=${1:-s}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1; echo build rc=$?
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_distributed.py -q -m gpu -x -p no:cacheprovider -k "smem or enumerate_matches or completions or overflow or chunking or reroot or different_bounds or shards" > gpurun_out/${TAG}_pytest.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/${TAG}_pytest.log
for w in 99 8 4 16; do
  K=thr; case $w in tile*) K=tile; w=${w#tile};; esac
  MCE_SMEM_KIND=$K MCE_SMEM_MIN_W=$w timeout 300 python bench.py --config dense800 --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_dense_w$w.log 2>&1
  python - "$w" gpurun_out/${TAG}_dense_w$w.log <<'PY'
import json,sys,os
l=[x for x in open(sys.argv[2]) if x.startswith('{')]
if l:
    d=json.loads(l[-1]); print("dense800 minw", sys.argv[1], os.environ.get("MCE_SMEM_KIND"), "ms", round(d["ms_per_step"],2), "count_ms", round(d["details"]["phases_ms"]["expand_count_ms"],2), d["verified"]["ok"])
else: print("dense800 minw", sys.argv[1], "FAILED"); print(open(sys.argv[2]).read()[-2000:])
PY
done
for w in 99 4; do
  MCE_SMEM_MIN_W=$w timeout 300 python bench.py --config rmat22 --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_rmat22_w$w.log 2>&1
  python - "$w" gpurun_out/${TAG}_rmat22_w$w.log <<'PY'
import json,sys
l=[x for x in open(sys.argv[2]) if x.startswith('{')]
if l:
    d=json.loads(l[-1]); p=d["details"]["phases_ms"]; print("rmat22 minw", sys.argv[1], "ms", round(d["ms_per_step"],2), "expand", round(p["expand_ms"],2), "host_enum", round(p["host_enum_ms"],2), "levels", len(d["details"]["levels"]), d["details"]["omega"], d["details"]["multiplicity"])
else: print("rmat22 minw", sys.argv[1], "FAILED"); print(open(sys.argv[2]).read()[-2000:])
PY
done
MCE_VERBOSE=1 timeout 120 python -c "
import sys; sys.path.insert(0,'.')
import paper_conf_ipps_geilpo23_b200 as m
from synth import graphs as G
g=G.make_config('dense800'); gg=m.Graph(g.rowptr.cuda(), g.col.cuda())
r=gg.find_one(window=64); print(r.omega)
g=G.make_config('rmat22', device='cuda'); gg=m.Graph(g.rowptr, g.col)
r=gg.enumerate(max_cliques=1<<16); print(r.omega, r.count)
" > gpurun_out/${TAG}_verbose.log 2>&1; echo verbose rc=$?
grep -c level gpurun_out/${TAG}_verbose.log
if [ -n "$RMAT26" ]; then
  MCE_VERBOSE=1 timeout 900 python scripts/dense_once.py rmat26 > gpurun_out/${TAG}_rmat26.log 2>&1; echo rmat26 rc=$?
  tail -1 gpurun_out/${TAG}_rmat26.log
fi
