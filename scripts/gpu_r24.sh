mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r24_build.log 2>&1
for bps in 1 2 3 4; do for sl in 64 128 512; do
  echo "bps=$bps sleep=$sl $(MCE_KCORE_BPS=$bps MCE_KCORE_SLEEP=$sl timeout 120 python bench.py --config ba1m --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["ms_per_step"], d["config"]["phases_ms"]["preprocess_ms"])')"
  echo "rmat22 bps=$bps sleep=$sl $(MCE_KCORE_BPS=$bps MCE_KCORE_SLEEP=$sl timeout 120 python bench.py --config rmat22 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["ms_per_step"], d["config"]["phases_ms"]["preprocess_ms"])')"
done; done > gpurun_out/r24_sweep.log 2>&1
