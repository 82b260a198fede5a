mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r25_build.log 2>&1
run() { echo "$1 $(env $2 timeout 120 python bench.py --config $1 --steps $3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["ms_per_step"], d["config"]["phases_ms"]["preprocess_ms"])') $2"; }
for thr in 128 256 512 1024; do for sms in 0 74; do
  run ba1m "MCE_KCORE_THREADS=$thr MCE_KCORE_SMS=$sms" 10
  run rmat22 "MCE_KCORE_THREADS=$thr MCE_KCORE_SMS=$sms" 2
done; done > gpurun_out/r25_sweep.log 2>&1
for sl in 256 1024 2048; do run ba1m "MCE_KCORE_SLEEP=$sl" 10; run rmat22 "MCE_KCORE_SLEEP=$sl" 2; done >> gpurun_out/r25_sweep.log 2>&1
timeout 600 python -m pytest tests -q -m gpu -x -k "core or enumerate_matches or distributed" > gpurun_out/r25_pytest.log 2>&1
