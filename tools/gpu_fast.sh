# fast-precision variant: parity tests + bench of both workloads in both precisions
timeout 900 python -m pytest tests/test_gpu_fast.py -x -q > gpurun_out/fast_tests.log 2>&1; echo fast-tests rc=$?
tail -15 gpurun_out/fast_tests.log
for W in reddit products; do
  timeout 400 python bench.py --workload $W --precision fast --no-cpu-baseline > gpurun_out/fast_bench_$W.json 2> gpurun_out/fast_bench_$W.err; echo bench $W rc=$?
  tail -3 gpurun_out/fast_bench_$W.err
  python -c "import json;d=json.load(open('gpurun_out/fast_bench_$W.json'));print(d['value'],d['phases_ms_per_step'],d.get('loss'))"
done
