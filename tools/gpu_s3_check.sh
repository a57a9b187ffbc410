timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s3b_gputests.log 2>&1; echo tests rc=$?; tail -3 gpurun_out/s3b_gputests.log
timeout 400 python bench.py > gpurun_out/s3b_bench_reddit.json 2> gpurun_out/s3b_bench_reddit.err; echo bench rc=$?
timeout 400 python bench.py --workload products --no-cpu-baseline > gpurun_out/s3b_bench_products.json 2> gpurun_out/s3b_bench_products.err; echo bench rc=$?
for W in reddit products; do python -c "import json;d=json.load(open('gpurun_out/s3b_bench_$W.json'));print('$W', d['value'], d['e2e']['value'], d['phases_ms_per_step'], d['variants'])"; done
