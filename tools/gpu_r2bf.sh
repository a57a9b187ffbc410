# round 2, call bf: short-row SpMM with the row's (col, val) loaded up front — A/B vs the previous build, tests, epochs
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_ops.py -x -q -k "spmm" > gpurun_out/r2bf_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bf_pytest.txt
timeout 1200 python tools/exp_short_ab.py > gpurun_out/r2bf_ab.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bf_bench.json 2>> gpurun_out/r2bf.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bf_products.json 2>> gpurun_out/r2bf.err
echo done
