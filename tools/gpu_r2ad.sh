# round 2, call ad: CTA-pair GEMM policy (auto) — all GPU tests, Reddit + products bench lines
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2ad_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ad_pytest.txt
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/r2ad_bench.json 2> gpurun_out/r2ad_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2ad_products.json 2>> gpurun_out/r2ad_bench.err
echo done
