# round 2, call be: masked products on 256-wide pair tiles by default — GPU suite, bench lines
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2be_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2be_pytest.txt
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/r2be_bench.json 2>> gpurun_out/r2be.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2be_products.json 2>> gpurun_out/r2be.err
echo done
