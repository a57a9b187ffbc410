# round 2, call r: GPU tests with the folded fast-variant cast; fast-variant benches (Reddit, products)
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2r_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2r_pytest.txt
timeout 600 python bench.py --precision fast --steps 20 --warmup 5 --no-cpu-baseline --no-variants > gpurun_out/r2r_reddit_fast.json 2> gpurun_out/r2r_reddit_fast.err
timeout 900 python bench.py --workload products --precision fast --steps 10 --warmup 3 --no-cpu-baseline --no-variants > gpurun_out/r2r_products_fast.json 2> gpurun_out/r2r_products_fast.err
echo done
