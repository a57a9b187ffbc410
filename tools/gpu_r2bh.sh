# round 2, call bh: short-row threshold 64 for w <= 100 — SpMM/GEMM/GCN tests, epochs, papers emulation
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2bh_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bh_pytest.txt
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/r2bh_bench.json 2>> gpurun_out/r2bh.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2bh_products.json 2>> gpurun_out/r2bh.err
timeout 1500 python bench.py --emulate 8 --steps 3 --warmup 3 > gpurun_out/r2bh_papers.json 2>> gpurun_out/r2bh.err
echo done
