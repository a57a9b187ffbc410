# round 2, call t: ReLU sign bits for GEMM Hadamards — GPU tests, products bench (bits on / off)
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2t_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2t_pytest.txt
for b in 1 0; do RDM_MASK_BITS=$b timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-variants --no-e2e >> gpurun_out/r2t_products.jsonl 2>> gpurun_out/r2t_products.err; done
echo done
