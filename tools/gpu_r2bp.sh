# round 2, call bp: double-buffered TMA-store boxes for the 8-epilogue-warp GEMMs — tests, per-call times, epochs
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gemm_pair.py tests/test_gpu_gemm_f16.py tests/test_gpu_fast.py tests/test_gpu_gcn.py -x -q > gpurun_out/r2bp_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bp_pytest.txt
timeout 300 python tools/time_gemm.py > gpurun_out/r2bp_gemm.txt 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2bp_bench.json 2>> gpurun_out/r2bp.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2bp_products.json 2>> gpurun_out/r2bp.err
echo done
