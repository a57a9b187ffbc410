# round 2, call ag: kind::f16 GEMM partial-accumulator fix; fast tests; per-K timing vs 1xTF32
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_f16.py -x -q > gpurun_out/r2ag_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ag_pytest.txt
timeout 600 python -m pytest tests/test_gpu_fast.py -x -q >> gpurun_out/r2ag_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ag_pytest.txt
timeout 300 python tools/time_gemm_f16.py > gpurun_out/r2ag_f16_k.txt 2>&1
echo done
