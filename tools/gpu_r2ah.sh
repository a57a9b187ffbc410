# round 2, call ah: kind::f16 GEMM with 128-byte bf16 panel rows; per-K timing
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_f16.py -x -q > gpurun_out/r2ah_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ah_pytest.txt
timeout 300 python tools/time_gemm_f16.py > gpurun_out/r2ah_f16_k.txt 2>&1
echo done
