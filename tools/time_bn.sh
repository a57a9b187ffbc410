timeout 300 python -m pytest tests/test_gpu_ops.py -q -x -k "gemm" 2>&1 | tail -1
echo "--- BN128"; timeout 300 python tools/time_gemm.py 2>&1 | grep -E "602|products"
echo "--- BN256"; RDM_BN256=1 timeout 300 python tools/time_gemm.py 2>&1 | grep -E "602|products"
