timeout 300 python -m pytest tests/test_gpu_ops.py -q -x -k "gemm or hub_core" 2>&1 | tail -1
echo "--- prefetch on"; timeout 300 python tools/time_gemm.py 2>&1 | grep -E "NN|core"
echo "--- prefetch off"; RDM_NO_PF=1 timeout 300 python tools/time_gemm.py 2>&1 | grep -E "NN|core"
