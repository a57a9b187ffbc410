# round 2, call y: decoupled TMEM-A ring (smem ring deeper than the TMEM ring), pair vs single
set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_pair.py tests/test_gpu_ops.py -k "gemm" -x -q > gpurun_out/r2y_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2y_pytest.txt
for p in 0 1; do RDM_PAIR=$p timeout 300 python tools/time_gemm.py > gpurun_out/r2y_gemm_pair$p.txt 2>&1; done
echo done
