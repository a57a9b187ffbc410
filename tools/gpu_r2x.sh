# round 2, call x: CTA-pair GEMM with the grid sized by cudaOccupancyMaxActiveClusters
set -x
mkdir -p gpurun_out
for p in 0 1; do RDM_PAIR_LOG=1 RDM_PAIR=$p timeout 300 python tools/time_gemm.py > gpurun_out/r2x_gemm_pair$p.txt 2>&1; done
timeout 300 python -m pytest tests/test_gpu_gemm_pair.py -x -q > gpurun_out/r2x_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2x_pytest.txt
echo done
