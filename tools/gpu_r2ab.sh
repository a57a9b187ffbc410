# round 2, call ab: CTA-pair GEMM with CTA-scope remote arrivals (no MEMBAR per arrival)
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_pair.py -x -q > gpurun_out/r2ab_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ab_pytest.txt
timeout 300 python tools/time_gemm_pair.py > gpurun_out/r2ab_pair_dbg.txt 2>&1
for p in 0 1; do RDM_PAIR=$p timeout 300 python tools/time_gemm.py > gpurun_out/r2ab_gemm_pair$p.txt 2>&1; done
echo done
