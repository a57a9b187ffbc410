# round 2, call ac: CTA pair with A split in smem + two partial accumulators (RDM_PAIR_ASMEM=1)
mkdir -p gpurun_out
RDM_PAIR_ASMEM=1 timeout 300 python -m pytest tests/test_gpu_gemm_pair.py -x -q > gpurun_out/r2ac_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ac_pytest.txt
RDM_PAIR_ASMEM=1 timeout 300 python tools/time_gemm_pair.py > gpurun_out/r2ac_pair_dbg.txt 2>&1
RDM_PAIR_ASMEM=1 RDM_PAIR=1 timeout 300 python tools/time_gemm.py > gpurun_out/r2ac_gemm.txt 2>&1
echo done
