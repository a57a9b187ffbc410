# round 2, call as: (col, val) batch prefetch in the residual SpMM (A/B vs a build without it) + G=16 at w=128; SpMM tests
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_ops.py -x -q -k "spmm" > gpurun_out/r2as_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2as_pytest.txt
for i in 1 2; do
timeout 600 python tools/exp_spmm_calls.py >> gpurun_out/r2as_calls.txt 2>&1
RDM_LIB_VARIANT=nopf timeout 600 python tools/exp_spmm_calls.py >> gpurun_out/r2as_calls.txt 2>&1
done
echo done
