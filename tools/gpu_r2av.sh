# round 2, call av: G=16 residual mapping actually active for the 119 MB Reddit slice; pair threshold 148*256 rows; saint + Reddit bench
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gemm_pair.py -x -q > gpurun_out/r2av_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2av_pytest.txt
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2av_bench.json 2>> gpurun_out/r2av.err
for i in 1 2; do timeout 600 python bench.py --saint --no-cpu-baseline > gpurun_out/r2av_saint.$i.json 2>> gpurun_out/r2av.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:spmm_kernel -c 8 --csv --log-file gpurun_out/r2av_spmm_launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-variants --no-cpu-baseline > /dev/null 2>&1
echo done
