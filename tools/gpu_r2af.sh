# round 2, call af: fast variant kind::f16 GEMM — parity, per-call times vs 1xTF32, fast bench lines
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_f16.py -x -q > gpurun_out/r2af_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2af_pytest.txt
timeout 600 python -m pytest tests/test_gpu_fast.py -x -q >> gpurun_out/r2af_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2af_pytest.txt
for f in 0 1; do RDM_F16_GEMM=$f RDM_PREC=fast timeout 300 python tools/time_gemm.py > gpurun_out/r2af_gemm_f16_$f.txt 2>&1; done
for f in 0 1; do RDM_F16_GEMM=$f timeout 600 python bench.py --precision fast --no-cpu-baseline --no-variants --no-e2e > gpurun_out/r2af_reddit_fast_$f.json 2>> gpurun_out/r2af.err; done
for f in 0 1; do RDM_F16_GEMM=$f timeout 900 python bench.py --workload products --precision fast --steps 10 --warmup 3 --no-cpu-baseline --no-variants --no-e2e > gpurun_out/r2af_products_fast_$f.json 2>> gpurun_out/r2af.err; done
echo done
