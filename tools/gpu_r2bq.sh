# round 2, call bq: paired k-block handshakes in the tcgen05 GEMM (RDM_GEMM_HS2=1) — parity, per-call times, epochs
mkdir -p gpurun_out
RDM_GEMM_HS2=1 timeout 900 python -m pytest tests/test_gpu_ops.py tests/test_gpu_gemm_pair.py tests/test_gpu_gemm_tn_pair.py tests/test_gpu_gcn.py -x -q > gpurun_out/r2bq_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bq_pytest.txt
for h in 0 1; do RDM_GEMM_HS2=$h timeout 300 python tools/time_gemm.py > gpurun_out/r2bq_gemm_hs$h.txt 2>&1; done
for h in 0 1; do
  RDM_GEMM_HS2=$h timeout 600 python bench.py --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bq_bench_hs$h.json 2>> gpurun_out/r2bq.err
  RDM_GEMM_HS2=$h timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bq_products_hs$h.json 2>> gpurun_out/r2bq.err
done
echo done
