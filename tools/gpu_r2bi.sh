# round 2, call bi: weight-gradient (TN) GEMM on CTA pairs — parity, per-call times, epochs
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_gemm_tn_pair.py tests/test_gpu_ops.py -k "tn or gemm" -x -q > gpurun_out/r2bi_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2bi_pytest.txt
for p in 0 1; do RDM_TN_PAIR=$p timeout 300 python tools/time_gemm.py > gpurun_out/r2bi_gemm_tn$p.txt 2>&1; done
for p in 0 1; do
  timeout 600 env RDM_TN_PAIR=$p python bench.py --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bi_bench_tn$p.json 2>> gpurun_out/r2bi.err
  timeout 900 env RDM_TN_PAIR=$p python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --no-variants > gpurun_out/r2bi_products_tn$p.json 2>> gpurun_out/r2bi.err
done
echo done
