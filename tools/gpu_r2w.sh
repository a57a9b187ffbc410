# round 2, call w: CTA-pair (cta_group::2) GEMM — parity, per-call times pair vs single, bench
set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gemm_pair.py -x -q > gpurun_out/r2w_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2w_pytest.txt
for p in 0 1; do RDM_PAIR=$p timeout 300 python tools/time_gemm.py > gpurun_out/r2w_gemm_pair$p.txt 2>&1; done
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/r2w_bench.json 2> gpurun_out/r2w_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline --no-variants --no-e2e > gpurun_out/r2w_products.json 2>> gpurun_out/r2w_bench.err
echo done
