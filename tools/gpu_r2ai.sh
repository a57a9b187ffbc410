# round 2, call ai: 128-byte tf32 panel rows (RDM_PANEL_PAD) A/B; all GPU tests; bench lines fp32 + fast
mkdir -p gpurun_out
for pp in 0 1; do RDM_PANEL_PAD=$pp timeout 300 python tools/time_gemm.py > gpurun_out/r2ai_gemm_pad$pp.txt 2>&1; done
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2ai_pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/r2ai_pytest.txt
timeout 600 python bench.py > gpurun_out/r2ai_bench.json 2> gpurun_out/r2ai_bench.err
timeout 900 python bench.py --workload products --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2ai_products.json 2>> gpurun_out/r2ai_bench.err
echo done
