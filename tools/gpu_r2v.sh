# round 2, call v (re-entry after container restore): GPU tests, default bench line, GEMM per-call times
set -x
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r2v_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2v_pytest.txt
timeout 600 python bench.py > gpurun_out/r2v_bench.json 2> gpurun_out/r2v_bench.err
timeout 600 python tools/time_gemm.py > gpurun_out/r2v_gemm.txt 2>&1
echo done
