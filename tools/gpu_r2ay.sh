# round 2, call ay: tcgen05 GEMM timeline of CTA 0 (trace build)
mkdir -p gpurun_out
timeout 600 python tools/tc_trace.py > gpurun_out/r2ay_trace.txt 2>&1
echo done
