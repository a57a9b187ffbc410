# round 2, call z: CTA-pair GEMM diagnosis (pipeline parts switched off)
mkdir -p gpurun_out
timeout 300 python tools/time_gemm_pair.py > gpurun_out/r2z_pair_dbg.txt 2>&1
echo done
